#!/bin/bash
# compute-sanitizer over small fused runs (tools/round2/sanitize_run.py); logs -> gpurun_out/sanitize/
set -x
OUT=gpurun_out/sanitize
mkdir -p $OUT
nvidia-smi -L > $OUT/gpu.txt
CS=/usr/local/cuda/bin/compute-sanitizer
for w in "tiny pairs" "weather pairs" "weather points"; do
  tag=$(echo $w | tr ' ' '_')
  for tool in racecheck synccheck initcheck memcheck; do
    extra=""
    [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 900 $CS --tool $tool $extra --print-limit 50 python tools/round2/sanitize_run.py $w > $OUT/${tag}_${tool}.log 2>&1
    echo "$tag $tool rc=$?" >> $OUT/summary.txt
    tail -3 $OUT/${tag}_${tool}.log >> $OUT/summary.txt
  done
done
