#!/bin/bash
# round 2, call a: new GPU tests, sanitizer re-run (slot-bounded canvas loads, scratch fills), default bench
OUT=gpurun_out/r2a
mkdir -p $OUT
nvidia-smi -L > $OUT/gpu.txt
timeout 1500 python -m pytest tests/test_gpu_round2.py -x -q > $OUT/pytest_round2.txt 2>&1
echo "round2 tests rc=$?" >> $OUT/summary.txt
tail -3 $OUT/pytest_round2.txt >> $OUT/summary.txt
CS=/usr/local/cuda/bin/compute-sanitizer
for w in "weather pairs" "weather points"; do
  tag=$(echo $w | tr ' ' '_')
  for tool in racecheck initcheck; do
    extra=""
    [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 900 $CS --tool $tool $extra --print-limit 20 python tools/round2/sanitize_run.py $w > $OUT/san_${tag}_${tool}.log 2>&1
    echo "$tag $tool rc=$?" >> $OUT/summary.txt
    tail -2 $OUT/san_${tag}_${tool}.log >> $OUT/summary.txt
  done
done
timeout 1200 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
