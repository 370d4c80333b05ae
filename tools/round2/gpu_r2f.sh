#!/bin/bash
# round 2, call f: clamped loads (per-iteration bases), register fallback at R_est, V8 Eq. 3, sector fills
OUT=gpurun_out/r2f
mkdir -p $OUT
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
T1='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
P0='{"0": [[32, 8, 32], 2, 1, 0, -1, 0, 2, 0], "1": [[32, 8, 43], 2, 1, 0, -1, 0, 2, 1], "2": [[32, 8, 43], 2, 1, 0, -1, 0, 2, 1], "3": [[32, 8, 32], 2, 1, 0, -1, 0, 2, 0], "4": [[32, 8, 32], 2, 1, 0, -1, 0, 2, 0], "5": [[32, 8, 64], 3, 1, 0, -1, 0, 1, 1]}'
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $T1, \"rounds\": 5, \"variants\": [{\"name\": \"clamped sectorfill\", \"ghostwrite\": 0}, {\"name\": \"predicated sectorfill\", \"ghostwrite\": 0, \"override\": $P0}, {\"name\": \"clamped cellfill\", \"ghostwrite\": 0, \"env\": {\"KF_FILL_CELLS\": 1}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
CS=/usr/local/cuda/bin/compute-sanitizer
for w in "weather pairs" "weather points"; do
  tag=$(echo $w | tr ' ' '_')
  for tool in racecheck initcheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 900 $CS --tool $tool $extra --print-limit 20 python tools/round2/sanitize_run.py $w > $OUT/san_${tag}_${tool}.log 2>&1
    echo "$tag $tool rc=$?" >> $OUT/summary.txt; tail -2 $OUT/san_${tag}_${tool}.log >> $OUT/summary.txt
  done
done
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
