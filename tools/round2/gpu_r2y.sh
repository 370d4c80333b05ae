#!/bin/bash
# round 2, call y: partial canvas iterations (pipeline fill/drain at interior z-chunk boundaries on
# the canvas) vs the per-kernel slow path, committed configuration, same box; parity; racecheck
OUT=gpurun_out/r2y
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"slow path at chunk boundaries\", \"ghostwrite\": 0, \"env\": {\"KF_NO_PARTIAL\": 1}}, {\"name\": \"partial canvas iterations\", \"ghostwrite\": 0}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py -q -x -k "pairs or weather or per_group or suite or stress or inline" > $OUT/pytest_parity.txt 2>&1
echo "pytest parity rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_parity.txt >> $OUT/summary.txt
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x > $OUT/pytest_fullsize.txt 2>&1
echo "pytest fullsize rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_fullsize.txt >> $OUT/summary.txt
CS=/usr/local/cuda/bin/compute-sanitizer
for mode in pairs pairs_chunks; do
  for tool in racecheck synccheck; do
    extra=""; [ $tool = racecheck ] && extra="--racecheck-report all"
    timeout 600 $CS --tool $tool $extra --print-limit 50 python tools/round2/sanitize_run.py weather $mode > $OUT/san_weather_${mode}_${tool}.log 2>&1
    echo "sanitize $mode $tool rc=$?" >> $OUT/summary.txt; tail -2 $OUT/san_weather_${mode}_${tool}.log >> $OUT/summary.txt
  done
done
