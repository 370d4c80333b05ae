#!/bin/bash
# round 2, call ad: pair z-queue carries of the thread's own previous-plane results (z fluxes read
# at dz = -1) now taken whenever valid, vs the round-1 rectangle test; parity
OUT=gpurun_out/r2ad
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"rect test\", \"ghostwrite\": 0, \"env\": {\"KF_OWN_CARRY_RECT\": 1}}, {\"name\": \"own-result carries\", \"ghostwrite\": 0}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_round2.py -q -x -k "pairs or weather or per_group or suite or stress or inline" > $OUT/pytest_parity.txt 2>&1
echo "pytest parity rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_parity.txt >> $OUT/summary.txt
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x > $OUT/pytest_fullsize.txt 2>&1
echo "pytest fullsize rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_fullsize.txt >> $OUT/summary.txt
