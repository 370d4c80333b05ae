#!/bin/bash
# round 2, call w: inline recompute with two levels (values read only at offset 0 as inputs of
# inlined values: g0's flux producers read VELX computed in the group), per-group on/off, same box
OUT=gpurun_out/r2w
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
G0OFF=$(python -c "import json;c=json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config'][0];print(json.dumps(c+[0]))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"no inline\", \"ghostwrite\": 0, \"env\": {\"KF_INLINE\": 0}}, {\"name\": \"inline, two levels\", \"ghostwrite\": 0}, {\"name\": \"inline, g0 off\", \"ghostwrite\": 0, \"override\": {\"0\": $G0OFF}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "pairs or weather or per_group" > $OUT/pytest_parity.txt 2>&1
echo "pytest parity rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_parity.txt >> $OUT/summary.txt
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x > $OUT/pytest_fullsize.txt 2>&1
echo "pytest fullsize rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_fullsize.txt >> $OUT/summary.txt
