#!/bin/bash
# round 2, call t: programmatic dependent launches between the step's kernels (KF_PDL) vs plain
# launches, committed configuration, same box; wrapped-load GPU tests; GPU suite under KF_PDL=1
OUT=gpurun_out/r2t
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 9, \"variants\": [{\"name\": \"plain launches\", \"ghostwrite\": 0}, {\"name\": \"PDL\", \"ghostwrite\": 0, \"env\": {\"KF_PDL\": 1}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
timeout 900 python -m pytest tests/test_gpu_round2.py -q -k wrapload > $OUT/pytest_wrap.txt 2>&1
echo "pytest(wrap tests) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_wrap.txt >> $OUT/summary.txt
KF_PDL=1 timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu_pdl.txt 2>&1
echo "pytest(KF_PDL=1) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu_pdl.txt >> $OUT/summary.txt
