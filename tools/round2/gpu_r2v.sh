#!/bin/bash
# round 2, call v: inline recompute of in-group xy-offset reads in the pair canvas (KF_INLINE=1)
# vs shared-memory intermediates, committed configuration, same box; parity under KF_INLINE=1
OUT=gpurun_out/r2v
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"smem intermediates\", \"ghostwrite\": 0}, {\"name\": \"inline recompute\", \"ghostwrite\": 0, \"env\": {\"KF_INLINE\": 1}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
KF_INLINE=1 timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "pairs or weather or suite or stress or per_group" > $OUT/pytest_parity_inline.txt 2>&1
echo "pytest parity(inline) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_parity_inline.txt >> $OUT/summary.txt
KF_INLINE=1 timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x > $OUT/pytest_fullsize_inline.txt 2>&1
echo "pytest fullsize(inline) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_fullsize_inline.txt >> $OUT/summary.txt
