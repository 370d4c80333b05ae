#!/bin/bash
# round 2, call s: wrapped edge-tile loads (kf_target.wrapload: no periodic ghost fills) vs fills,
# committed configuration, same box; GPU suite with KF_WRAPLOAD=1 (parity of every plan under wrap)
OUT=gpurun_out/r2s
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"fills\", \"ghostwrite\": 0}, {\"name\": \"wrapped loads\", \"ghostwrite\": 0, \"target\": {\"wrapload\": 1}}, {\"name\": \"wrapped loads, g1 minblocks 0\", \"ghostwrite\": 0, \"target\": {\"wrapload\": 1}, \"override\": {\"1\": [[32, 8, 43], 2, 1, 0, 0, 1, 2, 1]}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
KF_WRAPLOAD=1 timeout 2400 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_wrap.txt 2>&1
echo "pytest(wrap) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu_wrap.txt >> $OUT/summary.txt
