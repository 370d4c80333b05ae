#!/bin/bash
# round 2, call af: ghost-fill spans of 64 bytes (KF_FILL_SPAN=64) vs 32-byte sectors, committed
# configuration, same box, 9 alternating rounds; parity of the periodic programs under 64-byte spans
OUT=gpurun_out/r2af
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 9, \"variants\": [{\"name\": \"32-byte fill spans\", \"ghostwrite\": 0}, {\"name\": \"64-byte fill spans\", \"ghostwrite\": 0, \"env\": {\"KF_FILL_SPAN\": 64}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
KF_FILL_SPAN=64 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "weather or suite or stress or random or full" > $OUT/pytest_span64.txt 2>&1
echo "pytest(span 64) rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_span64.txt >> $OUT/summary.txt
