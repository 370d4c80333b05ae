#!/bin/bash
# round 2, call u: L2 prefetch of the TMA boxes D planes ahead (KF_L2PF=D) vs none, committed
# configuration, same box, alternating rounds
OUT=gpurun_out/r2u
mkdir -p $OUT
PLAN=$(python -c "import json;print(json.load(open('profiles/bench_timed_config.json'))['plan_labels'])")
TUNED=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 1200 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"no L2 prefetch\", \"ghostwrite\": 0}, {\"name\": \"L2 prefetch D=1\", \"ghostwrite\": 0, \"env\": {\"KF_L2PF\": 1}}, {\"name\": \"L2 prefetch D=2\", \"ghostwrite\": 0, \"env\": {\"KF_L2PF\": 2}}, {\"name\": \"L2 prefetch D=4\", \"ghostwrite\": 0, \"env\": {\"KF_L2PF\": 4}}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
echo "abt rc=$?" >> $OUT/summary.txt
