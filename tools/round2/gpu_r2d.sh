#!/bin/bash
# round 2, call d: A/B ghost-write epilogue vs fills; slot-bounded vs round-1 unpredicated loads; ncu of g0 both ways
OUT=gpurun_out/r2d
mkdir -p $OUT
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
T1='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
T2='[[[32, 8, 64], 2, 1, 0, 0, 1, 1, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1]]'
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $T1, \"rounds\": 5, \"variants\": [{\"name\": \"r1cfg fills\", \"ghostwrite\": 0}, {\"name\": \"r1cfg gw\", \"ghostwrite\": 1}, {\"name\": \"r1cfg fills anyring\", \"ghostwrite\": 0, \"env\": {\"KF_LD_ANYRING\": 1}}, {\"name\": \"r1cfg gw anyring\", \"ghostwrite\": 1, \"env\": {\"KF_LD_ANYRING\": 1}}]}" > $OUT/abt1.jsonl 2> $OUT/abt1.err
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $T2, \"rounds\": 5, \"variants\": [{\"name\": \"r2cfg fills\", \"ghostwrite\": 0}, {\"name\": \"r2cfg gw\", \"ghostwrite\": 1}]}" > $OUT/abt2.jsonl 2> $OUT/abt2.err
for gw in 0 1; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_g0 -c 1 -o $OUT/g0_gw$gw python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $T2, \"rounds\": 1, \"steps\": 1, \"variants\": [{\"name\": \"x\", \"ghostwrite\": $gw}]}" > $OUT/ncu_gw$gw.log 2>&1
done
