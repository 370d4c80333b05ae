#!/bin/bash
# round 2, call q: ghost copies per iteration by the producer (noinline copy, sector-wide x images)
# vs ghost-fill launches, same box; GPU suite
OUT=gpurun_out/r2q
mkdir -p $OUT
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 3, 4, 1, 4, 4, 3, 4, 3, 4, 4, 3, 4, 3, 4]'
TUNED='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 64], 2, 1, 0, -1, 0, 2, 1]]'
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 7, \"variants\": [{\"name\": \"fills\", \"ghostwrite\": 0}, {\"name\": \"ghost copies by the producer\", \"ghostwrite\": 1}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
