#!/bin/bash
# round 2, call i: register cap ladder, row-wise shell copy; fills overlapped with interior tiles
# (loopback kf_dist over one part) vs plain fills; GPU suite; bench
OUT=gpurun_out/r2i
mkdir -p $OUT
PLAN='[0, 0, 0, 0, 0, 0, 0, 0, 0, 1, 1, 2, 1, 1, 1, 1, 1, 2, 2, 2, 2, 0, 0, 0, 0, 1, 1, 3, 1, 1, 4, 4, 2, 3, 3, 4, 4, 3, 3, 3, 4, 4, 3, 3]'
TUNED='[[[32, 8, 43], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 2, 1, 0, 0, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 64], 2, 1, 0, 0, 0, 1, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1]]'
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 5, \"variants\": [{\"name\": \"fills\", \"ghostwrite\": 0}, {\"name\": \"fills overlapped (dist loopback)\", \"ghostwrite\": 0, \"dist\": 1}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
