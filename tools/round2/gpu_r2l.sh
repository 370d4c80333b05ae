#!/bin/bash
# round 2, call l: in-group ring alignment A/B (odd pitch reverted), search objective min(points,
# pairs); SHFL vs LDS microbenchmark; re-selection bench; GPU suite
OUT=gpurun_out/r2l
mkdir -p $OUT
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 3, 4, 1, 4, 4, 3, 4, 3, 4, 4, 3, 4, 3, 4]'
TUNED='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 64], 2, 1, 0, -1, 0, 2, 1]]'
nvcc -arch=sm_100a -O3 -o /tmp/shfl_vs_lds tools/round2/shfl_vs_lds.cu && /tmp/shfl_vs_lds > $OUT/shfl_vs_lds.txt 2>&1
timeout 900 python tools/round2/abt.py "{\"plan\": $PLAN, \"tuned\": $TUNED, \"rounds\": 5, \"variants\": [{\"name\": \"legacy in-group origins\", \"ghostwrite\": 0, \"env\": {\"KF_RING_LEGACY\": 1}}, {\"name\": \"aligned in-group origins\", \"ghostwrite\": 0}]}" > $OUT/abt.jsonl 2> $OUT/abt.err
timeout 1500 python bench.py --plan select --steps 20 --warmup 5 --no-cpu > $OUT/bench_select.json 2> $OUT/bench_select.err
echo "bench select rc=$?" >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
