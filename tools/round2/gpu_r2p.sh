#!/bin/bash
# round 2, call p: retune the committed plan with the new tile candidates; GPU suite
OUT=gpurun_out/r2p
mkdir -p $OUT
timeout 1500 python bench.py --plan '[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 3, 4, 1, 4, 4, 3, 4, 3, 4, 4, 3, 4, 3, 4]' --steps 20 --warmup 5 --no-cpu > $OUT/bench_retune.json 2> $OUT/bench_retune.err
echo "retune rc=$?" >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
