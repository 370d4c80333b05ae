#!/bin/bash
# round 2, call b: ghost copies as a CTA epilogue -- bench A/B against fills, full GPU suite
OUT=gpurun_out/r2b
mkdir -p $OUT
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e --fills > $OUT/bench_fills.json 2> $OUT/bench_fills.err
echo "bench fills rc=$?" >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt
tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
