#!/bin/bash
# round 2, call g: register limit per sub-partition (V8 Eq. 3), full GPU suite, default bench, unroll-2 bench
OUT=gpurun_out/r2g
mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --steps 20 --warmup 5 --unroll 2 --no-cpu --no-e2e > $OUT/bench_unroll2.json 2> $OUT/bench_unroll2.err
echo "bench unroll rc=$?" >> $OUT/summary.txt
