#!/bin/bash
# round 2, call x: bench of the committed configuration with inline recompute (default), a fresh
# measured plan selection + autotune under inline, and the whole GPU suite
OUT=gpurun_out/r2x
mkdir -p $OUT
timeout 900 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --steps 20 --warmup 5 --plan select --no-cpu > $OUT/bench_select.json 2> $OUT/bench_select.err
echo "bench select rc=$?" >> $OUT/summary.txt
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
