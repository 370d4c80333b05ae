#!/bin/bash
# round 2, call ag: after the NEXT-2 refit (search objective changed): GPU suite, configs 2 and 5
OUT=gpurun_out/r2ag
mkdir -p $OUT
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
timeout 1200 python bench.py --workload suite --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench_suite.json 2> $OUT/bench_suite.err
echo "bench suite rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload stress --steps 5 --warmup 3 --no-cpu --no-e2e > $OUT/bench_stress.json 2> $OUT/bench_stress.err
echo "bench stress rc=$?" >> $OUT/summary.txt
