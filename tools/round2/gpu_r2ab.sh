#!/bin/bash
# round 2, call ab: parity leg reading windows (and device-generated crops) from the device: weather
# bench, stress (config 5) and weak (config 4, N = 1) benches now carry parity; GPU suite
OUT=gpurun_out/r2ab
mkdir -p $OUT
timeout 900 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload stress --steps 5 --warmup 3 --no-cpu --no-e2e > $OUT/bench_stress.json 2> $OUT/bench_stress.err
echo "bench stress rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --workload weak --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/bench_weak.json 2> $OUT/bench_weak.err
echo "bench weak rc=$?" >> $OUT/summary.txt
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
