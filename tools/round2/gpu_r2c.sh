#!/bin/bash
# round 2, call c: V8 register budget (R_est as __maxnreg__), frozen-only scratch fills; resource pin,
# full GPU suite, bench (ghost writes vs fills)
OUT=gpurun_out/r2c
mkdir -p $OUT
timeout 2400 python -m pytest tests/test_gpu_resource_pin.py -q -x > $OUT/pytest_resource_pin.txt 2>&1
echo "resource pin rc=$?" >> $OUT/summary.txt
tail -3 $OUT/pytest_resource_pin.txt >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -q --deselect tests/test_gpu_resource_pin.py > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt
tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e --fills > $OUT/bench_fills.json 2> $OUT/bench_fills.err
echo "bench fills rc=$?" >> $OUT/summary.txt
