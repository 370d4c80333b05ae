#!/bin/bash
# round 2, call r (session 3 start): state check of the restored checkpoint -- smoke, bench, GPU suite
OUT=gpurun_out/r2r
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1
echo "smoke rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
