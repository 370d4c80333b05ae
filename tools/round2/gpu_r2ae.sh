#!/bin/bash
# round 2, call ae: final state -- smoke, bench (default, the driver's command), ncu launch list +
# --set full of every group of the timed configuration, GPU suite
OUT=gpurun_out/r2ae
mkdir -p $OUT
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1
echo "smoke rc=$?" >> $OUT/summary.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh $OUT/bench.json $OUT/ncu
echo "ncu rc=$?" >> $OUT/summary.txt
timeout 1800 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
