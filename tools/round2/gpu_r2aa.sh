#!/bin/bash
# round 2, call aa: ncu evidence of the committed configuration with inline recompute (launch list
# + --set full of every group), and configs 2 (suite) / 5 (stress) benches under inline
OUT=gpurun_out/r2aa
mkdir -p $OUT
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh $OUT/bench.json $OUT/ncu
echo "ncu rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --workload suite --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench_suite.json 2> $OUT/bench_suite.err
echo "bench suite rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload stress --steps 5 --warmup 3 --no-cpu --no-e2e > $OUT/bench_stress.json 2> $OUT/bench_stress.err
echo "bench stress rc=$?" >> $OUT/summary.txt
