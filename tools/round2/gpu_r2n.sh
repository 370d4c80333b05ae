#!/bin/bash
# round 2, call n: re-tune the committed plan with the 3-stage pair candidates; suite ncu; stress near-limit plan
OUT=gpurun_out/r2n
mkdir -p $OUT
timeout 1500 python bench.py --plan '[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 3, 4, 1, 4, 4, 3, 4, 3, 4, 4, 3, 4, 3, 4]' --steps 20 --warmup 5 --no-cpu > $OUT/bench_retune.json 2> $OUT/bench_retune.err
echo "retune rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --workload suite --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench_suite.json 2> $OUT/bench_suite.err
bash tools/round2/ncu_from_bench.sh $OUT/bench_suite.json $OUT/ncu_suite
echo "suite rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload stress --plan '[0,0,0,1,1,1]' --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/bench_stress_perfield.json 2> $OUT/bench_stress_perfield.err
echo "stress per-field rc=$?" >> $OUT/summary.txt
