#!/bin/bash
# round 2, call h: GPU suite, default bench + ncu of its configuration, config 2 all plans, configs 2/4/5
OUT=gpurun_out/r2h
mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
timeout 1200 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh $OUT/bench.json $OUT/ncu
echo "ncu rc=$?" >> $OUT/summary.txt
timeout 1800 python bench.py --workload suite --all-plans --steps 10 --warmup 3 > $OUT/suite_all_plans.json 2> $OUT/suite_all_plans.err
echo "all-plans rc=$?" >> $OUT/summary.txt
timeout 1200 python bench.py --workload suite --steps 20 --warmup 5 --no-cpu > $OUT/bench_suite.json 2> $OUT/bench_suite.err
echo "suite rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload stress --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/bench_stress.json 2> $OUT/bench_stress.err
echo "stress rc=$?" >> $OUT/summary.txt
timeout 1500 python bench.py --workload weak --steps 10 --warmup 3 --no-cpu --no-e2e > $OUT/bench_weak.json 2> $OUT/bench_weak.err
echo "weak rc=$?" >> $OUT/summary.txt
