#!/bin/bash
# round 2, call o: ncu of the suite (config 2) and stress (config 5) timed configurations
OUT=gpurun_out/r2o
mkdir -p $OUT
bash tools/round2/ncu_from_bench.sh profiles/round2_n_bench_suite.json $OUT/ncu_suite "--workload suite"
echo "suite ncu rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh profiles/round2_h_bench_stress.json $OUT/ncu_stress "--workload stress"
echo "stress ncu rc=$?" >> $OUT/summary.txt
