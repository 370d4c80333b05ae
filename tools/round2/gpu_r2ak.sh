#!/bin/bash
# round 2, call ak: config 2 every legal plan timed with the final executor (inline recompute,
# own-result carries) at the default launch configuration
OUT=gpurun_out/r2ak
mkdir -p $OUT
timeout 2400 python bench.py --workload suite --all-plans --steps 10 --warmup 3 > $OUT/suite_all_plans.json 2> $OUT/suite_all_plans.err
echo "all-plans rc=$?" >> $OUT/summary.txt
