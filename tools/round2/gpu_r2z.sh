#!/bin/bash
# round 2, call z: bench of the new committed configuration (4 groups, inline recompute), the
# previous committed configuration on the same box, and ncu evidence of the new one
OUT=gpurun_out/r2z
mkdir -p $OUT
timeout 900 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
P=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['plan_labels']))")
T=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['per_group_launch_config']))")
timeout 900 python bench.py --steps 20 --warmup 5 --plan "$P" --tuned "$T" --no-cpu --no-e2e > $OUT/bench_prev.json 2> $OUT/bench_prev.err
echo "bench prev rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh $OUT/bench.json $OUT/ncu
echo "ncu rc=$?" >> $OUT/summary.txt
