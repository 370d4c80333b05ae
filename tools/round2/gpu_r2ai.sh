#!/bin/bash
# round 2, call ai: re-autotune (after own-result carries) the committed plan's per-group launch configurations under inline
# recompute, against the committed configuration on the same box
OUT=gpurun_out/r2ai
mkdir -p $OUT
P=$(python -c "import json;print(json.dumps(json.load(open('profiles/bench_timed_config.json'))['plan_labels']))")
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
timeout 1800 python bench.py --plan "$P" --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench_retune.json 2> $OUT/bench_retune.err
echo "bench retune rc=$?" >> $OUT/summary.txt
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e > $OUT/bench2.json 2> $OUT/bench2.err
echo "bench again rc=$?" >> $OUT/summary.txt
