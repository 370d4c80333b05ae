#!/bin/bash
# ncu evidence of the exact configuration a bench JSON timed: launch list (gpu__time_duration of
# every kernel of 2 steps) and one --set full capture of every group kernel.
# usage: tools/round2/ncu_from_bench.sh <bench.json> <outdir> [extra bench args, e.g. --workload suite]
J=$1; OUT=$2; EXTRA=$3
mkdir -p $OUT
PLAN=$(python -c "import json,sys;print(json.dumps(json.load(open('$J'))['config']['plan_labels']))")
TUNED=$(python -c "import json,sys;print(json.dumps(json.load(open('$J'))['config']['per_group_launch_config']))")
NG=$(python -c "import json,sys;print(len(json.load(open('$J'))['config']['per_group_launch_config']))")
ARGS="$EXTRA --plan \"$PLAN\" --tuned \"$TUNED\" --steps 2 --warmup 3 --no-unfused --no-e2e --no-cpu --no-parity"
eval timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches.csv python bench.py $ARGS > $OUT/launches.log 2>&1
eval timeout 1500 ncu --set full --clock-control none --import-source on -k regex:kf_g -c $NG -o $OUT/groups python bench.py $ARGS > $OUT/full.log 2>&1
