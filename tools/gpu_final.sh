# Final measurement of a round: bench line, then the launch list and a full ncu capture of the
# exact timed configuration (plan and per-group launch configs read back from the bench line).
set -x
SECONDS=0
timeout 900 python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err
echo "bench wall s: $SECONDS" > gpurun_out/final_bench_wall.txt
PLAN=$(python -c "import json; print(json.dumps(json.load(open('gpurun_out/final_bench.json'))['config']['plan_labels']))")
TUNED=$(python -c "import json; print(json.dumps(json.load(open('gpurun_out/final_bench.json'))['config']['per_group_launch_config']))")
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final_launches.csv python bench.py --steps 3 --warmup 3 --autotune 0 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/final_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_g -c 8 -o gpurun_out/final_prof python tools/prof_plan.py "$PLAN" '{"tile":[32,8,64]}' 1 "$TUNED" > gpurun_out/final_prof.log 2>&1
for w in suite stress; do timeout 900 python bench.py --workload $w --steps 20 --no-e2e > gpurun_out/final_bench_$w.json 2> gpurun_out/final_bench_$w.err; done
