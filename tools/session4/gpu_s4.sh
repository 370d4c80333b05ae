# Session-4 validation of the committed build: GPU tests, smoke, bench line, reference arm,
# launch list of the timed configuration.
set -x
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s4_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/s4_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s4_smoke.log 2>&1; echo "smoke rc $?" >> gpurun_out/s4_smoke.log
timeout 900 python bench.py > gpurun_out/s4_bench.json 2> gpurun_out/s4_bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/s4_bench_ref.json 2> gpurun_out/s4_bench_ref.err
PLAN=$(python -c "import json; print(json.dumps(json.load(open('gpurun_out/s4_bench.json'))['config']['plan_labels']))")
TUNED=$(python -c "import json; print(json.dumps(json.load(open('gpurun_out/s4_bench.json'))['config']['per_group_launch_config']))")
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s4_launches.csv python bench.py --steps 3 --warmup 3 --autotune 0 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/s4_ncu_bench.log 2>&1
