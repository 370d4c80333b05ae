# Fill kernel rewrite (row/column threads, 32-bit indices): GPU tests, replayed bench of the s4
# plan and launch configs, launch list.
set -x
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 64], 3, 1, 0, -1, 1, 1, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s4b_pytest_gpu.log 2>&1; echo "pytest rc $?" >> gpurun_out/s4b_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s4b_smoke.log 2>&1; echo "smoke rc $?" >> gpurun_out/s4b_smoke.log
timeout 600 python bench.py --autotune 0 --plan "$PLAN" --tuned "$TUNED" --no-cpu > gpurun_out/s4b_bench_replay.json 2> gpurun_out/s4b_bench_replay.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s4b_launches.csv python bench.py --steps 3 --warmup 3 --autotune 0 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/s4b_ncu_bench.log 2>&1
timeout 900 python bench.py > gpurun_out/s4b_bench.json 2> gpurun_out/s4b_bench.err
