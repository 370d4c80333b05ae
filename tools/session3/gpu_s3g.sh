PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 64], 3, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 1, -1, 1]]'
for i in 1 2; do
python bench.py --steps 50 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/fill_batched_$i.json 2>>gpurun_out/fill.err
KF_FILL_SINGLE=1 python bench.py --steps 50 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/fill_single_$i.json 2>>gpurun_out/fill.err
done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests6.log 2>&1; echo tests=$? >> gpurun_out/gpu_tests6.log
