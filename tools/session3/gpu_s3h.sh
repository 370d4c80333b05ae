PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 64], 3, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 1, -1, 1]]'
for i in 1 2; do
python bench.py --steps 50 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/rot_$i.json 2>>gpurun_out/rot.err
KF_SLOT_COUNTERS=1 python bench.py --steps 50 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/cnt_$i.json 2>>gpurun_out/rot.err
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/gpu_tests7.log 2>&1; echo tests=$? >> gpurun_out/gpu_tests7.log
