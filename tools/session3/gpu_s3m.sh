timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "canvas" > gpurun_out/gpu_tests14.log 2>&1; echo tests=$? >> gpurun_out/gpu_tests14.log
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 64], 2, 1, 0, 0, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 1, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
for i in 1 2; do python bench.py --steps 10 --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/b8_$i.json 2>/dev/null; done
