PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 64], 3, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 64], 2, 1, 0, -1, 0], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 32], 2, 1, 0, -1, 1], [[32, 8, 64], 2, 1, 1, -1, 1]]'
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_g -c 6 -o gpurun_out/prof_s3f python tools/prof_plan.py "$PLAN" '{"tile":[32,8,64]}' 1 "$TUNED" > gpurun_out/ncu_s3f.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_s3f.csv python bench.py --steps 3 --warmup 3 --autotune 0 --plan best --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/b_ncu.log 2>&1
