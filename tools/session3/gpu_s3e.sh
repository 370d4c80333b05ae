PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 0, 0, 0, 0, 2, 2, 2, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 2, 3, 3, 4, 4, 3, 3, 3, 4, 4, 3, 3]'
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kf_g -c 5 -o gpurun_out/prof_s3e python tools/prof_plan.py "$PLAN" '{"tile":[32,8,64],"minblocks":-1}' 1 > gpurun_out/ncu_s3e.log 2>&1
