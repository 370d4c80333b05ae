# Full ncu capture of the group kernels in the configuration of round1_s4_bench_final.json.
set -x
PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
TUNED='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 43], 2, 1, 0, -1, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
timeout 840 ncu --set full --clock-control none --import-source on -k regex:kf_g -c 6 -o gpurun_out/s4f_prof python tools/prof_plan.py "$PLAN" '{"tile":[32,8,64]}' 1 "$TUNED" > gpurun_out/s4f_prof.log 2>&1
