PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 2, 2, 2, 2, 2, 2, 0, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 3, 5, 5, 4, 4, 3, 5, 5, 4, 4, 3, 5]'
V='[{"tile":[32,8,64],"minblocks":-1,"pblock":[2,1],"canvas_ld":0}]'
for st in 6 50 200 6; do AB_STEPS=$st python tools/ab.py "$V" "$PLAN" > gpurun_out/ab7_$st.jsonl 2>/dev/null; done
nvidia-smi -q -d PERFORMANCE,POWER,CLOCK > gpurun_out/smi_q.txt 2>&1
TUNED='[[[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 2, 1, 0, -1, 0, 2, 1], [[32, 8, 64], 2, 1, 0, 0, 1, 2, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 1, 1], [[32, 8, 32], 2, 1, 0, -1, 1, 2, 0], [[32, 8, 64], 3, 1, 0, -1, 1, 1, 1]]'
for st in 10 50 200; do python bench.py --steps $st --plan "$PLAN" --tuned "$TUNED" --no-unfused --no-e2e --no-cpu > gpurun_out/b7_$st.json 2>/dev/null; done
