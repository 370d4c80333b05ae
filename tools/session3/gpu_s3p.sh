PLAN='[0, 0, 0, 0, 0, 1, 1, 0, 2, 2]'
V='[{"tile":[64,4,64]},{"tile":[64,8,64]},{"tile":[32,16,64]},{"tile":[64,16,64]},{"tile":[32,32,64]},{"tile":[128,8,64]},{"tile":[64,8,64],"pblock":[2,1]},{"tile":[64,16,64],"pblock":[2,1]},{"tile":[32,16,64],"pblock":[2,1]},{"tile":[64,8,64],"zunroll":2},{"tile":[64,16,64],"minblocks":-1},{"tile":[128,16,64],"pblock":[2,1]}]'
AB_STEPS=10 python tools/ab.py "$V" "$PLAN" suite > gpurun_out/ab10.jsonl 2> gpurun_out/ab10.err
