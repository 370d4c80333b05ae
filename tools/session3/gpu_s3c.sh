PLAN='[0, 0, 0, 1, 1, 1, 1, 1, 1, 0, 0, 0, 0, 2, 2, 2, 2, 0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 3, 2, 2, 4, 4, 2, 3, 3, 4, 4, 3, 3, 3, 4, 4, 3, 3]'
python tools/ab.py '[{"tile":[32,8,64],"minblocks":-1},{"tile":[32,8,64],"minblocks":-1,"env":{"KF_PRODUCER0":"1"}},{"tile":[32,8,64],"minblocks":0},{"tile":[32,8,32],"minblocks":-1}]' "$PLAN" > gpurun_out/ab3.jsonl 2> gpurun_out/ab3.err
