V='[{"tile":[32,8,64]},{"tile":[32,8,64],"stages":3},{"tile":[32,8,64],"stages":4},{"tile":[64,8,64]},{"tile":[64,8,64],"stages":3},{"tile":[32,16,64]},{"tile":[64,16,64]},{"tile":[128,4,64]},{"tile":[64,4,0],"stages":4},{"tile":[32,8,32],"stages":3},{"tile":[64,8,0],"stages":3},{"tile":[32,8,64],"zunroll":2},{"tile":[64,8,64],"zunroll":2,"stages":2}]'
python tools/ab.py "$V" unfused suite > gpurun_out/ab_suite_unf.jsonl 2> gpurun_out/ab_suite.err
python tools/ab.py "$V" best suite > gpurun_out/ab_suite_best.jsonl 2>> gpurun_out/ab_suite.err
