#!/bin/bash
# round 2, call j: bench of the committed configuration (plan auto) + ncu of exactly it; reference arm
OUT=gpurun_out/r2j
mkdir -p $OUT
timeout 1200 python bench.py --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
echo "bench rc=$?" >> $OUT/summary.txt
bash tools/round2/ncu_from_bench.sh $OUT/bench.json $OUT/ncu
echo "ncu rc=$?" >> $OUT/summary.txt
timeout 600 python bench.py --impl reference --steps 5 --warmup 1 > $OUT/reference.json 2> $OUT/reference.err
echo "reference rc=$?" >> $OUT/summary.txt
