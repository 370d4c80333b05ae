#!/bin/bash
# round 2, call m: same-box A/B of the committed 5-group plan vs the 4-group plan of the new search
# objective; GPU suite
OUT=gpurun_out/r2m
mkdir -p $OUT
timeout 1200 python tools/round2/abt.py "$(cat tools/round2/abt_r2m.json)" > $OUT/abt.jsonl 2> $OUT/abt.err
timeout 2400 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.txt 2>&1
echo "pytest rc=$?" >> $OUT/summary.txt; tail -3 $OUT/pytest_gpu.txt >> $OUT/summary.txt
