#!/bin/bash
# round 2, call ah: NEXT-3 test-suite sweep (Table V ranges, Fig. 9-style speedups) with the round-2
# executor (canvas pairs, z-queues, clamped loads, inline recompute), same parameters as round 1
OUT=gpurun_out/r2ah
mkdir -p $OUT
timeout 2400 python tools/suite_sweep.py > $OUT/suite_sweep.jsonl 2> $OUT/suite_sweep.err
echo "sweep rc=$?" >> $OUT/summary.txt
