#!/bin/bash
# OOC (host-resident) c2 run with the per-stream timeline dumped; occupancy in 1 ms buckets.
mkdir -p gpurun_out
RGSQR_TIMELINE=gpurun_out/tl.csv timeout 300 python scripts/prof_run.py --host --reps 3 ${PROF_ARGS} > gpurun_out/tl_stats.log 2>&1
tail -c 1500 gpurun_out/tl_stats.log
python scripts/timeline.py gpurun_out/tl.csv 1.0
