#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:small_node -s 3 -c 1 \
  -o gpurun_out/small_full -f python scripts/prof_run.py --n 1024 > gpurun_out/ncu_small.log 2>&1
tail -n 2 gpurun_out/ncu_small.log
