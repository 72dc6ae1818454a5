#!/bin/bash
# ncu full capture (with source) of one leaf launch at m = 65536, w = 64.
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:leaf_cgs -s 6 -c 1 \
  -o gpurun_out/leaf_full -f python scripts/prof_run.py --n 1024 > gpurun_out/ncu_leaf.log 2>&1
tail -n 5 gpurun_out/ncu_leaf.log
