#!/bin/bash
# ncu launch list (per-launch durations, cold-cache, serialised) of one device-resident c2 factorization.
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2_device.csv \
  python scripts/prof_run.py > gpurun_out/launches.log 2>&1
tail -n 2 gpurun_out/launches.log
python scripts/launch_summary.py gpurun_out/launches_c2_device.csv
