#!/bin/bash
# Final evidence of the round-2 build: bench line, launch lists (device + host path), full ncu capture of the leaf.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; python -c "import json; d=json.load(open('gpurun_out/bench_final.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['device_resident']['ms_per_step'], d['device_resident']['kernels']['leaf']['ms'], d['clocks'])"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dev_final.csv python scripts/prof_run.py > gpurun_out/launches_dev_final.log 2>&1; python scripts/launch_summary.py gpurun_out/launches_dev_final.csv > gpurun_out/launches_dev_final_summary.md; head -8 gpurun_out/launches_dev_final_summary.md
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_host_final.csv python scripts/prof_run.py --host > gpurun_out/launches_host_final.log 2>&1; python scripts/launch_summary.py gpurun_out/launches_host_final.csv > gpurun_out/launches_host_final_summary.md; head -4 gpurun_out/launches_host_final_summary.md
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_cgs -s 20 -c 1 -o gpurun_out/prof_leaf_final python scripts/prof_run.py > gpurun_out/ncu_leaf_final.log 2>&1; tail -n 1 gpurun_out/ncu_leaf_final.log
ncu -i gpurun_out/prof_leaf_final.ncu-rep --page raw --csv > gpurun_out/prof_leaf_final_raw.csv 2>/dev/null; wc -l gpurun_out/prof_leaf_final_raw.csv
