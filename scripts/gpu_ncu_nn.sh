#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nn_kernel -s 2 -c 3 -o gpurun_out/prof_nn128 python scripts/prof_run.py > gpurun_out/ncu_nn.log 2>&1; tail -n 2 gpurun_out/ncu_nn.log
