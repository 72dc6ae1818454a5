#!/bin/bash
# ncu full captures of the fused bottom node and of a short-K (w1 = 256) NN outer product.
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none -k regex:small_node -s 3 -c 1 -o gpurun_out/small_full -f \
  python scripts/prof_run.py --n 1024 > gpurun_out/ncu_small.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:nn_kernel -s 2 -c 1 -o gpurun_out/nn128_full -f \
  python scripts/prof_run.py --n 1024 > gpurun_out/ncu_nn.log 2>&1
tail -n 1 gpurun_out/ncu_small.log gpurun_out/ncu_nn.log
