#!/bin/bash
# Leaf iteration: leaf/dyadic tests, exchange diagnostics, leaf width sweep, bench.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -x -q -m gpu -k "leaf or dyadic or gaussian_vs or cgs2" > gpurun_out/pytest_gpu.log 2>&1
tail -n 3 gpurun_out/pytest_gpu.log
RGSQR_LEAF_DEBUG2=1 timeout 120 python scripts/prof_run.py --n 1024 2>&1 | grep leaf2 | tail -n 1
timeout 300 python scripts/sweep.py --opt leaf_width=32,64 2>&1 | tail -n 2
