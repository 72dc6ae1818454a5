#!/bin/bash
# Leaf iteration: leaf/dyadic tests, exchange diagnostics, phase breakdown, leaf width sweep.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -x -q -m gpu -k "leaf or dyadic or gaussian_vs or cgs2 or kernels" > gpurun_out/pytest_gpu.log 2>&1
tail -n 3 gpurun_out/pytest_gpu.log; grep -E "Error|assert|FAIL" gpurun_out/pytest_gpu.log | head -20
RGSQR_LEAF_DEBUG2=1 timeout 120 python scripts/prof_run.py --n 1024 2>&1 | grep leaf2 | tail -n 1
RGSQR_LEAF_DEBUG=5 timeout 120 python scripts/prof_run.py --n 1024 2>&1 | grep "cycles/round" | tail -n 1
timeout 300 python scripts/sweep.py --opt leaf_width=64 2>&1 | tail -n 1
