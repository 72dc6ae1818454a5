#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -n 2 gpurun_out/pytest_gpu.log; grep -E "^FAILED|Error|assert" gpurun_out/pytest_gpu.log | head -20
timeout 300 python scripts/sweep.py --opt fuse_small=0,1 2>&1 | tail -n 2
timeout 300 python scripts/sweep.py --prec bf16 --opt fuse_small=0,1 2>&1 | tail -n 2
