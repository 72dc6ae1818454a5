#!/bin/bash
# Full GPU suite + paper-shape runs (c3 recursive vs blocked) with the current code.
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -n 2 gpurun_out/pytest_gpu.log; grep -E "^FAILED" gpurun_out/pytest_gpu.log | head -20
timeout 1500 python scripts/paper_runs.py --which c3 --out gpurun_out/paper_runs_c3.json > gpurun_out/paper_runs_c3.log 2>&1
tail -n 4 gpurun_out/paper_runs_c3.log
