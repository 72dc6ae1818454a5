#!/bin/bash
# A/B (bitwise + wall) of the previous and current builds, split-K scan, GPU suite, bench.
mkdir -p gpurun_out
for so in paper_conf_icpp_zhangw21_b200/librgsqr_prev.so paper_conf_icpp_zhangw21_b200/librgsqr.so; do
  timeout 300 python scripts/bitcheck.py $so 2>&1 | grep -v Warn | tail -1
done
bash scripts/gpu_splitk.sh 2>&1 | grep -E "rgsqr" | head -2
bash scripts/gpu_splitk.sh 2>&1 | grep -E "\(4, 2," | head -2
timeout 1200 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -n 1 gpurun_out/pytest_gpu.log; grep -E "^FAILED" gpurun_out/pytest_gpu.log | head
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; tail -n 1 gpurun_out/bench.log | cut -c1-200
