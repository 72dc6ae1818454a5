#!/bin/bash
# One gpurun call: GPU tests, smoke, bench, leaf phase breakdown.  Output under gpurun_out/.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err
RGSQR_LEAF_DEBUG=0 timeout 120 python scripts/prof_run.py --n 1024 > gpurun_out/leafdbg.log 2>&1
tail -3 gpurun_out/pytest_gpu.log gpurun_out/smoke.log; cat gpurun_out/bench.json; grep "cycles/round" gpurun_out/leafdbg.log | sort | uniq -c | head
