#!/bin/bash
# Quick GPU iteration: kernel tests, leaf phase breakdown, bench (no cpu baseline).
mkdir -p gpurun_out
timeout 600 python -m pytest tests -x -q -m gpu ${PYTEST_K} > gpurun_out/pytest_gpu.log 2>&1
RGSQR_LEAF_DEBUG=5 timeout 120 python scripts/prof_run.py --n 1024 > gpurun_out/leafdbg.log 2>&1
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -n 5 gpurun_out/pytest_gpu.log; grep "cycles/round" gpurun_out/leafdbg.log | tail -n 2; python - <<'PY'
import json
try:
    d = json.loads(open("gpurun_out/bench.json").read().strip().splitlines()[-1])
    print("value", round(d["value"], 1), "ms", round(d["ms_per_step"], 2), "e2e", round(d["e2e"]["value"], 1), d["e2e"]["ms_per_step"], "frac", round(d["e2e"]["roofline_frac"], 3))
    print({k: (round(v["ms"], 2), v["launches"]) for k, v in d["kernels"].items()})
except Exception as e:
    print("bench parse failed", e); print(open("gpurun_out/bench.err").read()[-2000:])
PY
