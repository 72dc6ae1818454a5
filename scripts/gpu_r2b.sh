#!/bin/bash
# Round-2 (second session) validation: smoke, full GPU suite, configs[3]-rows-on-one-GPU run, bench line.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -n 1 gpurun_out/smoke.log
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; tail -n 2 gpurun_out/pytest_gpu.log; grep -E "^(FAILED|ERROR)" gpurun_out/pytest_gpu.log | head
timeout 900 python scripts/c4_p1.py --n 4096 > gpurun_out/c4_p1.log 2>&1; tail -n 3 gpurun_out/c4_p1.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; python -c "import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['device_resident']['ms_per_step'], d['device_resident']['kernels']['leaf']['ms'])"
