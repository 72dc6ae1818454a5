#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
  (cd build_alt/r1src && timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed 's/^/r1: /')
  timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed 's/^/r2: /'
done
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -q -k "tf32x3 or inner or outer" 2>&1 | tail -n 2
