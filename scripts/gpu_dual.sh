#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do for dp in 0 1; do
  RGSQR_LEAF_DUAL_POLL=$dp timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed "s/^/dual=$dp: /"
done; done
RGSQR_LEAF_DUAL_POLL=1 timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -q -x 2>&1 | tail -n 2
