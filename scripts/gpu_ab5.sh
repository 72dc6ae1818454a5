#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do for k in 0 256 512 1024; do
  RGSQR_NN_LITE_K=$k timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed "s/^/lite_k=$k: /"
done; done
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -q 2>&1 | tail -n 2
