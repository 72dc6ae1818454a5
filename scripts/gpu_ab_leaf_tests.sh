#!/bin/bash
# A/B of a library change on the leaf and the device factorization: ab/librgsqr_base.so (HEAD, built by
# scripts/ab_base.sh) vs the working tree's library, interleaved twice; leaf phase breakdown; parity tests.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do for lib in ab/librgsqr_base.so paper_conf_icpp_zhangw21_b200/librgsqr.so; do
  echo "== $lib"; RGSQR_LIB=$lib python scripts/leaf_diag.py --m 65536 --reps 40 | tail -1
  RGSQR_LIB=$lib python scripts/prof_run.py --reps 3 --profile 2>&1 | tail -1
done; done
RGSQR_LEAF_DEBUG=75 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles/round" | tail -1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py tests/test_gpu_dist.py -q -x 2>&1 | tail -3
