#!/bin/bash
for pf in 0 1 0 1; do echo "prefetch=$pf"; RGSQR_LEAF_PREFETCH=$pf python scripts/sweep.py --reps 7 2>&1 | tail -1; done
RGSQR_LEAF_PREFETCH=1 RGSQR_LEAF_DEBUG=75 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles/round" | tail -1
python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py tests/test_gpu_dist.py -x -q 2>&1 | tail -2
