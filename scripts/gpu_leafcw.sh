#!/bin/bash
for cw in 8 7 6 8 7 6; do
  echo "CW=$cw"; RGSQR_LEAF_CW=$cw python scripts/sweep.py --reps 7 2>&1 | tail -1
done
for cw in 7 6; do RGSQR_LEAF_CW=$cw RGSQR_LEAF_DEBUG=75 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles/round" | tail -1; done
RGSQR_LEAF_CW=6 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -x -q 2>&1 | tail -2
RGSQR_LEAF_CW=7 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -x -q 2>&1 | tail -2
