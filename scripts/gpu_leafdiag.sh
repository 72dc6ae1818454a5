#!/bin/bash
# leaf timing + phase breakdown on one B200
mkdir -p gpurun_out
python scripts/leaf_diag.py --m 65536
python scripts/leaf_diag.py --m 32768
python scripts/leaf_diag.py --m 16384
for cta in 0 75 147; do RGSQR_LEAF_DEBUG=$cta python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles" | tail -2; done
RGSQR_LEAF_DEBUG=0 RGSQR_LEAF_SKIP=6 python scripts/leaf_diag.py --m 65536 --reps 3 2>&1 | grep -E "cycles|us/col" | tail -3
RGSQR_LEAF_DEBUG2=1 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "leaf2" | tail -1
