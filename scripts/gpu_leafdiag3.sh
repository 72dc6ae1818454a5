#!/bin/bash
# Leaf phase breakdown at the configs[1] panel (65536 x 64): debug stamps, exchange skew, warm launch time.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for s in 0 6; do echo "skip=$s"; RGSQR_LEAF_DEBUG=75 RGSQR_LEAF_SKIP=$s python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles" | tail -2; done
RGSQR_LEAF_DEBUG=3 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles" | tail -2
RGSQR_LEAF_DEBUG2=1 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "leaf2" | tail -1
python scripts/leaf_diag.py --m 65536 --reps 30
