#!/bin/bash
for s in 0 2 4 6; do echo "skip=$s"; RGSQR_LEAF_DEBUG=75 RGSQR_LEAF_SKIP=$s python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles" | tail -2; done
for ns in 0 20 64 128; do echo "poll_ns=$ns"; RGSQR_LEAF_POLL_NS=$ns RGSQR_LEAF_DEBUG2=1 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "leaf2" | tail -1; done
