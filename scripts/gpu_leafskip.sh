#!/bin/bash
# Leaf round time with bulk phases skipped (diagnostics only; results are wrong when skipping).
for s in 0 2 4 6; do
  echo "skip=$s"; RGSQR_LEAF_DEBUG=5 RGSQR_LEAF_SKIP=$s RGSQR_LEAF_DEBUG2=1 timeout 120 python scripts/prof_run.py --n 512 2>&1 | grep -E "leaf2|cycles/round" | tail -n 2
done
