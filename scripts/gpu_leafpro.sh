#!/bin/bash
for cta in 0 40 75 120 147; do RGSQR_LEAF_DEBUG=$cta python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "prologue" | tail -1; done
