#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
  (cd build_alt/r1src && timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed 's/^/r1: /')
  timeout 300 python scripts/sweep.py --reps 7 2>&1 | tail -n 1 | sed 's/^/r2: /'
done
RGSQR_LEAF_DEBUG=0 timeout 300 python scripts/prof_run.py --n 512 > gpurun_out/leafdbg.log 2>&1; grep -E "cycles" gpurun_out/leafdbg.log | head -12
