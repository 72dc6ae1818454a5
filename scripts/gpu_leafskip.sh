#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for sk in 0 2 4 6; do
  RGSQR_LEAF_DEBUG=0 RGSQR_LEAF_SKIP=$sk timeout 300 python scripts/prof_run.py --n 512 > gpurun_out/leafskip_$sk.log 2>&1
  echo "skip=$sk: $(grep 'cycles/round' gpurun_out/leafskip_$sk.log | tail -n 3 | head -n 1)"
done
