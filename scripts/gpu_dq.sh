#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for dq in 0 2 3 4 6; do RGSQR_DEFER_Q_CHUNKS=$dq timeout 300 python scripts/sweep_host.py --reps 5 2>&1 | cut -c1-120 | sed "s/^/dq=$dq /"; done
for dq in 0 3; do RGSQR_DEFER_Q_CHUNKS=$dq timeout 300 python scripts/sweep_host.py --reps 5 2>&1 | cut -c1-120 | sed "s/^/dq=$dq /"; done
