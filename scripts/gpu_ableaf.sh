#!/bin/bash
# A/B of the leaf: ab/librgsqr_base.so (HEAD) vs the working tree's library, interleaved.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do for lib in ab/librgsqr_base.so paper_conf_icpp_zhangw21_b200/librgsqr.so; do
  echo "== $lib"; RGSQR_LIB=$lib python scripts/leaf_diag.py --m 65536 --reps 40 | tail -1
  RGSQR_LIB=$lib python scripts/prof_run.py --reps 3 --profile 2>&1 | tail -1
done; done
RGSQR_LEAF_DEBUG=75 python scripts/leaf_diag.py --m 65536 --reps 2 2>&1 | grep -E "cycles/round" | tail -1
