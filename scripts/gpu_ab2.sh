#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2; do
for lib in paper_conf_icpp_zhangw21_b200/librgsqr.so build_alt/librgsqr_nogroup.so build_alt/librgsqr_r1.so; do
  RGSQR_LIB=$PWD/$lib timeout 300 python scripts/sweep.py --reps 7 > gpurun_out/ab_$(basename $lib).log 2>&1; echo "$lib: $(tail -n 1 gpurun_out/ab_$(basename $lib).log)"
done; done
