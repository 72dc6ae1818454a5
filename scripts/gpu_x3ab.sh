#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in ab/librgsqr_base.so paper_conf_icpp_zhangw21_b200/librgsqr.so; do echo "== $lib"; RGSQR_LIB=$lib timeout 600 python scripts/x3_quick.py 2>&1 | tail -7; done
