#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for gm in 0 4 8 16; do echo "GROUP_M=$gm"; RGSQR_GROUP_M=$gm timeout 600 python scripts/x3_quick.py 2>&1 | tail -1; done
