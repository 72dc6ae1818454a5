#!/bin/bash
# Tall leaf panels (> 2048 rows per CTA): parity tests, launch times; c2 device path unchanged.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_factor_device.py -q -x -k "leaf or tall" 2>&1 | tail -3
for mw in "400000 15" "600000 9" "1048576 4"; do set -- $mw; python scripts/leaf_diag.py --m $1 --w $2 --reps 10; done
python scripts/prof_run.py --reps 3 --profile 2>&1 | tail -1
