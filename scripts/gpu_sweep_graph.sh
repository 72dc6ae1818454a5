#!/bin/bash
# host-path option sweeps with CUDA-graph replay (the bench's value path)
for o in split_pct=50,56,62,68,75 eager_pct=25,50,75,100 phasea_pct=0,25,50,75,100 chunk_mib=16,32,64 ring_depth=2,3,4 tile_rows_max=8192,16384,32768 colchunk=0,1; do
  timeout 600 python scripts/sweep_host.py --reps 5 --opt $o 2>&1 | grep '^{' | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(d['opts'], round(d['ms'], 2), round(d['tflops'], 1), 'tail', d['tail_cols'])"
done
