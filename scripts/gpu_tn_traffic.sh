#!/bin/bash
# DRAM traffic of the configs[1] top-node inner product (gemm_kernel grid 32 x 16) with x-fastest vs grouped
# rasterization (RGSQR_GROUP_M), from full ncu captures; plus device-path time with each setting.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for gm in 0 4 16; do
  RGSQR_GROUP_M=$gm timeout 600 ncu --set full --clock-control none -k regex:gemm_kernel --launch-skip-before-match 0 \
    --kernel-name-base demangled -c 200 --csv --page raw --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active,launch__grid_size \
    python scripts/prof_run.py > gpurun_out/tn_gm$gm.csv 2> gpurun_out/tn_gm$gm.err
  echo "GROUP_M=$gm"; python - <<PY
import csv
rows=list(csv.reader(open("gpurun_out/tn_gm$gm.csv")))
i=next(k for k,r in enumerate(rows) if r and r[0]=="ID")
h=rows[i]; best=None
for r in rows[i+2:]:
    d=dict(zip(h,r))
    if d.get("launch__grid_size")=="512":
        print("grid 512:", {k:d.get(k) for k in ("gpu__time_duration.sum","dram__bytes_read.sum","dram__bytes_write.sum","sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active")})
PY
  RGSQR_GROUP_M=$gm python scripts/prof_run.py --reps 3 --profile 2>&1 | tail -1
done
