#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/splitk.csv \
  python scripts/splitk_scan.py > gpurun_out/splitk.log 2>&1
tail -n 3 gpurun_out/splitk.log
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/splitk.csv')) if len(r) > 10 and r[0].isdigit()]
for r in rows:
    print(r[4][:40], r[8], r[-1])
PY
