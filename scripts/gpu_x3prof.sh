python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for p in tf32 tf32x3; do echo "prec=$p"; python scripts/prof_run.py --prec $p --reps 2 --profile --budget-gib 8 2>&1 | tail -1; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_x3.csv python scripts/prof_run.py --prec tf32x3 --budget-gib 8 > gpurun_out/launches_x3.log 2>&1; tail -n 2 gpurun_out/launches_x3.log
python scripts/launch_summary.py gpurun_out/launches_x3.csv > gpurun_out/launches_x3_summary.md 2>&1; head -30 gpurun_out/launches_x3_summary.md
