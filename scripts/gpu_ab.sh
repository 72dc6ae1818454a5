#!/bin/bash
# A/B of the TN rasterization on the device path, host-path option sweep, ncu launch list of the
# bench value path (host, out-of-core) and full captures of the leaf and the top-node TN.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for g in 0 16; do RGSQR_GROUP_M=$g timeout 300 python scripts/sweep.py --reps 5 > gpurun_out/sweep_group$g.log 2>&1; echo "group $g: $(tail -n 1 gpurun_out/sweep_group$g.log)"; done
timeout 900 python scripts/sweep_host.py --reps 5 --opt defer_pieces=0,2,4 --opt chunk_mib=32,64 > gpurun_out/sweep_host.log 2>&1; cut -c1-200 gpurun_out/sweep_host.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_host.csv python scripts/prof_run.py --host > gpurun_out/launches_host.log 2>&1; python scripts/launch_summary.py gpurun_out/launches_host.csv > gpurun_out/launches_host_summary.md; head -12 gpurun_out/launches_host_summary.md
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_dev.csv python scripts/prof_run.py > gpurun_out/launches_dev.log 2>&1; python scripts/launch_summary.py gpurun_out/launches_dev.csv > gpurun_out/launches_dev_summary.md; head -12 gpurun_out/launches_dev_summary.md
timeout 900 ncu --set full --clock-control none --import-source on -k regex:leaf_cgs -s 20 -c 1 -o gpurun_out/prof_leaf python scripts/prof_run.py > gpurun_out/ncu_leaf.log 2>&1; tail -n 2 gpurun_out/ncu_leaf.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_kernel -s 60 -c 2 -o gpurun_out/prof_tn python scripts/prof_run.py > gpurun_out/ncu_tn.log 2>&1; tail -n 2 gpurun_out/ncu_tn.log
echo ab done
