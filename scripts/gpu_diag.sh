mkdir -p gpurun_out
RGSQR_LEAF_DEBUG2=1 timeout 120 python scripts/prof_run.py --n 1024 2>&1 | grep leaf2 | tail -n 2
cd scripts; timeout 60 ./crit_bench 2>&1 | tail -20; timeout 60 ./exchange_g 2>&1 | tail -20; timeout 60 ./barrier_bench 2>&1 | tail -12; cd ..
timeout 300 python scripts/sweep.py --opt leaf_width=32,48,64 2>&1 | tail -n 4
