#!/bin/bash
# One gpurun call: STEPS (space-separated) selects what runs; every output under gpurun_out/.
#   smoke tests tests_fast x3 bench probe cpuc2 launches ncu_leaf
mkdir -p gpurun_out
STEPS=${STEPS:-"smoke tests bench"}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for s in $STEPS; do
  case $s in
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -n 1 gpurun_out/smoke.log ;;
    tests) timeout 2400 python -m pytest tests -q -m gpu ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; tail -n 3 gpurun_out/pytest_gpu.log; grep -E "^(FAILED|ERROR)" gpurun_out/pytest_gpu.log | head -30 ;;
    tests_fast) timeout 1500 python -m pytest tests -q -m gpu --deselect tests/test_gpu_c3.py ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; tail -n 3 gpurun_out/pytest_gpu.log; grep -E "^(FAILED|ERROR)" gpurun_out/pytest_gpu.log | head -30 ;;
    x3) timeout 900 python scripts/x3_chain.py > gpurun_out/x3_chain.log 2>&1; tail -n 30 gpurun_out/x3_chain.log ;;
    bench) timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -c 3000 gpurun_out/bench.json; tail -n 5 gpurun_out/bench.err ;;
    probe) timeout 600 python scripts/probe.py > gpurun_out/probe.log 2>&1; tail -n 40 gpurun_out/probe.log ;;
    cpuc2) timeout 1200 python scripts/cpu_oracle_c2.py > gpurun_out/cpuc2.log 2>&1; tail -n 2 gpurun_out/cpuc2.log ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python scripts/prof_run.py ${PROF_ARGS} > gpurun_out/launches.log 2>&1; tail -n 3 gpurun_out/launches.log ;;
    timeline) RGSQR_TIMELINE=gpurun_out/timeline_c2.csv timeout 300 python scripts/prof_run.py --host --reps 3 > gpurun_out/timeline.log 2>&1; python scripts/timeline.py gpurun_out/timeline_c2.csv > gpurun_out/timeline_summary.txt; head -1 gpurun_out/timeline_summary.txt; tail -n 2 gpurun_out/timeline.log ;;
    hosttests) timeout 1200 python -m pytest tests/test_gpu_factor_host.py -q -x ${PYTEST_ARGS} > gpurun_out/pytest_host.log 2>&1; tail -n 3 gpurun_out/pytest_host.log; grep -E "^(FAILED|ERROR)|Error" gpurun_out/pytest_host.log | head -20 ;;
    pyfiles) timeout 1500 python -m pytest ${PYFILES} -q ${PYTEST_ARGS} > gpurun_out/pytest_files.log 2>&1; tail -n 3 gpurun_out/pytest_files.log; grep -E "^(FAILED|ERROR)|Error" gpurun_out/pytest_files.log | head -20 ;;
    sweephost) timeout 1200 python scripts/sweep_host.py ${SWEEP_ARGS} > gpurun_out/sweep_host.log 2>&1; cat gpurun_out/sweep_host.log | cut -c1-220 ;;
    tables) timeout 1800 python scripts/paper_gemm_tables.py ${TABLES_ARGS} > gpurun_out/paper_gemm_tables.log 2>&1; cut -c1-260 gpurun_out/paper_gemm_tables.log ;;
    *) echo "unknown step $s" ;;
  esac
done
echo session done
