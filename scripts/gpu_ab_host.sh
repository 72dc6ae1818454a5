#!/bin/bash
# A/B of a library change on the bench's value path (host-resident configs[1], 1 GiB budget, graph replay):
# ab/librgsqr_base.so (HEAD, scripts/ab_base.sh) vs the working tree, interleaved; host-path parity tests.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in 1 2 3; do for lib in ab/librgsqr_base.so paper_conf_icpp_zhangw21_b200/librgsqr.so; do
  echo "== $lib"; RGSQR_LIB=$lib timeout 300 python scripts/sweep_host.py --reps 5 2>&1 | tail -1 | cut -c1-160
done; done
timeout 1200 python -m pytest tests/test_gpu_factor_host.py tests/test_gpu_graph.py tests/test_gpu_edge_cases.py -q -x 2>&1 | tail -2
