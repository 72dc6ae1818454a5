"""TN split-K factor at the narrow c2 node widths: run op_inner (m = 65536) under ncu and read
per-launch GPU durations (gemm_kernel + splitk_reduce) -- no host overhead in the numbers.

    ncu --metrics gpu__time_duration.sum --csv --log-file X.csv python scripts/splitk_scan.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

h = Handle(0)
m = 65536
for w in [128, 256, 512]:
    Q1 = (torch.randn((w, m), device="cuda") / m ** 0.5).half()
    A2 = torch.randn((w, m), device="cuda").half()
    R12 = torch.empty((w, w), dtype=torch.float32, device="cuda")
    R12op = torch.empty((w, w), dtype=torch.float16, device="cuda")
    for sk in [0, 16, 37, 74, 148, 222]:
        h.set_option("splitk", sk)
        for _ in range(2):
            h.op_inner(Q1, m, A2, m, m, w, w, R12, w, R12op, precision="fp16")
        torch.cuda.synchronize()
        print(f"w={w} splitk={sk}", flush=True)
