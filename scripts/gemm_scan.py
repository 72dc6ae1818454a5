"""Per-shape throughput of the two node contractions (rgsqr_op_inner / rgsqr_op_outer) at the
widths the c2 recursion visits (m = 65536, w1 = w2 = w), CUDA events on the launching stream.
Total GEMM flops are the same per recursion level (2 m n w1), so the level with w = 4096 and
w = 2048 carry 3/4 of them.

    python scripts/gemm_scan.py [--m 65536] [--prec fp16]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_zhangw21_b200 import Handle, build  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=65536)
ap.add_argument("--prec", default="fp16")
ap.add_argument("--reps", type=int, default=20)
a = ap.parse_args()
build.build()
dt = {"fp16": torch.float16, "bf16": torch.bfloat16, "tf32": torch.float32}[a.prec]
h = Handle(0)
h.set_stream(torch.cuda.current_stream().cuda_stream)
m = a.m
for w in [128, 256, 512, 1024, 2048, 4096]:
    g = torch.Generator(device="cuda").manual_seed(w)
    Q1 = (torch.randn((w, m), device="cuda", generator=g) / m ** 0.5).to(dt)
    A2 = torch.randn((w, m), device="cuda", generator=g).to(dt)
    R12 = torch.empty((w, w), dtype=torch.float32, device="cuda")
    R12op = torch.empty((w, w), dtype=dt, device="cuda")
    out = {}
    for name in ["inner", "outer"]:
        ts = []
        for r in range(a.reps + 3):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            if name == "inner":
                h.op_inner(Q1, m, A2, m, m, w, w, R12, w, R12op, precision=a.prec)
            else:
                h.op_outer(Q1, m, R12op, w, A2, m, m, w, w, precision=a.prec)
            e1.record()
            torch.cuda.synchronize()
            if r >= 3:
                ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        out[name] = (ms, 2.0 * m * w * w / ms / 1e9)
    print(f"m={m} w1=w2={w} {a.prec}: inner {out['inner'][0]*1e3:.1f} us {out['inner'][1]:.0f} TF | "
          f"outer {out['outer'][0]*1e3:.1f} us {out['outer'][1]:.0f} TF", flush=True)
