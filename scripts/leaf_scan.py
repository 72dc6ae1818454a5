"""Leaf kernel timing vs panel width (through rgsqr_op_leaf): slope = cost per column
(one grid exchange round), intercept = fixed cost per launch.

    python scripts/leaf_scan.py [--m 65536] [--prec fp16]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle, build  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=65536)
ap.add_argument("--prec", default="fp16")
ap.add_argument("--reps", type=int, default=50)
a = ap.parse_args()
build.build()
st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}[a.prec]
h = Handle(0)
A = gi.gaussian(a.m, 64, seed=2, dtype=st)
A0 = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
P = A0.clone()
R = torch.empty((64, 64), dtype=torch.float32, device="cuda")
res = []
for w in [1, 2, 4, 8, 16, 24, 32, 48, 64]:
    ts = []
    for r in range(a.reps + 2):
        P.copy_(A0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h.op_leaf(P, a.m, a.m, w, R, 64, precision=a.prec)
        e1.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1) * 1e3)
    us = float(np.median(ts))
    res.append((w, us))
    print(f"m={a.m} w={w}: {us:.1f} us  ({us / w:.2f} us/col)", flush=True)
W = np.array([r[0] for r in res if r[0] >= 8], dtype=float)
T = np.array([r[1] for r in res if r[0] >= 8])
slope, icpt = np.polyfit(W, T, 1)
print(f"fit (w>=8): {slope:.3f} us per column + {icpt:.1f} us per launch")
