"""Option sweep of the device-resident factorization (timing + per-kernel breakdown).

    python scripts/sweep.py --m 65536 --n 8192 --prec fp16 --opt leaf_width=32,48,64 [--opt reorth=0,1]
Prints one line per option combination: ms per factorization (CUDA events, median of reps)
and the per-kernel-class ms of one profiled run.
"""
import argparse
import itertools
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle, build  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=65536)
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--prec", default="fp16")
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--opt", action="append", default=[])
a = ap.parse_args()
build.build()
st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}[a.prec]
A = gi.gaussian(a.m, a.n, seed=2, dtype=st)
if st == "bf16":
    Ad = torch.from_numpy(np.ascontiguousarray(A.T).view(np.int16)).view(torch.bfloat16).cuda()
else:
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
Qd = torch.empty_like(Ad)
Rd = torch.empty((a.n, a.n), dtype=torch.float32, device="cuda")
h = Handle(0)
names, values = [], []
for o in a.opt:
    k, v = o.split("=")
    names.append(k)
    values.append([int(x) for x in v.split(",")])
for combo in itertools.product(*values) if values else [()]:
    for k, v in zip(names, combo):
        h.set_option(k, v)
    ts = []
    for r in range(a.reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h.factor_device(Ad, a.m, a.m, a.n, Qd, Rd, precision=a.prec, budget=1 << 30)
        e1.record()
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    h.set_option("profile", 1)
    h.factor_device(Ad, a.m, a.m, a.n, Qd, Rd, precision=a.prec, budget=1 << 30)
    torch.cuda.synchronize()
    s = h.stats()
    h.set_option("profile", 0)
    ms = float(np.median(ts))
    tf = 2.0 * a.m * a.n * a.n / ms / 1e9
    kern = " ".join(f"{nm}={s['kern_ms'][i]:.2f}/{s['kern_launches'][i]}" for i, nm in enumerate(["leaf", "inner", "outer", "other"]))
    print(f"{dict(zip(names, combo))} {a.m}x{a.n} {a.prec}: {ms:.2f} ms {tf:.1f} TFLOPS | {kern}", flush=True)
