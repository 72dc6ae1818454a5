"""Option sweep of the HOST-resident (out-of-core) factorization, the bench's value path.

    python scripts/sweep_host.py [--m 65536 --n 8192 --prec fp16 --budget-mib 1024] --opt chunk_mib=16,32,64
One JSON line per option combination: median ms of `reps` calls (wall of the host-synchronous
rgsqr_factor, CUDA events), bytes moved and the stream busy times of the last call.
"""
import argparse
import ctypes
import itertools
import json
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
ap.add_argument("--budget-mib", type=int, default=1024)
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--opt", action="append", default=[])
a = ap.parse_args()
build.build()
st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}[a.prec]
A = gi.gaussian(a.m, a.n, seed=2, dtype=st)
h = Handle(0)
nb = A.nbytes
pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(a.n * a.n * 4)
np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
names, values = [], []
for o in a.opt:
    k, v = o.split("=")
    names.append(k)
    values.append([int(x) for x in v.split(",")])
budget = a.budget_mib << 20
for combo in itertools.product(*values) if values else [()]:
    for k, v in zip(names, combo):
        h.set_option(k, v)
    h.factor(pa, a.m, a.m, a.n, pq, pr, precision=a.prec, budget=budget)
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h.factor(pa, a.m, a.m, a.n, pq, pr, precision=a.prec, budget=budget)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    s = h.stats()
    ms = float(np.median(ts))
    print(json.dumps({"opts": dict(zip(names, combo)), "ms": ms, "tflops": 2 * a.m * a.n ** 2 / ms / 1e9,
                      "h2d": s["h2d_bytes"], "d2h": s["d2h_bytes"], "busy": [s["h2d_busy_ms"], s["d2h_busy_ms"],
                                                                             s["compute_busy_ms"]],
                      "colchunk_nodes": s["n_colchunk_nodes"], "tail_cols": s["colchunk_tail_cols"]}), flush=True)
for p_ in (pa, pq, pr):
    h.host_free(p_)
