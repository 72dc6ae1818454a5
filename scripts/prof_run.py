"""One device-resident factorization of a bench workload, for ncu launch lists / captures.

    python scripts/prof_run.py [--m 65536] [--n 8192] [--prec fp16] [--reps 1]
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
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--prec", default="fp16")
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--host", action="store_true", help="use the host (out-of-core) path, 1 GiB budget")
ap.add_argument("--pinned", action="store_true", help="host path with rgsqr_host_alloc buffers (CUDA-graph replay)")
ap.add_argument("--budget-gib", type=float, default=1.0)
ap.add_argument("--profile", action="store_true", help="per-kernel-class CUDA-event accounting (RGSQR_OPT_PROFILE)")
a = ap.parse_args()
build.build()
st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}[a.prec]
A = gi.gaussian(a.m, a.n, seed=2, dtype=st)
h = Handle(0)
if a.profile:
    h.set_option("profile", 1)
if a.host and a.pinned:
    import ctypes
    nb = A.nbytes
    pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(a.n * a.n * 4)
    np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
    for _ in range(a.reps):
        h.factor(pa, a.m, a.m, a.n, pq, pr, precision=a.prec, budget=1 << 30)
elif a.host:
    Q = np.empty_like(A, order="F")
    R = np.empty((a.n, a.n), dtype=np.float32, order="F")
    for _ in range(a.reps):
        h.factor(A, a.m, a.m, a.n, Q, R, precision=a.prec, budget=1 << 30)
else:
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
    Qd = torch.empty_like(Ad)
    Rd = torch.empty((a.n, a.n), dtype=torch.float32, device="cuda")
    for _ in range(a.reps):
        h.factor_device(Ad, a.m, a.m, a.n, Qd, Rd, precision=a.prec, budget=int(a.budget_gib * (1 << 30)))
torch.cuda.synchronize()
st = h.stats()
print("stats", st)
if a.profile:
    print("kern_ms leaf/inner/outer/other", [round(x, 3) for x in st["kern_ms"]], "sum", round(sum(st["kern_ms"]), 3),
          "wall", round(st["wall_ms"], 3))
