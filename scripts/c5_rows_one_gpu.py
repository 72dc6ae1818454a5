"""configs[4]'s per-GPU share on ONE GPU (c5 at p = 8: 262144 rows per GPU), TF32X3 (the north star's 1e-5 mode):
fp32 A = U Sigma V^T, kappa = 1e3, m = 262144 x N, host-resident (pinned), rgsqr_factor in-core (budget 0) and
out-of-core (a budget of 1/4 of A); the WHOLE R against Gram-Cholesky of the stored A (oracle), backward error on a
row sample.  Writes gpurun_out/c5_rows.json.

    python scripts/c5_rows_one_gpu.py [--n 2048]
"""
import argparse, ctypes, json, os, sys, time
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=262144)
ap.add_argument("--n", type=int, default=2048)
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
m, n = a.m, a.n
t0 = time.perf_counter()
A64, sigma = gi.usv(m, n, kappa=1e3, seed=5)
A = gi.to_storage(A64, "fp32")
del A64
X = gi.to_float64(A, "fp32")
Rref = oracle.gram_cholesky_r(X)
t_ref = time.perf_counter() - t0
h = Handle(0)
nb = A.nbytes
pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(n * n * 4)
np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
rows = np.random.default_rng(0).choice(m, 20000, replace=False)
rows.sort()
out = []
for budget in (0, nb // 4):
    ts = []
    for _ in range(a.reps):
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        rc = h.factor(pa, m, m, n, pq, pr, precision="tf32x3", budget=budget)
        ts.append(time.perf_counter() - t1)
    st = h.stats()
    Q = np.ctypeslib.as_array((ctypes.c_float * (m * n)).from_address(pq)).reshape((m, n), order="F")
    R = np.ctypeslib.as_array((ctypes.c_float * (n * n)).from_address(pr)).reshape((n, n), order="F").astype(np.float64)
    Qs = Q[rows].astype(np.float64)
    rec = {"m": m, "n": n, "precision": "tf32x3", "kappa": 1e3, "budget": int(budget), "rc": rc, "s": min(ts),
           "tflops": 2 * m * n * n / min(ts) / 1e12, "ooc_nodes": st["n_ooc_nodes"],
           "h2d_GB": st["h2d_bytes"] / 1e9, "d2h_GB": st["d2h_bytes"] / 1e9,
           "r_rel_err_vs_gram_cholesky": oracle.r_rel_error(R, Rref),
           "north_star_bound": 1e-5,
           "backward_err_sampled_rows": float(np.linalg.norm(X[rows] - Qs @ R) / np.linalg.norm(X[rows])),
           "reference_seconds": t_ref}
    print(json.dumps(rec), flush=True)
    out.append(rec)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/c5_rows.json", "w"), indent=1)
