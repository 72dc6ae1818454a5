"""configs[3]'s rows on ONE GPU (tall leaf panels, R31): bf16 A 1048576 x N host-resident (pinned),
rgsqr_factor in-core (budget 0) and out-of-core (4 GiB budget); R's leading block vs Gram-Cholesky of the stored
A (oracle), ||q_j|| on sampled columns.  Writes gpurun_out/c4_p1.json.

    python scripts/c4_p1.py [--n 4096]
"""
import argparse, ctypes, json, os, sys, time
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=1048576)
ap.add_argument("--n", type=int, default=4096)
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
m, n = a.m, a.n
h = Handle(0)
A = gi.gaussian(m, n, seed=2, dtype="bf16")
nb = A.nbytes
pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(n * n * 4)
np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
out = []
for budget in (0, 4 << 30):
    ts = []
    for _ in range(a.reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        rc = h.factor(pa, m, m, n, pq, pr, precision="bf16", budget=budget)
        ts.append(time.perf_counter() - t0)
    st = h.stats()
    Qh = np.ctypeslib.as_array((ctypes.c_uint16 * (m * n)).from_address(pq)).reshape((m, n), order="F")
    Rh = np.ctypeslib.as_array((ctypes.c_float * (n * n)).from_address(pr)).reshape((n, n), order="F").astype(np.float64)
    k = 256
    Xk = gi.to_float64(A[:, :k], "bf16")
    Rref = oracle.gram_cholesky_r(Xk)
    cols = np.linspace(0, n - 1, 8).astype(int)
    qn = [float(np.linalg.norm(gi.to_float64(Qh[:, [j]].view(np.uint16).copy(), "bf16"))) for j in cols]
    rec = {"m": m, "n": n, "precision": "bf16", "budget": budget, "rc": rc, "s": min(ts),
           "tflops": 2 * m * n * n / min(ts) / 1e12, "leaf_launches": st["n_leaf_launches"],
           "ooc_nodes": st["n_ooc_nodes"], "h2d_GB": st["h2d_bytes"] / 1e9, "d2h_GB": st["d2h_bytes"] / 1e9,
           "r_lead256_rel_err_vs_gram_cholesky": oracle.r_rel_error(Rh[:k, :k], Rref),
           "diag_positive": bool(np.all(np.diag(Rh) > 0)), "q_norms_sampled": qn}
    print(json.dumps(rec), flush=True)
    out.append(rec)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/c4_p1.json", "w"), indent=1)
