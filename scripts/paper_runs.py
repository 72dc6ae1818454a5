"""Out-of-core runs at the paper's / BASELINE's larger shapes, recursive vs blocked.

    python scripts/paper_runs.py [--which c3,t4a,t4b] [--out gpurun_out/paper_runs.json]

* c3  : BASELINE.json configs[2] -- fp16 262144 x 32768 Gaussian, 8 GiB device budget,
        recursive (Eq. 2) vs blocked (panel 8192).
* t4a : PAPER.md Table 4 shape 65536 x 65536, fp32 host data (TF32 MMA), 16 GiB cap
        ("limiting the memory usage to be less than 16GB"), blocksize 8192.
* t4b : PAPER.md Table 4 shape 262144 x 65536, same settings.
Each line reports wall time, TFLOPS (2 m n^2), bytes moved, busy times and overlap ratio.
Correctness at these sizes is checked by the parity tests at smaller sizes; here the
backward error is sampled on random row blocks against the Gram-Cholesky relation
(||R^T R - A^T A|| / ||A^T A|| on a column block) -- cheap and independent.
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

GiB = 1 << 30
RUNS = {
    "c3": dict(m=262144, n=32768, prec="fp16", budget=8 * GiB, block=8192),
    "t4a": dict(m=65536, n=65536, prec="tf32", budget=16 * GiB, block=8192),
    "t4b": dict(m=262144, n=65536, prec="tf32", budget=16 * GiB, block=8192),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--which", default="c3")
    ap.add_argument("--algos", default="recursive,blocked,fused")
    ap.add_argument("--out", default="gpurun_out/paper_runs.json")
    a = ap.parse_args()
    h = Handle(0)
    results = []
    for name in a.which.split(","):
        cfg = RUNS[name]
        m, n = cfg["m"], cfg["n"]
        st = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}[cfg["prec"]]
        t0 = time.time()
        pa = h.host_alloc(m * n * gi.storage_bytes(st))
        pq = h.host_alloc(m * n * gi.storage_bytes(st))
        pr = h.host_alloc(n * n * 4)
        import ctypes
        A = np.ctypeslib.as_array((ctypes.c_uint8 * (m * n * gi.storage_bytes(st))).from_address(pa))
        A = A.view(gi.storage_numpy_dtype(st)).reshape((n, m)).T          # column-major view
        gi.gaussian(m, n, seed=3, dtype=st, out=A)
        gen_s = time.time() - t0
        for algo in a.algos.split(","):
            h.set_option("algo", {"recursive": 0, "blocked": 1, "fused": 2}[algo])
            h.set_option("block_cols", cfg["block"])
            h.factor(pa, m, m, n, pq, pr, precision=cfg["prec"], budget=cfg["budget"])   # warm-up
            s = h.stats()
            t = time.time()
            h.factor(pa, m, m, n, pq, pr, precision=cfg["prec"], budget=cfg["budget"])
            wall = time.time() - t
            s = h.stats()
            # sampled check: R^T R vs A^T A on the first 256 columns (fp64)
            k = 256
            R = np.ctypeslib.as_array((ctypes.c_float * (n * n)).from_address(pr)).reshape((n, n)).T
            Rk = R[:k, :k].astype(np.float64)
            Xk = gi.to_float64(np.asarray(A[:, :k]), st)
            G = Xk.T @ Xk
            rel = float(np.linalg.norm(Rk.T @ Rk - G) / np.linalg.norm(G))
            line = {"run": name, "algo": algo, "m": m, "n": n, "precision": cfg["prec"], "budget_bytes": cfg["budget"],
                    "block_cols": cfg["block"], "wall_s": wall, "tflops": 2.0 * m * n * n / wall / 1e12,
                    "h2d_bytes": s["h2d_bytes"], "d2h_bytes": s["d2h_bytes"], "h2d_busy_ms": s["h2d_busy_ms"],
                    "d2h_busy_ms": s["d2h_busy_ms"], "compute_busy_ms": s["compute_busy_ms"],
                    "overlap_ratio": s["overlap_ratio"], "ooc_nodes": s["n_ooc_nodes"],
                    "arena_bytes": s["arena_bytes"], "gram_rel_err_first256": rel, "gen_s": gen_s}
            print(json.dumps(line), flush=True)
            results.append(line)
        h.set_option("algo", 0)
        for p in (pa, pq, pr):
            h.host_free(p)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    json.dump(results, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
