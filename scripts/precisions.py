"""Device-resident factorization time per precision (c2 shape) and the c1 correctness config.

    python scripts/precisions.py [--out gpurun_out/precisions.json]
CUDA events around rgsqr_factor_device (median of reps), plus the backward error of one run
sampled on the first 4096 rows (c2) / all rows (c1) against the stored input.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle, build  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--out", default="gpurun_out/precisions.json")
a = ap.parse_args()
build.build()
h = Handle(0)
STOR = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32", "tf32x3": "fp32"}
rows = []
for (m, n, cfg) in [(4096, 256, "c1"), (65536, 8192, "c2")]:
    for prec in ["fp16", "bf16", "tf32", "tf32x3"]:
        st = STOR[prec]
        A = gi.gaussian(m, n, seed=1 if cfg == "c1" else 2, dtype=st)
        if st == "bf16":
            Ad = torch.from_numpy(np.ascontiguousarray(A.T).view(np.int16)).view(torch.bfloat16).cuda()
        else:
            Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
        Qd = torch.empty_like(Ad)
        Rd = torch.empty((n, n), dtype=torch.float32, device="cuda")
        ts = []
        for r in range(4):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            h.factor_device(Ad, m, m, n, Qd, Rd, precision=prec, budget=0 if prec == "tf32x3" else 1 << 30)
            e1.record()
            torch.cuda.synchronize()
            if r:
                ts.append(e0.elapsed_time(e1))
        ms = float(np.median(ts))
        R = Rd.cpu().numpy().T.astype(np.float64)
        if st == "bf16":
            Q = gi.to_float64(Qd.cpu().view(torch.int16).numpy().T, "bf16")
        else:
            Q = gi.to_float64(Qd.cpu().numpy().T, st)
        X = gi.to_float64(A, st)
        k = min(m, 4096)
        be = float(np.linalg.norm(X[:k] - Q[:k] @ R) / np.linalg.norm(X[:k]))
        row = {"config": cfg, "m": m, "n": n, "precision": prec, "ms": ms, "tflops": 2.0 * m * n * n / ms / 1e9,
               "backward_error_first_rows": be}
        print(json.dumps(row), flush=True)
        rows.append(row)
        del Ad, Qd, Rd
json.dump(rows, open(a.out, "w"), indent=1)
