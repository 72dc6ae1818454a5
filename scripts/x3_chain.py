"""TF32X3 accuracy vs the tensor-core accumulation chain (split-K count / x3_chain option):
kappa = 1e3 UΣV^T inputs, R error against Gram-Cholesky of the stored matrix (oracle),
backward error.  Writes gpurun_out/x3_chain.json."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402

h = Handle(0)
out = []
for (m, n) in [(8192, 256), (65536, 256), (65536, 2048)]:
    A64, _ = gi.usv(m, n, kappa=1e3, seed=3)
    A = gi.to_storage(A64, "fp32")
    X = gi.to_float64(A, "fp32")
    ref = oracle.gram_cholesky_r(X)
    for splitk, chain in [(0, 2), (1, 2), (16, 2), (0, 4), (1, 4), (4, 4), (16, 4), (0, 8), (1, 8)]:
        h.set_option("splitk", splitk)
        h.set_option("x3_chain", chain)
        Ad = to_dev(A, "fp32")
        R = torch.empty((n, n), dtype=torch.float32, device="cuda")
        rc = h.factor_device(Ad, m, m, n, Ad, R, precision="tf32x3")
        Q = from_dev(Ad)
        Rn = R.cpu().numpy().T.astype(np.float64)
        rec = {"m": m, "n": n, "splitk": splitk, "x3_chain": chain, "rc": rc,
               "backward": oracle.backward_error(X, Q, Rn), "r_err": oracle.r_rel_error(Rn, ref)}
        out.append(rec)
        print(json.dumps(rec), flush=True)
h.set_option("splitk", 0)
h.set_option("x3_chain", 4)
# throughput of the TF32X3 device path at configs[1]'s shape (fp32 storage), chains bounded vs not
A = gi.gaussian(65536, 8192, seed=2, dtype="fp32")
Ad = to_dev(A, "fp32")
Qd = torch.empty_like(Ad)
R = torch.empty((8192, 8192), dtype=torch.float32, device="cuda")
for chain in (2, 4, 8):
    h.set_option("x3_chain", chain)
    h.factor_device(Ad, 65536, 65536, 8192, Qd, R, precision="tf32x3")
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        h.factor_device(Ad, 65536, 65536, 8192, Qd, R, precision="tf32x3")
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    rec = {"m": 65536, "n": 8192, "x3_chain": chain, "ms": ms, "tflops": 2 * 65536 * 8192 ** 2 / ms / 1e9}
    out.append(rec)
    print(json.dumps(rec), flush=True)
h.set_option("x3_chain", 4)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/x3_chain.json", "w"), indent=1)
