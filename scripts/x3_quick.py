"""TF32X3 quick check: kappa = 1e3 R error vs Gram-Cholesky (splits 0/1/16) and configs[1]-shaped device time."""
import json, os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402
h = Handle(0)
for (m, n) in [(8192, 256), (65536, 2048)]:
    A64, _ = gi.usv(m, n, kappa=1e3, seed=3)
    A = gi.to_storage(A64, "fp32")
    X = gi.to_float64(A, "fp32")
    ref = oracle.gram_cholesky_r(X)
    for splitk in (0, 1, 16):
        h.set_option("splitk", splitk)
        Ad = to_dev(A, "fp32")
        R = torch.empty((n, n), dtype=torch.float32, device="cuda")
        rc = h.factor_device(Ad, m, m, n, Ad, R, precision="tf32x3", budget=8 << 30)
        Rn = R.cpu().numpy().T.astype(np.float64)
        print(json.dumps({"m": m, "n": n, "splitk": splitk, "rc": rc, "backward": oracle.backward_error(X, from_dev(Ad), Rn),
                          "r_err": oracle.r_rel_error(Rn, ref)}), flush=True)
h.set_option("splitk", 0)
A = gi.gaussian(65536, 8192, seed=2, dtype="fp32")
Ad = to_dev(A, "fp32")
Qd = torch.empty_like(Ad)
R = torch.empty((8192, 8192), dtype=torch.float32, device="cuda")
h.factor_device(Ad, 65536, 65536, 8192, Qd, R, precision="tf32x3", budget=8 << 30)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(3):
    h.factor_device(Ad, 65536, 65536, 8192, Qd, R, precision="tf32x3", budget=8 << 30)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 3
print(json.dumps({"m": 65536, "n": 8192, "ms": ms, "tflops": 2 * 65536 * 8192 ** 2 / ms / 1e9}))
