"""Write R and Q of a TF32X3 device factorization (fp32 Gaussian 16384 x 1536) to gpurun_out/x3_bits_<tag>.npz
(bitwise A/B of a library change via RGSQR_LIB)."""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402
from tests.gpu_util import to_dev, from_dev  # noqa: E402
tag = sys.argv[1]
m, n = 16384, 1536
A = gi.gaussian(m, n, seed=8, dtype="fp32")
h = Handle(0)
Ad = to_dev(A, "fp32")
R = torch.empty((n, n), dtype=torch.float32, device="cuda")
h.factor_device(Ad, m, m, n, Ad, R, precision="tf32x3", budget=2 << 30)
np.savez(f"gpurun_out/x3_bits_{tag}.npz", Q=from_dev(Ad), R=R.cpu().numpy())
print(tag, "launches other", h.stats()["n_other_launches"])
