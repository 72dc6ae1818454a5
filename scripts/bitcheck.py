"""Bitwise A/B of two builds: sha256 of Q and R from one c2 device factorization and one
host out-of-core factorization.   python scripts/bitcheck.py <path-to-librgsqr.so>"""
import hashlib
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle, load_library  # noqa: E402

load_library(sys.argv[1])
h = Handle(0)
A = gi.gaussian(65536, 8192, seed=2, dtype="fp16")
At = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
Qt = torch.empty_like(At)
R = torch.empty((8192, 8192), dtype=torch.float32, device="cuda")
for _ in range(3):
    h.factor_device(At, 65536, 65536, 8192, Qt, R, precision="fp16", budget=1 << 30)
torch.cuda.synchronize()
import time  # noqa: E402
t = time.perf_counter()
for _ in range(5):
    h.factor_device(At, 65536, 65536, 8192, Qt, R, precision="fp16", budget=1 << 30)
torch.cuda.synchronize()
ms = (time.perf_counter() - t) / 5 * 1e3
d = hashlib.sha256(Qt.cpu().numpy().tobytes() + R.cpu().numpy().tobytes()).hexdigest()[:16]
B = gi.gaussian(16384, 1024, seed=7, dtype="fp16")
Q = np.empty_like(B, order="F")
R2 = np.empty((1024, 1024), dtype=np.float32, order="F")
h.factor(np.asfortranarray(B), 16384, 16384, 1024, Q, R2, precision="fp16", budget=12 << 20)
d2 = hashlib.sha256(Q.tobytes() + R2.tobytes()).hexdigest()[:16]
print(f"{sys.argv[1]}: device {d} ({ms:.2f} ms wall/factorization)  host-ooc {d2}")
