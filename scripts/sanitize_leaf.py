"""One small leaf panel and one small inner/outer product, for compute-sanitizer racecheck/synccheck."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

h = Handle(0)
h.set_option("leaf_ctas", 8)
m, w = 2048, 32
A = gi.gaussian(m, w, seed=1, dtype="fp16")
P = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
R = torch.zeros((w, w), dtype=torch.float32, device="cuda")
print("leaf", h.op_leaf(P, m, m, w, R, w, precision="fp16"), flush=True)
Q = gi.gaussian(m, 128, seed=2, dtype="fp16")
A2 = gi.gaussian(m, 128, seed=3, dtype="fp16")
Qd = torch.from_numpy(np.ascontiguousarray(Q.T)).cuda()
Ad = torch.from_numpy(np.ascontiguousarray(A2.T)).cuda()
R12 = torch.zeros((128, 128), dtype=torch.float32, device="cuda")
Rop = torch.zeros((128, 128), dtype=torch.float16, device="cuda")
h.op_inner(Qd, m, Ad, m, m, 128, 128, R12, 128, Rop, precision="fp16")
h.op_outer(Qd, m, Rop, 128, Ad, m, m, 128, 128, precision="fp16")
torch.cuda.synchronize()
print("done", flush=True)
