import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import Handle
from tests.gpu_util import to_dev, from_dev
h = Handle(0)
m, w1, w2 = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
Q = gi.gaussian(m, w1, seed=5, dtype="fp16"); A = gi.gaussian(m, w2, seed=6, dtype="fp16")
R = np.asfortranarray(np.random.default_rng(1).standard_normal((w1, w2)).astype(np.float32) / 16)
Xq, Xa = gi.to_float64(Q, "fp16"), gi.to_float64(A, "fp16")
Rop = R.astype(np.float16).astype(np.float64)
ref = Xa - Xq @ Rop
for ser in (1, 0):
  for tiling, block in ((0, 2048), (0, 0), (1, 1024)):
    h.set_option("serialize", ser)
    A2 = np.array(A, order="F", copy=True)
    h.ooc_outer(Q, m, R, w1, A2, m, m, w1, w2, precision="fp16", tiling=tiling, block=block, budget=48 << 20)
    got = gi.to_float64(A2, "fp16")
    bad = ~np.isfinite(got)
    err = np.nanmax(np.abs(got - ref))
    print("ser", ser, "tiling", tiling, "block", block, "nan", bad.sum(), "first", np.argwhere(bad)[:3].tolist(), "maxerr", err, "changed", np.mean(A2 != A), h.stats()["h2d_bytes"], h.stats()["d2h_bytes"])
# direct device op_outer
Qd, Ad = to_dev(Q, "fp16"), to_dev(A, "fp16")
Rd = torch.from_numpy(np.ascontiguousarray(R.astype(np.float16).T)).cuda()
h.op_outer(Qd, m, Rd, w1, Ad, m, m, w1, w2, precision="fp16")
print("device op_outer maxerr", np.max(np.abs(from_dev(Ad) - ref)))
