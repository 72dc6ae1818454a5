"""Small factorizations for compute-sanitizer runs (memcheck / racecheck / synccheck): device path
(fp16 and TF32X3) and the host out-of-core path (column-chunked node) at small sizes."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402
from paper_conf_icpp_zhangw21_b200 import Handle  # noqa: E402

which = sys.argv[1] if len(sys.argv) > 1 else "all"
h = Handle(0)
if which in ("all", "device"):
    for prec, st in (("fp16", "fp16"), ("tf32x3", "fp32")):
        m, n = 4096, 256
        A = gi.gaussian(m, n, seed=1, dtype=st)
        Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
        R = torch.empty((n, n), dtype=torch.float32, device="cuda")
        print(prec, "device rc", h.factor_device(Ad, m, m, n, Ad, R, precision=prec), flush=True)
if which in ("all", "host"):
    m, n = 16384, 1024
    A = gi.gaussian(m, n, seed=2, dtype="fp16")
    Q = np.empty_like(A, order="F")
    R = np.empty((n, n), dtype=np.float32, order="F")
    h.set_option("chunk_mib", 2)
    print("host rc", h.factor(A, m, m, n, Q, R, precision="fp16", budget=38 << 20), h.stats()["n_colchunk_nodes"],
          flush=True)
torch.cuda.synchronize()
h.close()
print("done")
