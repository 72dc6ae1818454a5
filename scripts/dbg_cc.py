import sys; sys.path.insert(0, '/root/repo')
import numpy as np, rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import Handle
MiB = 1 << 20
m, n = 16384, 1024
A = gi.gaussian(m, n, seed=14, dtype="fp16")
plain = Handle(0); plain.set_option("fuse_small", 0); dist = Handle(0, rank=0, nranks=1, unique_id=Handle.unique_id())
for b in (34, 35, 36, 37, 38, 40):
  for nm, h in (("plain", plain), ("dist", dist)):
    h.set_option("chunk_mib", 2)
    Q = np.empty_like(A, order="F"); R = np.zeros((n, n), dtype=np.float32, order="F")
    try:
      rc = h.factor(A, m, m, n, Q, R, precision="fp16", budget=b * MiB)
    except Exception as e:
      print(b, nm, 'ERR', e); continue
    st = h.stats(); print(b, nm, rc, {k: st[k] for k in ("n_ooc_nodes", "n_colchunk_nodes", "colchunk_tail_cols", "h2d_bytes")})
