"""A/B of RGSQR_OPT_GRAPH (CUDA-graph replay) on configs[1]: host path (pinned buffers, 1 GiB budget)
and device path; wall per call with CUDA events and bitwise comparison of Q and R between modes."""
import argparse, ctypes, sys
sys.path.insert(0, "/root/repo")
import numpy as np, torch
import rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import Handle

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=65536)
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--budget_mib", type=int, default=1024)
a = ap.parse_args()
m, n = a.m, a.n
A = gi.gaussian(m, n, seed=2, dtype="fp16")
h = Handle(0)
nb = A.nbytes
pa, pq, pr = h.host_alloc(nb), h.host_alloc(nb), h.host_alloc(n * n * 4)
np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
Qv = np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(pq))
Rv = np.ctypeslib.as_array((ctypes.c_uint8 * (n * n * 4)).from_address(pr))
stream = torch.cuda.current_stream()
out = {}
for g in (0, 1, 0, 1):
    h.set_option("graph", g)
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h.factor(pa, m, m, n, pq, pr, precision="fp16", budget=a.budget_mib << 20)
        e1.record(stream); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    st = h.stats()
    out[g] = (Qv.copy(), Rv.copy())
    print(f"host graph={g}: ms {np.median(ts):.2f} (min {min(ts):.2f})  replay={st['graph_replay']} captures={st['graph_captures']} "
          f"h2d={st['h2d_bytes']} d2h={st['d2h_bytes']} leaf={st['n_leaf_launches']}", flush=True)
print("host Q bitwise equal:", np.array_equal(out[0][0], out[1][0]), " R bitwise equal:", np.array_equal(out[0][1], out[1][1]))
Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
Qd = torch.empty_like(Ad); Rd = torch.empty((n, n), dtype=torch.float32, device="cuda")
dout = {}
for g in (0, 1, 0, 1):
    h.set_option("graph", g)
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        h.factor_device(Ad, m, m, n, Qd, Rd, precision="fp16")
        e1.record(stream); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    st = h.stats()
    dout[g] = (Qd.clone(), Rd.clone())
    print(f"device graph={g}: ms {np.median(ts):.2f} (min {min(ts):.2f}) replay={st['graph_replay']}", flush=True)
print("device Q bitwise equal:", torch.equal(dout[0][0], dout[1][0]), " R bitwise equal:", torch.equal(dout[0][1], dout[1][1]))
