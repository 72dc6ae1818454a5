"""Launch-bound chains under copy-engine traffic: eager launches vs one CUDA graph; and the leaf kernel."""
import sys
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_icpp_zhangw21_b200 import Handle
hb_in = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_in = torch.empty_like(hb_in, device="cuda")
hb_out = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_out = torch.empty_like(hb_out, device="cuda")
s1, s2, sc = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
z = torch.randn(148 * 1024, device="cuda")
def alu():
    w = z
    for _ in range(200): w = torch.sin(w)
    return w
with torch.cuda.stream(sc):
    alu(); torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=sc):
        alu()
h = Handle(0)
m, w = 65536, 64
P0 = torch.randn(w, m, device="cuda").half(); P = P0.clone(); R = torch.zeros(w, w, device="cuda")
def leaf():
    for _ in range(8):
        h.op_leaf(P, m, m, w, R, w, precision="fp16")
ops = {"alu_eager": alu, "alu_graph": lambda: g.replay()}
def bg(copies):
    for _ in range(20):
        if copies in ("h2d", "both"):
            with torch.cuda.stream(s1): db_in.copy_(hb_in, non_blocking=True)
        if copies in ("d2h", "both"):
            with torch.cuda.stream(s2): hb_out.copy_(db_out, non_blocking=True)
def timeit(f, copies):
    torch.cuda.synchronize()
    bg(copies)
    with torch.cuda.stream(sc):
        f()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sc)
        for _ in range(5): f()
        e1.record(sc)
    e1.synchronize()
    t = e0.elapsed_time(e1) / 5
    torch.cuda.synchronize()
    return t
h.set_stream(sc.cuda_stream) if hasattr(h, "set_stream") else None
for name, f in ops.items():
    for copies in ("", "h2d", "d2h", "both"):
        print(f"{name:10s} copies={copies or 'none':5s} {timeit(f, copies)*1e3:9.1f} us")
