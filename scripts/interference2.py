"""Kernel slowdown under concurrent copy-engine traffic: torch bf16 GEMM, an HBM copy kernel and a
pure-ALU kernel, each timed with CUDA events alone and while pinned D2H / H2D copies run."""
import torch, time
torch.backends.cuda.matmul.allow_tf32 = False
a = torch.randn(8192, 8192, device="cuda", dtype=torch.bfloat16); b = torch.randn_like(a)
x = torch.empty(1 << 28, device="cuda", dtype=torch.float32); y = torch.empty_like(x)
hb_in = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_in = torch.empty_like(hb_in, device="cuda")
hb_out = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_out = torch.empty_like(hb_out, device="cuda")
s1, s2, sc = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
z = torch.randn(148 * 1024, device="cuda")
def alu():
    w = z
    for _ in range(200): w = torch.sin(w)  # ~ALU-bound elementwise chain on a small L2-resident tensor
    return w
ops = {"gemm": lambda: a @ b, "hbm_copy": lambda: y.copy_(x), "alu_small": alu}
def timeit(f, copies):
    torch.cuda.synchronize()
    if copies:
        for _ in range(20):
            if copies in ("h2d", "both"):
                with torch.cuda.stream(s1): db_in.copy_(hb_in, non_blocking=True)
            if copies in ("d2h", "both"):
                with torch.cuda.stream(s2): hb_out.copy_(db_out, non_blocking=True)
    with torch.cuda.stream(sc):
        f(); f()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sc)
        for _ in range(10): f()
        e1.record(sc)
    e1.synchronize()
    t = e0.elapsed_time(e1) / 10
    torch.cuda.synchronize()
    return t
for name, f in ops.items():
    for copies in ("", "h2d", "d2h", "both"):
        print(f"{name:10s} copies={copies or 'none':5s} {timeit(f, copies)*1e3:9.1f} us")
