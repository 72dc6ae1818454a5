"""Leaf phase breakdown (RGSQR_LEAF_DEBUG=<cta> / RGSQR_LEAF_DEBUG2=1 print per-phase cycles to stderr)
and warm per-launch time with CUDA events at a given panel height."""
import argparse, sys
sys.path.insert(0, "/root/repo")
import numpy as np, torch
import rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import Handle

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=65536)
ap.add_argument("--w", type=int, default=64)
ap.add_argument("--reps", type=int, default=20)
ap.add_argument("--prec", default="fp16")
a = ap.parse_args()
st = {"fp16": torch.float16, "bf16": torch.bfloat16, "tf32": torch.float32}[a.prec]
h = Handle(0)
A = torch.randn(a.w, a.m, device="cuda").to(st)
P = A.clone()
R = torch.zeros(a.w, a.w, device="cuda")
for _ in range(3):
    P.copy_(A); h.op_leaf(P, a.m, a.m, a.w, R, a.w, precision=a.prec)
torch.cuda.synchronize()
ts = []
for _ in range(a.reps):
    P.copy_(A)
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(); h.op_leaf(P, a.m, a.m, a.w, R, a.w, precision=a.prec); e1.record()
    torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1) * 1e3)
print(f"leaf m={a.m} w={a.w} {a.prec}: median {np.median(ts):.1f} us min {min(ts):.1f} us  ({np.median(ts)/a.w:.3f} us/col)")
