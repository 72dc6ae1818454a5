"""The paper's OOC GEMM experiments on B200 (section 5.1, Tables 1/2): the largest
inner / outer products of the recursive and the blocking QR at 131072^2 with their tilings (Figs.
3-6), synchronous (one stream, RGSQR_OPT_SERIALIZE) and asynchronous, fp32 host data (TF32 tensor
cores, the paper's fp32 words) and fp16 host data.  Device budget 32 GiB (the paper's V100).

    python scripts/paper_gemm_tables.py [--prec tf32,fp16] [--reps 2]
Writes gpurun_out/paper_gemm_tables.json.  Operands: seeded synthetic values (a repeated seeded
tile; the timing does not depend on them)."""
import argparse
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icpp_zhangw21_b200 import Handle, build  # noqa: E402

GiB = 1 << 30
PAPER = {  # V100 async / sync TFLOPS (Tables 1/2; Q12: trust the TFLOPS cells)
    ("inner", 0): {"async": 87.1, "sync": 62.0}, ("inner", 1): {"async": 43.6, "sync": 33.0},
    ("outer", 0): {"async": 97.7, "sync": 60.3}, ("outer", 1): {"async": 96.2, "sync": 34.7}}
SHAPES = {  # (op, tiling): (w1, m, w2, block)
    ("inner", 0): (65536, 131072, 65536, 16384),     # Table 1 recursive: 65536 x 131072 x 65536, bs 16384
    ("inner", 1): (16384, 131072, 114688, 16384),    # Table 1 blocking: 16384 x 131072 x 114688
    ("outer", 0): (65536, 131072, 65536, 8192),      # Table 2 recursive: 131072 x 65536 x 65536, bs 8192
    ("outer", 1): (16384, 131072, 114688, 16384)}    # Table 2 blocking: 131072 x 16384 x 114688, b1=b2=16384

ap = argparse.ArgumentParser()
ap.add_argument("--prec", default="tf32,fp16")
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--budget-gib", type=int, default=32)
a = ap.parse_args()
build.build()
h = Handle(0)
out = []
for prec in a.prec.split(","):
    s = 4 if prec == "tf32" else 2
    mq = max(m * w1 for (w1, m, w2, b) in SHAPES.values()) * s
    ma = max(m * w2 for (w1, m, w2, b) in SHAPES.values()) * s
    mr = max(w1 * w2 for (w1, m, w2, b) in SHAPES.values()) * 4
    t0 = time.time()
    pq, pa, pr = h.host_alloc(mq), h.host_alloc(ma), h.host_alloc(mr)
    rng = np.random.default_rng(2)
    dt = np.float32 if s == 4 else np.float16
    tile = (rng.standard_normal(1 << 24) * 0.01).astype(dt).view(np.uint8)
    for p_, nb in ((pq, mq), (pa, ma), (pr, mr)):
        buf = np.ctypeslib.as_array((ctypes.c_uint8 * nb).from_address(p_))
        for o in range(0, nb, tile.size):
            k = min(tile.size, nb - o)
            buf[o:o + k] = tile[:k]
    alloc_s = time.time() - t0
    for (op, tiling), (w1, m, w2, block) in SHAPES.items():
        for ser in (0, 1):
            h.set_option("serialize", ser)
            ts = []
            for _ in range(a.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                if op == "inner":
                    h.ooc_inner(pq, m, pa, m, m, w1, w2, pr, w1, precision=prec, tiling=tiling, block=block,
                                budget=a.budget_gib * GiB)
                else:
                    h.ooc_outer(pq, m, pr, w1, pa, m, m, w1, w2, precision=prec, tiling=tiling, block=block,
                                budget=a.budget_gib * GiB)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            st = h.stats()
            ms = min(ts)
            rec = {"gemm": op, "tiling": "recursive" if tiling == 0 else "blocking", "prec": prec,
                   "mode": "sync" if ser else "async", "shape": f"{w1 if op == 'inner' else m}x"
                   f"{m if op == 'inner' else w1}x{w2}", "block": block, "ms": ms,
                   "tflops": 2.0 * w1 * m * w2 / ms / 1e9, "h2d_bytes": st["h2d_bytes"], "d2h_bytes": st["d2h_bytes"],
                   "busy_ms": {"h2d": st["h2d_busy_ms"], "d2h": st["d2h_busy_ms"], "compute": st["compute_busy_ms"]},
                   "overlap_ratio": st["overlap_ratio"], "paper_v100_tflops": PAPER[(op, tiling)]["sync" if ser else "async"]}
            out.append(rec)
            print(json.dumps(rec), flush=True)
    h.set_option("serialize", 0)
    for p_ in (pq, pa, pr):
        h.host_free(p_)
    print(json.dumps({"prec": prec, "host_alloc_fill_s": alloc_s}), flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/paper_gemm_tables.json", "w"), indent=1)
