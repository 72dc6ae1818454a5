"""Does concurrent host<->device copy traffic slow the device-resident factorization's kernels?
Times rgsqr_factor_device (configs[1]) alone and while two side streams run pinned H2D / D2H copies."""
import sys, threading
sys.path.insert(0, "/root/repo")
import numpy as np, torch
import rgsqr_inputs as gi
from paper_conf_icpp_zhangw21_b200 import Handle

m, n = 65536, 8192
A = gi.gaussian(m, n, seed=2, dtype="fp16")
Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda()
Qd = torch.empty_like(Ad); Rd = torch.empty((n, n), dtype=torch.float32, device="cuda")
h = Handle(0); h.set_option("profile", 1)
hb_in = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_in = torch.empty_like(hb_in, device="cuda")
hb_out = torch.empty(256 << 20, dtype=torch.uint8).pin_memory(); db_out = torch.empty_like(hb_out, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

import pynvml
pynvml.nvmlInit()
dev = pynvml.nvmlDeviceGetHandleByIndex(0)
clk = []
stop = False
def sampler():
    while not stop:
        clk.append(pynvml.nvmlDeviceGetClockInfo(dev, pynvml.NVML_CLOCK_SM))
threading.Thread(target=sampler, daemon=True).start()

def run(copies):
    if copies:
        for _ in range(12):
            if copies in ("h2d", "both"):
                with torch.cuda.stream(s1): db_in.copy_(hb_in, non_blocking=True)
            if copies in ("d2h", "both"):
                with torch.cuda.stream(s2): hb_out.copy_(db_out, non_blocking=True)
    clk.clear()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    h.factor_device(Ad, m, m, n, Qd, Rd, precision="fp16")
    e1.record(); torch.cuda.synchronize()
    st = h.stats()
    return e0.elapsed_time(e1), [round(x, 2) for x in st["kern_ms"]], (min(clk) if clk else 0, int(np.median(clk)) if clk else 0)

for _ in range(2): run(False)
for copies in ("", "h2d", "d2h", "both", "", "both"):
    t, k, c = run(copies)
    print(f"copies={copies or 'none'}: {t:.2f} ms  kern_ms leaf/inner/outer/other {k} sum {sum(k):.2f}  sm clock min/median {c}")
stop = True
