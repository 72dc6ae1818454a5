"""Phase-0 probes on the GPU box: host link bandwidth (pinned, 1D and 2D strided,
H2D / D2H / duplex), tensor-core peaks via torch.matmul, host RAM / cores.
Writes gpurun_out/probe.json."""
import json
import os
import subprocess
import time

import torch


def bw(fn, nbytes, reps=10):
    fn()
    torch.cuda.synchronize()
    s = torch.cuda.Event(enable_timing=True)
    e = torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps):
        fn()
    e.record()
    torch.cuda.synchronize()
    return nbytes * reps / (s.elapsed_time(e) / 1e3) / 1e9


def main():
    out = {}
    out["cpu_count"] = os.cpu_count()
    out["affinity"] = len(os.sched_getaffinity(0))
    with open("/proc/meminfo") as f:
        out["meminfo"] = {l.split(":")[0]: l.split(":")[1].strip() for l in f if l.split(":")[0] in ("MemTotal", "MemAvailable")}
    try:
        out["topo"] = subprocess.run(["nvidia-smi", "topo", "-m"], capture_output=True, text=True).stdout
        out["lscpu"] = subprocess.run(["lscpu"], capture_output=True, text=True).stdout[:1500]
    except Exception as ex:
        out["topo"] = str(ex)
    dev = torch.device("cuda")
    N = 1 << 30
    h = torch.empty(N, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(N, dtype=torch.uint8).pin_memory()
    d = torch.empty(N, dtype=torch.uint8, device=dev)
    d2 = torch.empty(N, dtype=torch.uint8, device=dev)
    s1 = torch.cuda.Stream()
    s2 = torch.cuda.Stream()
    out["h2d_GBps_1GiB"] = bw(lambda: d.copy_(h, non_blocking=True), N)
    out["d2h_GBps_1GiB"] = bw(lambda: h.copy_(d, non_blocking=True), N)

    def duplex():
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.current_stream().wait_stream(s1)
        torch.cuda.current_stream().wait_stream(s2)
    out["duplex_GBps_total"] = bw(duplex, 2 * N)
    # 2D strided: tile of t rows x w cols from a column-major m x n fp16 matrix
    m = 65536
    for t in (2048, 4096, 8192, 16384):
        w = (N // 2) // m
        hv = h[: m * w * 2].view(torch.float16).view(w, m)
        dv = d[: t * w * 2].view(torch.float16).view(w, t)
        out[f"h2d_2d_GBps_t{t}"] = bw(lambda: dv.copy_(hv[:, :t], non_blocking=True), t * w * 2)
        out[f"d2h_2d_GBps_t{t}"] = bw(lambda: hv[:, :t].copy_(dv, non_blocking=True), t * w * 2)
    # tensor peaks
    for name, dt, tf32 in (("fp16", torch.float16, False), ("bf16", torch.bfloat16, False), ("tf32", torch.float32, True)):
        torch.backends.cuda.matmul.allow_tf32 = tf32
        a = torch.randn(8192, 8192, device=dev, dtype=dt)
        b = torch.randn(8192, 8192, device=dev, dtype=dt)
        fl = 2 * 8192 ** 3
        out[f"matmul_{name}_TFLOPs"] = bw(lambda: torch.mm(a, b), fl, reps=20) / 1e3
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k not in ("topo", "lscpu")}, indent=1))


if __name__ == "__main__":
    main()
