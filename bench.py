#!/usr/bin/env python
"""Benchmark of the out-of-core recursive CGS QR (BASELINE.json metric: TFLOPS = 2 m n^2 / t,
and the fraction of the min(tensor-peak, host-link) roofline).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c2] [--impl ours|reference]

Workload (N = 1): BASELINE.json configs[1] -- fp16 A 65536 x 8192 Gaussian with the device
budget capped at 1 GiB (out-of-core).

* ``value`` (the metric): rgsqr_factor through the C ABI with A, Q and R in pinned HOST
  memory -- the paper's out-of-core setting: every host->device tile
  upload and Q / R download is inside the timed region (h2d/d2h bytes per step are the
  library's own counters).  CUDA events on the library's compute stream around K
  host-synchronous calls, barrier + synchronize on both sides, max over ranks.
* ``e2e``: the same measurement (the value path already starts from host buffers).
* ``roofline``: the binding host-link term of the north-star roofline (bytes the schedule
  moves over the 2D-tile link bandwidth the library's own copies reach, probed live), i.e.
  max(T_tensor, T_link) / T_wall.
* ``device_resident``: rgsqr_factor_device with A / Q / R already in HBM (workspace <= the
  budget) and its per-kernel-class breakdown; ``kernel_roofline``: the dominant kernel.

N > 1: rows of ONE global (N*65536) x 8192 matrix are sharded over the ranks (row-sharded
NCCL path); the bench fails instead of silently falling back to replicas.
``--impl reference`` times the CPU oracle (fp64 recursive CGS, numpy/OpenBLAS) on a
bounded sample of the same workload; it is a baseline, not the target.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import rgsqr_inputs as gi  # noqa: E402

MiB = 1 << 20
WORKLOADS = {
    "c1": dict(m=4096, n=256, prec="tf32", budget=0,
               desc="in-core TF32 A 4096x256 Gaussian (BASELINE.json configs[0])"),
    "c2": dict(m=65536, n=8192, prec="fp16", budget=1 << 30,
               desc="fp16 A 65536x8192 Gaussian, device budget 1 GiB (out-of-core), 1 GPU (BASELINE.json configs[1])"),
    "c3": dict(m=262144, n=32768, prec="fp16", budget=8 << 30,
               desc="fp16 A 262144x32768 Gaussian, device budget 8 GiB (BASELINE.json configs[2])"),
    # the paper's whole-QR shapes (Table 4; memory-capped simulation PAPER.md:324):
    # fp32 host data on TF32 tensor cores, device capped at 16 GiB, QR blocksize 8192 for --algo blocked
    "t4a": dict(m=65536, n=65536, prec="tf32", budget=16 << 30,
                desc="fp32 A 65536x65536 Gaussian, TF32, device budget 16 GiB (PAPER.md Table 4 shape)"),
    "t4b": dict(m=262144, n=65536, prec="tf32", budget=16 << 30,
                desc="fp32 A 262144x65536 Gaussian, TF32, device budget 16 GiB (PAPER.md Table 4 shape)"),
}
DTYPE_NAME = {"fp16": "f16", "bf16": "bf16", "tf32": "tf32"}
STORAGE = {"fp16": "fp16", "bf16": "bf16", "tf32": "fp32"}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed regions."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []
        self.active = False

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            if self.active:
                self.lines.append(line.strip())

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def link_bandwidth(torch):
    """Pinned host<->device copy bandwidth (GB/s), measured live: H2D, D2H, duplex total."""
    n = 256 * MiB
    h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
    d1 = torch.empty(n, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def timed(fn, nbytes, reps=4):
        fn()
        torch.cuda.synchronize()
        t = time.perf_counter()
        for _ in range(reps):
            fn()
        torch.cuda.synchronize()
        return nbytes * reps / (time.perf_counter() - t) / 1e9

    def duplex():
        with torch.cuda.stream(s1):
            d1.copy_(h1, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        s1.synchronize()
        s2.synchronize()

    out = {"h2d": timed(lambda: d1.copy_(h1, non_blocking=True), n),
           "d2h": timed(lambda: h1.copy_(d1, non_blocking=True), n),
           "duplex_total": timed(duplex, 2 * n)}
    del h1, h2, d1, d2
    return out


def cpu_oracle_sample(A, storage, cols, leaf=64):
    """The oracle's O3 (fp64 recursive CGS, numpy/OpenBLAS) on the first `cols` columns."""
    import oracle
    X = gi.to_float64(np.asarray(A[:, :cols]), storage)
    try:
        from threadpoolctl import threadpool_limits
        ctx = threadpool_limits(limits=len(os.sched_getaffinity(0)))
    except Exception:  # pragma: no cover
        ctx = None
    t = time.perf_counter()
    oracle.rgs(X, leaf=leaf)
    dt = time.perf_counter() - t
    if ctx is not None:
        ctx.unregister() if hasattr(ctx, "unregister") else None
    m = X.shape[0]
    return 2.0 * m * cols * cols / dt / 1e12, dt


METRIC = "OOC QR TFLOPS (2mn^2) and % of min(tensor-peak, PCIe roofline)"


def run_reference(args, wl, rank):
    if rank != 0:
        return
    m, n, prec = wl["m"], wl["n"], wl["prec"]
    # the same 2048-column sample as our arm's cpu_baseline (~9 s per step on 16 cores; the whole
    # configs[1] run is recorded separately in profiles/r2_cpu_oracle_c2.json)
    cols = min(n, 2048)
    A = gi.gaussian(m, cols, seed=2, dtype=STORAGE[prec])
    cores = len(os.sched_getaffinity(0))
    for _ in range(args.warmup):
        cpu_oracle_sample(A, STORAGE[prec], cols)
    vals, times = [], []
    for _ in range(args.steps):
        v, dt = cpu_oracle_sample(A, STORAGE[prec], cols)
        vals.append(v)
        times.append(dt)
    value = float(np.mean(vals))
    sample = (f"oracle O3 (fp64 recursive CGS, numpy/OpenBLAS, leaf 64) on {m}x{cols} "
              f"(first {cols} columns of the {args.workload} input), per step")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": "TFLOPS",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * float(np.mean(times)), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl["desc"], "m": m, "n": n, "precision": prec,
                       "device_budget_bytes": wl["budget"], "sample_cols": cols},
            "cpu_baseline": {"value": value, "unit": "TFLOPS", "cores": cores, "kind": "oracle", "sample": sample,
                             **({"full_c2_measured": json.load(open(os.path.join(ROOT, "profiles", "r2_cpu_oracle_c2.json")))}
                                if args.workload == "c2" and os.path.exists(os.path.join(ROOT, "profiles", "r2_cpu_oracle_c2.json"))
                                else {})},
            "e2e": {"value": value, "unit": "TFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default="c2", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--skip-device", action="store_true", help="skip the HBM-resident secondary measurement")
    ap.add_argument("--algo", default="recursive", choices=["recursive", "blocked"],
                    help="blocked = the paper's conventional blocked OOC CGS (PAPER.md:113), panel 8192")
    ap.add_argument("--no-ablation", action="store_true", help="skip the split-ratio e2e ablation")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3) if args.impl == "ours" else args.warmup
    wl = WORKLOADS[args.workload]
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        run_reference(args, wl, rank)
        return

    import torch
    import torch.distributed as dist
    if world > 1:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_icpp_zhangw21_b200 import Handle, build
    from paper_conf_icpp_zhangw21_b200.rgsqr import KERNEL_CLASSES
    build.build()

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    m, n, prec, budget = wl["m"], wl["n"], wl["prec"], wl["budget"]
    st_name = STORAGE[prec]
    s_bytes = 2 if st_name != "fp32" else 4
    peaks, peak_src = load_peaks()
    parallelism = "single"
    if world > 1:
        # row-sharded: each rank holds m rows of ONE global (m*world) x n factorization; no
        # silent fallback to replicas (a failure to build the distributed context is fatal)
        from paper_conf_icpp_zhangw21_b200 import dist as rdist
        h = rdist.create_handle(local, rank, world)
        parallelism = f"rows sharded over {world} GPUs (R12 ncclAllReduce + in-kernel leaf exchange)"
    else:
        h = Handle(local)
    flops = 2.0 * m * n * n          # per rank's rows; the job's flops are world x this
    stream = torch.cuda.current_stream()
    h.set_stream(stream.cuda_stream)
    if args.algo == "blocked":
        h.set_option("algo", 1)
        h.set_option("block_cols", 8192)
    tf32_peak = json.load(open(os.path.join(ROOT, "profiles", "r2_probe.json"))).get("matmul_tf32_TFLOPs") \
        if os.path.exists(os.path.join(ROOT, "profiles", "r2_probe.json")) else None
    tensor_peak = peaks["bf16_tflops_sustained"] * (1.0 if prec != "tf32" else
                                                    (tf32_peak / peaks["bf16_tflops"] if tf32_peak else 0.5))

    # ---- input (host, seeded; rank r holds global rows [r m, (r+1) m)) ----
    A = gi.gaussian(m, n, seed=2, dtype=st_name, row0=rank * ((m + gi.ROW_BLOCK - 1) // gi.ROW_BLOCK) * gi.ROW_BLOCK)
    clocks = ClockSampler(local)
    clocks.start()
    import ctypes
    nbytes = A.nbytes
    pa, pq, pr = h.host_alloc(nbytes), h.host_alloc(nbytes), h.host_alloc(n * n * 4)
    np.ctypeslib.as_array((ctypes.c_uint8 * nbytes).from_address(pa))[:] = A.reshape(-1, order="F").view(np.uint8)
    lda = m

    # ---- host link: the executor's own 2D copies (in-core column chunks and ring row tiles) ----
    link_geoms = {"columns": h.probe_link(pq, lda, m, min(n, (64 << 20) // (m * s_bytes)), s_bytes),
                  "tile_16384": h.probe_link(pq, lda, min(m, 16384), min(n, 2048), s_bytes)}
    link = {k: max(g[k] for g in link_geoms.values()) for k in ("h2d", "d2h", "duplex_total")}

    # ---- value: host-resident (out-of-core) through rgsqr_factor, pinned host buffers ----
    for _ in range(args.warmup):
        h.factor(pa, lda, m, n, pq, pr, precision=prec, budget=budget)
    barrier()
    torch.cuda.synchronize()
    clocks.active = True
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(args.steps):
        h.factor(pa, lda, m, n, pq, pr, precision=prec, budget=budget)
    e1.record(stream)
    torch.cuda.synchronize()
    clocks.active = False
    barrier()
    ms = max_over_ranks(e0.elapsed_time(e1) / args.steps)
    so = h.stats()
    value = world * flops / (ms / 1e3) / 1e12
    launches_per_step = sum(so[k] for k in ("n_leaf_launches", "n_tn_launches", "n_nn_launches", "n_other_launches"))
    t_tensor = flops / (tensor_peak * 1e12)
    terms = {"h2d": (so["h2d_bytes"], link["h2d"]), "d2h": (so["d2h_bytes"], link["d2h"]),
             "duplex": (so["h2d_bytes"] + so["d2h_bytes"], link["duplex_total"])}
    bind = max(terms, key=lambda k: terms[k][0] / terms[k][1])
    t_link = terms[bind][0] / (terms[bind][1] * 1e9)
    roof = {"bound": "pcie" if t_link >= t_tensor else "tensor",
            "achieved": terms[bind][0] / (ms / 1e3) / 1e9, "peak": terms[bind][1], "unit": "GB/s",
            "frac": max(t_tensor, t_link) / (ms / 1e3),
            "traffic": so["h2d_bytes"] + so["d2h_bytes"],
            "binding_term": bind, "t_link_ms": 1e3 * t_link, "t_tensor_ms": 1e3 * t_tensor,
            "peak_source": "host link probed live with the library's own cudaMemcpy2DAsync tile copies "
                           "(rgsqr_probe_link; best of the in-core column-chunk and 16384-row ring-tile "
                           "geometries); T_tensor against MEASURED_PEAKS.json bf16 sustained",
            "link_gbps_measured": link_geoms,
            "compulsory_bytes": {"h2d": m * n * s_bytes, "d2h": m * n * s_bytes + 2 * n * (n + 1)},
            "frac_vs_compulsory": max(t_tensor, max(m * n * s_bytes / (link["h2d"] * 1e9),
                                                    (m * n * s_bytes + 2 * n * (n + 1)) / (link["d2h"] * 1e9),
                                                    (2 * m * n * s_bytes + 2 * n * (n + 1)) /
                                                    (link["duplex_total"] * 1e9))) / (ms / 1e3)}
    e2e = {"value": value, "unit": "TFLOPS", "ms_per_step": ms,
           "h2d_bytes_per_step": so["h2d_bytes"], "d2h_bytes_per_step": so["d2h_bytes"],
           "path": "rgsqr_factor (C ABI), A/Q/R in pinned host memory, budget %d MiB (same run as value)"
                   % (budget // MiB),
           "graph_replay": bool(so["graph_replay"]),
           "ooc_nodes": so["n_ooc_nodes"], "arena_bytes": so["arena_bytes"],
           "ctx_device_bytes": so["ctx_device_bytes"], "colchunk_nodes": so["n_colchunk_nodes"],
           "arena_high_water": so["arena_high_water"]}
    # per-stream busy times / overlap ratio: not measured inside a replayed CUDA graph, so one
    # untimed eager call of the same schedule (RGSQR_OPT_GRAPH = 0) reports them
    h.set_option("graph", 0)
    h.factor(pa, lda, m, n, pq, pr, precision=prec, budget=budget)
    torch.cuda.synchronize()
    se = h.stats()
    h.set_option("graph", 1)
    e2e["eager_diagnostic"] = {"wall_ms": se["wall_ms"], "overlap_ratio": se["overlap_ratio"],
                               "busy_ms": {"h2d": se["h2d_busy_ms"], "d2h": se["d2h_busy_ms"],
                                           "compute": se["compute_busy_ms"]},
                               "note": "one untimed call with eager launches (RGSQR_OPT_GRAPH=0); the timed "
                                       "steps replay the captured CUDA graph (DESIGN.md R30)"}
    # ablation (not the headline): OOC left child 62.5% of the columns instead of the paper's halves
    if world == 1 and not args.no_ablation:
        h.set_option("split_pct", 62)
        h.factor(pa, lda, m, n, pq, pr, precision=prec, budget=budget)
        torch.cuda.synchronize()
        a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(stream)
        for _ in range(2):
            h.factor(pa, lda, m, n, pq, pr, precision=prec, budget=budget)
        a1.record(stream)
        torch.cuda.synchronize()
        ms_ab = a0.elapsed_time(a1) / 2
        e2e["ablation_split_pct_62"] = {"value": flops / (ms_ab / 1e3) / 1e12, "ms_per_step": ms_ab}
        h.set_option("split_pct", 50)

    # ---- secondary: device-resident factorization (A / Q / R in HBM) and its kernels ----
    dev = None
    kroof = None
    if not args.skip_device:
        tdt = {"fp16": torch.float16, "bf16": torch.bfloat16, "fp32": torch.float32}[st_name]
        at_host = torch.from_numpy(np.ascontiguousarray(A.T).view(np.int16 if st_name == "bf16" else A.dtype))
        if st_name == "bf16":
            at_host = at_host.view(torch.bfloat16)
        Ad = at_host.to("cuda")
        Qd = torch.empty_like(Ad)
        Rd = torch.empty((n, n), dtype=torch.float32, device="cuda")
        for _ in range(args.warmup):
            h.factor_device(Ad, m, m, n, Qd, Rd, precision=prec, budget=budget)
        barrier()
        torch.cuda.synchronize()
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        clocks.active = True
        ev0.record(stream)
        for _ in range(args.steps):
            h.factor_device(Ad, m, m, n, Qd, Rd, precision=prec, budget=budget)
        ev1.record(stream)
        torch.cuda.synchronize()
        clocks.active = False
        barrier()
        ms_dev = max_over_ranks(ev0.elapsed_time(ev1) / args.steps)
        h.set_option("profile", 1)
        h.factor_device(Ad, m, m, n, Qd, Rd, precision=prec, budget=budget)
        prof = h.stats()
        h.set_option("profile", 0)
        kms = prof["kern_ms"]
        dom = int(np.argmax(kms))
        dom_name = KERNEL_CLASSES[dom]
        if dom_name in ("inner", "outer"):
            achieved = prof["kern_flops"][dom] / (kms[dom] / 1e3) / 1e12
            kroof = {"bound": "tensor", "achieved": achieved, "peak": tensor_peak, "unit": "TFLOP/s"}
        else:
            achieved = prof["kern_bytes"][dom] / (kms[dom] / 1e3) / 1e9
            kroof = {"bound": "hbm", "achieved": achieved, "peak": peaks["hbm_gbs"], "unit": "GB/s"}
        kroof["frac"] = kroof["achieved"] / kroof["peak"]
        kroof["kernel"] = dom_name
        kroof["peak_source"] = f"{peak_src} (MEASURED_PEAKS.json)"
        tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        kroof["traffic"] = json.load(open(tp)).get(args.workload, {}).get(dom_name) if os.path.exists(tp) else None
        kroof["share_of_step"] = kms[dom] / sum(kms) if sum(kms) else None
        if dom_name == "leaf":
            us_col = kms[dom] * 1e3 / n
            floor = 0.914
            kroof["latency"] = {"unit": "us per column", "achieved": us_col, "floor": floor, "frac": floor / us_col,
                                "floor_source": "exchange-only round of 148 CTAs, measured on B200 (crit_bench V12)"}
        kernels = {KERNEL_CLASSES[i]: {"ms": kms[i], "launches": prof["kern_launches"][i],
                                       "tflops": (prof["kern_flops"][i] / (kms[i] / 1e3) / 1e12) if kms[i] else None,
                                       "gbps": (prof["kern_bytes"][i] / (kms[i] / 1e3) / 1e9) if kms[i] else None}
                   for i in range(4)}
        dev = {"value": world * flops / (ms_dev / 1e3) / 1e12, "unit": "TFLOPS", "ms_per_step": ms_dev,
               "path": "rgsqr_factor_device: A/Q/R resident in HBM, library workspace <= budget",
               "kernels": kernels, "kernel_timing": "per-kernel CUDA events in one profiled step after the timed region"}
        del Ad, Qd, Rd
    for p_ in (pa, pq, pr):
        h.host_free(p_)
    clocks.stop()

    # ---- CPU baseline: the oracle on a bounded sample (rank 0, N = 1) ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cols = 2048 if m >= 65536 else n          # ~10-20 s of fp64 CGS on the host cores
        v, dt = cpu_oracle_sample(A, st_name, cols)
        cpu = {"value": v, "unit": "TFLOPS", "cores": len(os.sched_getaffinity(0)), "kind": "oracle",
               "sample": f"oracle O3 (fp64 recursive CGS, numpy/OpenBLAS) on {m}x{cols} (first {cols} columns "
                         f"of the same input), {dt:.1f} s; extrapolated to the full {m}x{n} at this rate: "
                         f"{2.0 * m * n * n / (v * 1e12):.0f} s (the rate grows with n, so this over-states "
                         f"the CPU time)"}
        full = os.path.join(ROOT, "profiles", "r2_cpu_oracle_c2.json")
        if os.path.exists(full) and args.workload == "c2":
            cpu["full_c2_measured"] = json.load(open(full))

    if rank == 0:
        line = {"metric": METRIC,
                "value": value, "unit": "TFLOPS", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
                "dtype": DTYPE_NAME[prec], "data": "synthetic",
                "config": {"workload": wl["desc"], "m": m, "n": n, "precision": prec, "device_budget_bytes": budget,
                           "value_path": "rgsqr_factor: A/Q/R in pinned host memory, out-of-core under the budget",
                           "l2": "inputs (>= 1 GiB) larger than L2 (126 MB); no flush needed",
                           "parallelism": parallelism, "m_global": m * world, "algo": args.algo},
                "roofline": roof, "e2e": e2e, "device_resident": dev, "kernel_roofline": kroof,
                "cpu_baseline": cpu, "gpu_launches": args.steps * launches_per_step, "clocks": clocks.summary()}
        print(json.dumps(line), flush=True)
    h.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
