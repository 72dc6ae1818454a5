"""Time the oracle O3 (fp64 recursive CGS, numpy/OpenBLAS, all host cores) on the WHOLE
configs[1] input (fp16 65536 x 8192, seed 2 -- bench.py's matrix): the cpu_baseline
extrapolation check.  Writes gpurun_out/cpu_oracle_c2.json."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import rgsqr_inputs as gi  # noqa: E402

m, n = 65536, 8192
A = gi.gaussian(m, n, seed=2, dtype="fp16")
X = gi.to_float64(A, "fp16")
del A
t = time.perf_counter()
res = oracle.rgs(X, leaf=64)
dt = time.perf_counter() - t
out = {"m": m, "n": n, "seconds": dt, "tflops": 2.0 * m * n * n / dt / 1e12, "cores": len(os.sched_getaffinity(0)),
       "what": "oracle O3 (fp64 recursive CGS, leaf 64, numpy/OpenBLAS) on the whole configs[1] input (seed 2)"}
try:
    import subprocess
    out["cpu"] = [l for l in subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines()
                  if l.startswith("Model name")][0]
except Exception:
    pass
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/cpu_oracle_c2.json", "w"), indent=1)
print(json.dumps(out))
