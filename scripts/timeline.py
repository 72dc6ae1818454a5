"""Coarse per-stream occupancy of an RGSQR_TIMELINE csv (2 ms buckets)."""
import collections
import csv
import math
import sys

rows = list(csv.DictReader(open(sys.argv[1])))
B = float(sys.argv[2]) if len(sys.argv) > 2 else 2.0
busy = collections.defaultdict(float)
for r in rows:
    busy[r["stream"]] += float(r["end_ms"]) - float(r["start_ms"])
end = max(float(r["end_ms"]) for r in rows)
print({k: round(v, 2) for k, v in busy.items()}, "end", round(end, 2))
nb = int(math.ceil(end / B))
occ = {s: [0.0] * nb for s in busy}
for r in rows:
    a, b = float(r["start_ms"]), float(r["end_ms"])
    i = int(a // B)
    while a < b and i < nb:
        e = min(b, (i + 1) * B)
        occ[r["stream"]][i] += e - a
        a = e
        i += 1
for i in range(nb):
    print(f"{i * B:6.1f}", " ".join(f"{s}:{occ[s][i] / B:4.2f}" for s in sorted(occ)))
