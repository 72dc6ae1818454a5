"""Summarise an ncu --csv launch list (gpu__time_duration.sum): total / count / mean per kernel + grid."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[start]
agg = collections.defaultdict(lambda: [0, 0.0])
total = 0.0
for r in rows[start + 1:]:
    if len(r) < len(hdr):
        continue
    x = dict(zip(hdr, r))
    if x["Metric Name"] != "gpu__time_duration.sum":
        continue
    unit = x["Metric Unit"]
    v = float(x["Metric Value"].replace(",", "")) * {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0,
                                                    "ms": 1e3, "msecond": 1e3}.get(unit, 1.0)   # -> us
    k = x["Kernel Name"].split("(")[0].replace("void ", "") + " grid" + x["Grid Size"]
    agg[k][0] += 1
    agg[k][1] += v
    total += v
print(f"total {total / 1e3:.3f} ms over {sum(a[0] for a in agg.values())} launches")
print("| kernel | grid | launches | total ms | avg us | share |")
print("|---|---|---|---|---|---|")
for k, (n, t) in sorted(agg.items(), key=lambda z: -z[1][1]):
    name, grid = k.rsplit(" grid", 1)
    print(f"| `{name}` | {grid} | {n} | {t / 1e3:.3f} | {t / n:.1f} | {100 * t / total:.1f}% |")
