"""Per-kernel table of an ncu launch list (`ncu --metrics gpu__time_duration.sum --csv`).

usage: python tools/launch_table.py launches.csv [launches-per-forward]
Keeps the library's kernels (namespace et::), takes the last `launches-per-forward` of them (one
12-layer C3 forward = 84) and prints count / average / share per (kernel, grid).  ncu serialises the
launches and runs them with cold caches: use the shares, not the absolute times.
"""
import collections
import csv
import sys

path = sys.argv[1]
per_fwd = int(sys.argv[2]) if len(sys.argv) > 2 else 84
rows = []
with open(path) as fh:
    lines = [l for l in fh if l.startswith('"')]
for r in csv.DictReader(lines):
    if r.get("Metric Name") != "gpu__time_duration.sum" or "et::" not in r["Kernel Name"]:
        continue
    scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}[r["Metric Unit"]]
    rows.append((r["Kernel Name"], r["Grid Size"], float(r["Metric Value"].replace(",", "")) * scale))
rows = rows[-per_fwd:]
agg = collections.OrderedDict()
for name, grid, us in rows:
    short = name.split("(")[0].replace("void ", "").replace("(anonymous namespace)", "<unnamed>")
    agg.setdefault((short, grid), []).append(us)
tot = sum(us for _, _, us in rows)
print(f"ncu --metrics gpu__time_duration.sum --clock-control none: last {len(rows)} library launches = one forward")
for (name, grid), v in agg.items():
    print(f"{name[:60]:60s} grid{grid:14s} n={len(v):3d} avg={sum(v) / len(v):7.2f} us share={sum(v) / tot:.3f}")
print(f"total {tot:.1f} us per forward (serialised, cold caches under ncu)")
