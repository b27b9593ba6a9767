"""Aggregate ncu source-page stall samples per CUDA source line (cuda,sass view).
usage: python tools/ncu_lines.py REP [kernel-index] [top-n]"""
import collections, csv, subprocess, sys

def num(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


rep = sys.argv[1]
kidx = int(sys.argv[2]) if len(sys.argv) > 2 else 0
topn = int(sys.argv[3]) if len(sys.argv) > 3 else 40
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
kernels, cur = [], None
for r in csv.reader(txt.splitlines()):
    if not r:
        continue
    if r[0] == "File Path":
        fpath = r[1]
        continue
    if r[0] == "Function Name":
        cur = {"name": r[1], "rows": [], "hdr": None, "file": fpath.split("/")[-1]}
        kernels.append(cur)
        continue
    if r[0] == "Line No":
        cur["hdr"] = r
        continue
    if cur is not None and cur["hdr"] and len(r) == len(cur["hdr"]):
        cur["rows"].append(r)
# the same function may appear once per file; merge those with equal name
byname = collections.OrderedDict()
for k in kernels:
    byname.setdefault(k["name"], []).append(k)
names = list(byname)
name = names[kidx]
print("kernel:", name[:120])
agg = collections.defaultdict(lambda: collections.Counter())
src = {}
for k in byname[name]:
    h = k["hdr"]
    iall = h.index("Warp Stall Sampling (All Samples)")
    iexe = h.index("Instructions Executed")
    stalls = [(i, c) for i, c in enumerate(h) if c.startswith("stall_") and "(Not" not in c]
    line = None
    for r in k["rows"]:
        if r[0]:
            line = (k["file"], int(r[0]))
            src[line] = r[1].strip()
            continue
        if r[2] in ("", "-"):
            continue
        c = agg[line]
        c["samples"] += num(r[iall])
        c["inst"] += num(r[iexe])
        for i, s in stalls:
            c[s[6:]] += num(r[i])
tot = sum(c["samples"] for c in agg.values()) or 1
tinst = sum(c["inst"] for c in agg.values()) or 1
print(f"total samples {tot:.0f}, warp-instructions {tinst:.0f}")
for line, c in sorted(agg.items(), key=lambda x: -x[1]["samples"])[:topn]:
    rs = sorted(((k, v) for k, v in c.items() if k not in ("samples", "inst")), key=lambda x: -x[1])[:3]
    rs = " ".join(f"{k}:{100 * v / tot:.1f}" for k, v in rs)
    print(f"{line[0][:10]:>10}:{line[1]:<4} {100 * c['samples'] / tot:5.1f}% i{100 * c['inst'] / tinst:5.1f}% {src.get(line, '')[:60]:60s} {rs}")
