"""Stall reasons of the eval2 kernel from an ncu report: totals, and the
top source lines with their dominant reasons.  usage: python scripts/ncu_stalls.py REPORT [N]"""
import csv, io, subprocess, sys

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hi]
cols = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
idx = {c: h.index(c) for c in cols}
tot = {c: 0.0 for c in cols}
per, src = {}, {}
for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    try:
        ln = int(r[0])
    except ValueError:
        continue
    a = per.setdefault(ln, {c: 0.0 for c in cols})
    for c in cols:
        try:
            v = float(r[idx[c]] or 0)
        except ValueError:
            v = 0.0
        a[c] += v
        tot[c] += v
    if r[1]:
        src[ln] = r[1]
T = sum(tot.values()) or 1
print("totals: " + ", ".join("%s %.1f%%" % (c[6:], 100 * v / T) for c, v in sorted(tot.items(), key=lambda x: -x[1]) if v / T > 0.005))
for ln, a in sorted(per.items(), key=lambda kv: -sum(kv[1].values()))[:N]:
    s = sum(a.values())
    top = sorted(a.items(), key=lambda x: -x[1])[:3]
    print("%5.1f%% L%4d %-28s %s" % (100 * s / T, ln, " ".join("%s:%.0f%%" % (c[6:], 100 * v / s) for c, v in top if v),
                                   src.get(ln, "").strip()[:80]))
