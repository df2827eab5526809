"""Per-source-line instructions / stall samples / shared wavefronts of the
eval2 kernel from an ncu report.  usage: python scripts/ncu_lines.py REPORT K [N]"""
import csv, io, subprocess, sys

rep, K = sys.argv[1], int(sys.argv[2])
N = int(sys.argv[3]) if len(sys.argv) > 3 else 50
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hi]
ie, sm = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
wf, wi = h.index("L1 Wavefronts Shared"), h.index("L1 Wavefronts Shared Ideal")
agg, src = {}, {}
for r in rows[hi + 1:]:
    if len(r) < len(h):
        continue
    try:
        ln = int(r[0])
    except ValueError:
        continue
    a = agg.setdefault(ln, [0.0] * 4)
    for j, col in enumerate((ie, sm, wf, wi)):
        try:
            a[j] += float(r[col] or 0)
        except ValueError:
            pass
    if r[1]:
        src[ln] = r[1]
T = sum(v[0] for v in agg.values()) or 1
S = sum(v[1] for v in agg.values()) or 1
print("total warp-inst / candidate %.0f" % (T / K))
for ln, (x, y, w, wi_) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:N]:
    print("%7.0f %5.1f%% smp %5.1f%% wf %6.0f/%6.0f L%4d %s" % (x / K, 100 * x / T, 100 * y / S, w / K, wi_ / K, ln,
                                                              src.get(ln, "").strip()[:90]))
