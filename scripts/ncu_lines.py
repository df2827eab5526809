"""Per-source-line stall samples / instructions of one ncu report (cuda,sass page).
usage: python scripts/ncu_lines.py REPORT [first_line last_line] [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
lo = int(sys.argv[2]) if len(sys.argv) > 3 else 0
hi_l = int(sys.argv[3]) if len(sys.argv) > 3 else 10**9
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr_i = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hdr_i]
idx = {}
for i, k in enumerate(h): idx.setdefault(k, i)
stalls = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
agg = {}
for r in rows[hdr_i + 1:]:
    if len(r) < len(h) or r[0] == "Line No": continue
    try: ln = int(r[0])
    except ValueError: continue
    a = agg.setdefault(ln, {"src": r[1][:70], "smp": 0, "ie": 0, **{s: 0 for s in stalls}})
    def num(k):
        try: return int(float(r[idx[k]] or 0))
        except ValueError: return 0
    a["smp"] += num("Warp Stall Sampling (All Samples)"); a["ie"] += num("Instructions Executed")
    for s in stalls: a[s] += num(s)
tot = sum(a["smp"] for a in agg.values()) or 1
sel = [(ln, a) for ln, a in agg.items() if lo <= ln <= hi_l]
print("selected %.1f%% of samples" % (100 * sum(a["smp"] for _, a in sel) / tot))
for ln, a in sorted(sel, key=lambda x: -x[1]["smp"])[:top]:
    st = sorted(((a[s], s[6:]) for s in stalls), reverse=True)[:3]
    print("%5d %5.1f%% ie=%9d %-70s %s" % (ln, 100 * a["smp"] / tot, a["ie"], a["src"],
          " ".join("%s:%d%%" % (n, 100 * v / max(a["smp"], 1)) for v, n in st if v)))
