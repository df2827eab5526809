"""Instructions / stall samples per kernel phase of magis_eval2.cu from an ncu
report (source page), phases located by their comment markers in the source.
usage: python scripts/ncu_phases.py REPORT [K]"""
import csv, io, re, subprocess, sys

rep = sys.argv[1]
K = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"][0]
h = rows[hi]
ie, sm = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
agg = {}
for r in rows[hi + 1:]:
    if len(r) < len(h) or r[0] == "Line No":
        continue
    try:
        ln = int(r[0])
    except ValueError:
        continue
    a = agg.setdefault(ln, [0, 0])
    for j, col in ((0, ie), (1, sm)):
        try:
            a[j] += int(float(r[col] or 0))
        except ValueError:
            pass
src = open("paper_conf_asplos_chend0zll024_b200/csrc/magis_eval2_kernel.cuh").read().split("\n")
marks = [("helpers", r"^// -+ packed u16"), ("latency helpers", r"^// The event steps of a swapping"),
         ("kernel setup", r"^template <int P, int LMAX, int MODE, int TEAMS>"),
         ("latency warps", r"latency warps \(reading P7\)"), ("main setup", r"= main warps ="),
         ("ph0 decisions", r"---- phase 0"), ("ph1 scatter", r"---- phase 1"), ("ph2 optional", r"---- phase 2"),
         ("ph3 rows", r"---- phase 3"), ("status/marks", r"per-candidate status, 4 bits"),
         ("ph5 scan", r"---- phase 5"), ("ph6 hand-off", r"---- phase 6"), ("ph7 clear", r"clear pos and the event marks"),
         ("host", r"^template <int P, int MODE, int TEAMS>")]
starts = []
for name, pat in marks:
    for i, l in enumerate(src):
        if re.search(pat, l):
            starts.append((i + 1, name))
            break
starts.sort()
T = sum(a[0] for a in agg.values()) or 1
S = sum(a[1] for a in agg.values()) or 1
for k, (s0, name) in enumerate(starts):
    s1 = starts[k + 1][0] if k + 1 < len(starts) else 10**9
    x = sum(v[0] for l, v in agg.items() if s0 <= l < s1)
    y = sum(v[1] for l, v in agg.items() if s0 <= l < s1)
    print("%-16s inst %5.1f%% (%6.0f warp-inst / candidate)  stall samples %5.1f%%" % (name, 100 * x / T, x / K, 100 * y / S))
print("total warp-instructions per candidate: %.0f" % (T / K))
