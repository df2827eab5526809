"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv):
per-kernel launches, average duration, share of the step (setup kernels
excluded)."""
import collections
import csv
import sys

SETUP = ("gen_kernel", "gen2_kernel", "at::", "widen", "base_kernel")
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 5]
h = rows[0]
ki, mi, vi, ui = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
agg = collections.OrderedDict()
for r in rows[1:]:
    if r[mi] != "gpu__time_duration.sum":
        continue
    v = float(r[vi].replace(",", ""))
    v = v / 1000.0 if r[ui] in ("ns", "nsecond") else v * 1000.0 if r[ui] in ("ms", "msecond") else v
    a = agg.setdefault(r[ki], [0, 0.0])
    a[0] += 1
    a[1] += v
step = sum(t for k, (c, t) in agg.items() if not any(s in k for s in SETUP))
print(sys.argv[2] if len(sys.argv) > 2 else "")
print("cold-cache, serialised launches (us); setup kernels listed but excluded from the step share")
for k, (c, t) in agg.items():
    tag = "setup" if any(s in k for s in SETUP) else f"{100 * t / step:5.1f}% of step"
    print(f"{k[:70]:70s} launches {c:3d}  avg {t / c:10.1f} us  {tag}")
