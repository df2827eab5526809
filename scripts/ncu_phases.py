"""Aggregate ncu source-level samples/instructions of eval2 by phase (line ranges)."""
import csv, io, subprocess, sys, re
rep = sys.argv[1]
src_file = "paper_conf_asplos_chend0zll024_b200/csrc/magis_eval2.cu"
lines = open(src_file).read().splitlines()
marks = []
for i, l in enumerate(lines, 1):
    m = re.search(r"// (=+ (latency sweep|main warps)|---- phase \d)", l)
    if m:
        marks.append((i, m.group(1).strip("= ")))
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
src = list(csv.reader(io.StringIO(out)))
hi = [i for i, r in enumerate(src) if r and r[0] == "Line No"][0]
hdr = src[hi]; idx = {}
for i, k in enumerate(hdr): idx.setdefault(k, i)
agg = {}
cur_file_ok = True
for r in src[hi + 1:]:
    if len(r) < 10 or not r[0]: continue
    try:
        ln = int(r[0]); ie = int(r[idx["Instructions Executed"]]); smp = int(r[idx["Warp Stall Sampling (All Samples)"]])
        wf = int(r[idx["L1 Wavefronts Shared"]] or 0)
    except Exception: continue
    name = "helpers/other"
    for (l0, nm) in marks:
        if ln >= l0: name = nm
    if ln > len(lines) or ln < marks[0][0]: name = "helpers/other"
    a = agg.setdefault(name, [0, 0, 0]); a[0] += smp; a[1] += ie; a[2] += wf
ts = sum(v[0] for v in agg.values()); ti = sum(v[1] for v in agg.values()); tw = sum(v[2] for v in agg.values())
for k, v in sorted(agg.items(), key=lambda x: -x[1][0]):
    print(f"{k:28s} samples {100*v[0]/ts:5.1f}%  instr {100*v[1]/ti:5.1f}%  smem wf {100*v[2]/max(tw,1):5.1f}%")
