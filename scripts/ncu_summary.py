"""Summarise an ncu report: headline metrics + hottest source lines."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25


def run(args):
    return subprocess.run(["ncu", "-i", rep] + args, capture_output=True, text=True).stdout


det = list(csv.reader(io.StringIO(run(["--page", "details", "--csv"]))))
h = det[0]
keep = ["Duration", "Elapsed Cycles", "DRAM Throughput", "Memory Throughput", "L1/TEX Cache Throughput",
        "Compute (SM) Throughput", "Executed Ipc Active", "Issue Slots Busy", "Achieved Active Warps Per SM",
        "Theoretical Occupancy", "Registers Per Thread", "Dynamic Shared Memory Per Block",
        "Executed Instructions", "Warp Cycles Per Issued Instruction", "Avg. Active Threads Per Warp",
        "Branch Efficiency", "L2 Hit Rate", "L1/TEX Hit Rate", "Mem Pipes Busy"]
for row in det[1:]:
    d = dict(zip(h, row))
    if d.get("Metric Name") in keep:
        print(f"{d['Metric Name']:40s} {d['Metric Value']:>16s} {d.get('Metric Unit','')}")
raw = list(csv.reader(io.StringIO(run(["--page", "raw", "--csv"]))))
hr, units, vals = raw[0], raw[1], raw[2]
for k in ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
          "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
          "smsp__thread_inst_executed_per_inst_executed.ratio",
          "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed_pipe_lsu.sum",
          "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__time_duration.sum"]:
    if k in hr:
        i = hr.index(k)
        print(f"{k:60s} {vals[i]:>18s} {units[i]}")
src = list(csv.reader(io.StringIO(run(["--page", "source", "--csv", "--print-source", "cuda,sass"]))))
hi = [i for i, r in enumerate(src) if r and r[0] == "Line No"]
if hi:
    hdr = src[hi[0]]
    idx = {}
    for i, k in enumerate(hdr):
        idx.setdefault(k, i)
    data = []
    for r in src[hi[0] + 1:]:
        if len(r) < 10 or not r[0]:
            continue
        try:
            ie = int(r[idx["Instructions Executed"]])
            smp = int(r[idx["Warp Stall Sampling (All Samples)"]])
        except Exception:
            continue
        data.append((smp, ie, r[0], r[1][:90], r[idx.get("L1 Wavefronts Shared", 0)],
                     r[idx.get("L1 Wavefronts Shared Ideal", 0)]))
    ts = sum(d[0] for d in data) or 1
    ti = sum(d[1] for d in data) or 1
    print(f"\nsource lines by stall samples (total {ts}), instructions {ti}")
    for d in sorted(data, reverse=True)[:top]:
        print(f"{100*d[0]/ts:5.1f}% smp {100*d[1]/ti:5.1f}% inst L{d[2]:>4} {d[3]:90s} wf={d[4]} ideal={d[5]}")
