#!/bin/bash
# Phase profile (MAGIS_PROFILE) of the variant-2 kernel on each config + a C2 bench line.
mkdir -p gpurun_out
MAGIS_DEBUG=1 MAGIS_PROFILE=1 timeout 300 python - > gpurun_out/prof.log 2>&1 <<'PY'
from magis_inputs import build_workload, CandidateGenerator, CandidateSpec
from paper_conf_asplos_chend0zll024_b200 import Graph
import torch
for c in ["c2", "c5", "c3"]:
    wl = build_workload(c); g = Graph.from_workload(wl)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=1)).generate(0, 8192)
    p = torch.from_numpy(P).cuda(); d = torch.from_numpy(D).cuda()
    for i in range(2): g.eval_schedules(p, d)
    torch.cuda.synchronize()
    print("cfg", c, flush=True)
PY
grep "magis-prof\|^cfg\|Error" gpurun_out/prof.log | awk 'NR%2==0 || /cfg|Error/'
