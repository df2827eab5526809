#!/bin/bash
# One ncu --set full capture (with source) of the variant-2 kernel on C2, 8192 candidates.
mkdir -p gpurun_out
cat > gpurun_out/one.py <<'PY'
import sys, os; sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload, CandidateGenerator, CandidateSpec
from paper_conf_asplos_chend0zll024_b200 import Graph
import torch
wl = build_workload(sys.argv[1] if len(sys.argv) > 1 else "c2"); g = Graph.from_workload(wl)
P, D = CandidateGenerator(wl, CandidateSpec(seed=1)).generate(0, 16384)
p = torch.from_numpy(P).cuda(); d = torch.from_numpy(D).cuda()
for i in range(3): g.eval_schedules(p, d)
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 2 -c 1 -o gpurun_out/${NCU_NAME:-one} python gpurun_out/one.py ${NCU_CFG:-c2} > gpurun_out/ncu_one.log 2>&1
tail -3 gpurun_out/ncu_one.log
