#!/bin/bash
# Device generator timing + one ncu --set full capture of the fast kernel (C2 by default).
mkdir -p gpurun_out
C=${GEN_CFG:-c2}
timeout 600 python scripts/gen_time.py $C c4 2>&1 | tee gpurun_out/gen_time.log
cat > gpurun_out/gone.py <<'PY'
import sys, os; sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload
from paper_conf_asplos_chend0zll024_b200 import Graph
import torch
wl = build_workload(sys.argv[1]); g = Graph.from_workload(wl)
P, D = g.generate_candidates(0, 65536, seed=1)
for i in range(2): g.generate_candidates(0, 65536, seed=1, perm=P, dec=D)
torch.cuda.synchronize()
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gen2_kernel -s 2 -c 1 -o gpurun_out/gen2_$C python gpurun_out/gone.py $C > gpurun_out/ncu_gen.log 2>&1
tail -2 gpurun_out/ncu_gen.log
python scripts/ncu_summary.py gpurun_out/gen2_$C.ncu-rep 30 > gpurun_out/ncu_full_gen2_$C.txt 2>&1
python scripts/ncu_stalls.py gpurun_out/gen2_$C.ncu-rep 40 > gpurun_out/ncu_stalls_gen2_$C.txt 2>&1
head -40 gpurun_out/ncu_full_gen2_$C.txt
head -30 gpurun_out/ncu_stalls_gen2_$C.txt
