"""Small parity probe for sanitizer runs: python scripts/dbg_small.py CFG K"""
import os, sys
import numpy as np
import torch
sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload, CandidateGenerator, CandidateSpec
from paper_conf_asplos_chend0zll024_b200 import Graph
from oracle import OracleGraph
cfg, K = sys.argv[1], int(sys.argv[2])
wl = build_workload(cfg)
P, D = CandidateGenerator(wl, CandidateSpec(seed=11)).generate(0, K)
g = Graph.from_workload(wl)
st, pk, lt = g.eval_schedules(torch.from_numpy(P).cuda(), torch.from_numpy(D).cuda())
rs, rp, rl = OracleGraph.from_workload(wl).eval_batch(P, D)
print(cfg, K, "pack", g.info["pack"], "status mismatches", int((st.cpu().numpy() != rs).sum()),
      "peak mismatches", int((pk.cpu().numpy() != rp).sum()))
