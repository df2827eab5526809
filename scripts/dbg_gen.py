"""Device generator vs the CPU generator on one config (sanitizer runs):
python scripts/dbg_gen.py CFG K"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.getcwd())
from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402

cfg, K = sys.argv[1], int(sys.argv[2])
wl = build_workload(cfg)
g = Graph.from_workload(wl)
Pg, Dg = g.generate_candidates(100, K, seed=3)
torch.cuda.synchronize()
Pc, Dc = CandidateGenerator(wl, CandidateSpec(seed=3)).generate(100, K)
bad = int((Pg.cpu().numpy() != Pc).any(axis=1).sum() + (Dg.cpu().numpy() != Dc).any(axis=1).sum())
print(f"generator {cfg} K={K}: mismatches {bad}")
