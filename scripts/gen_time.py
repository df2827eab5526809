"""Time the device candidate generator (magis_generate_candidates) per config:
python scripts/gen_time.py [cfg ...]"""
import os
import sys

import torch

sys.path.insert(0, os.getcwd())
from magis_inputs import CONFIGS, build_workload  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402

for cfg in sys.argv[1:] or ["c2", "c3", "c4", "c5"]:
    wl = build_workload(cfg)
    g = Graph.from_workload(wl)
    K = 65536
    P, D = g.generate_candidates(0, K, seed=1)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        g.generate_candidates(0, K, seed=1, perm=P, dec=D)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    print(f"{cfg} device generator {ms:.2f} ms per {K} candidates ({K / ms * 1e3:.3g} cand/s)", flush=True)
