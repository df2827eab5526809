"""Launch the device candidate generator a few times (for ncu)."""
import os
import sys

import torch

sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402

g = Graph.from_workload(build_workload(sys.argv[1] if len(sys.argv) > 1 else "c2"))
P, D = g.generate_candidates(0, 65536, seed=1)
for _ in range(2):
    g.generate_candidates(0, 65536, seed=1, perm=P, dec=D)
torch.cuda.synchronize()
