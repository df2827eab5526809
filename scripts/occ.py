import os, sys, ctypes
sys.path.insert(0, os.getcwd())
os.environ["MAGIS_DEBUG"] = "1"
import torch
from magis_inputs import build_workload
from paper_conf_asplos_chend0zll024_b200 import Graph
for c in sys.argv[1:]:
    g = Graph.from_workload(build_workload(c))
    print(c, g.info, flush=True)
print(torch.cuda.get_device_properties(0))
lib = ctypes.CDLL(None)
