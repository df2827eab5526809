"""Print every candidate plan of the eval kernel per config (MAGIS_DEBUG=2): python scripts/plan_dump.py c3 ..."""
import os, sys
os.environ.setdefault("MAGIS_DEBUG", "2")
sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402
for c in sys.argv[1:]:
    print("==", c, flush=True)
    g = Graph.from_workload(build_workload(c))
