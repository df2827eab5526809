import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload, CandidateGenerator, CandidateSpec
from oracle import OracleGraph
from paper_conf_asplos_chend0zll024_b200 import Graph
wl = build_workload(sys.argv[1] if len(sys.argv) > 1 else "c2")
P, D = CandidateGenerator(wl, CandidateSpec(seed=11)).generate(0, 2048)
o = OracleGraph.from_workload(wl)
rs, rp, rl = o.eval_batch(P, D)
U = [len(u) for u in wl.U]
nev = np.array([sum(3 + U[r] for r in range(wl.R) if d[r] == 2) for d in D])
for var in ["v1", "p1", "p2", "p4"]:
    os.environ.pop("MAGIS_VARIANT", None); os.environ.pop("MAGIS_P", None)
    if var == "v1": os.environ["MAGIS_VARIANT"] = "1"
    else: os.environ["MAGIS_P"] = var[1]
    g = Graph.from_workload(wl)
    st, pk, lt = [t.cpu().numpy() for t in g.eval_schedules(torch.from_numpy(P).cuda(), torch.from_numpy(D).cuda())]
    ok = rs == 0
    bad = ok & (np.abs(lt - rl) > 1e-9 * np.abs(rl))
    print(var, g.info["variant"], g.info["pack"], "peak mismatches", int((pk != rp).sum()), "lat mismatches", int(bad.sum()),
          "nev of bad", sorted(set(nev[bad].tolist()))[:20], "max nev", nev.max(), "n>64", int((nev > 64).sum()))
