import os, sys, numpy as np, torch
sys.path.insert(0, os.getcwd())
from magis_inputs import build_workload, CandidateGenerator, CandidateSpec
from paper_conf_asplos_chend0zll024_b200 import Graph
from oracle import OracleGraph
wl = build_workload(sys.argv[1])
P, D = CandidateGenerator(wl, CandidateSpec(seed=11)).generate(0, int(sys.argv[2]))
g = Graph.from_workload(wl)
print(g.info)
st, pk, lt = [t.cpu().numpy() for t in g.eval_schedules(torch.from_numpy(P).cuda(), torch.from_numpy(D).cuda())]
rs, rp, rl = OracleGraph.from_workload(wl).eval_batch(P, D)
ok = rs == 0
bad = ok & (np.abs(lt - rl) > 1e-9 * np.abs(rl))
print("ok", ok.sum(), "st mism", (st != rs).sum(), "pk mism", (pk != rp).sum(), "lat mism", bad.sum(), np.where(bad)[0][:20])
Pk = g.info["pack"]; grid = g.info["grid"]
U = [len(u) for u in wl.U]
nev = np.array([sum(3 + U[r] for r in range(wl.R) if d[r] == 2) for d in D])
idx = np.where(bad)[0]
grp = idx // Pk
print("gi of bad", sorted(set((grp // grid).tolist())), "nev of bad", nev[idx][:30].tolist(), "c of bad", (idx % Pk)[:30].tolist())
print("fraction nev>64 among ok", (nev[ok] > 64).mean(), "gi>=2 count", (np.arange(len(st)) // Pk // grid >= 2).sum())
