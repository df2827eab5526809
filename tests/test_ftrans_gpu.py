"""NEXT-4 parity on the B200: graphs with F-Trans variant regions through
magis_graph_load_regions and magis_eval_schedules, against the oracle's gated
evaluation (itself pinned to the materialised F-Trans graphs,
tests/test_ftrans_variants.py).  Bar: status / peak bit-exact, latency 1e-9."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph, MagisError, pareto_merge  # noqa: E402
from tests.test_parity_gpu import assert_parity  # noqa: E402

DEV = "cuda:0"


def gpu_eval(g, P, D):
    st, pk, lt = g.eval_schedules(torch.from_numpy(P).to(DEV), torch.from_numpy(np.ascontiguousarray(D)).to(DEV))
    torch.cuda.synchronize()
    return st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy()


# the packed kernel (variant 2) on every plan tier, and the gated v1 kernel
REGION_VARIANTS = {"auto": {}, "v1": {"MAGIS_VARIANT": "1"},
                   "p1": {"MAGIS_P": "1", "MAGIS_TEAMS": "1"},
                   "tier1p4": {"MAGIS_TIER": "1", "MAGIS_P": "4", "MAGIS_TEAMS": "1"},
                   "tier2p1": {"MAGIS_TIER": "2", "MAGIS_P": "1", "MAGIS_TEAMS": "1"},
                   "tier3p2": {"MAGIS_TIER": "3", "MAGIS_P": "2", "MAGIS_TEAMS": "1"}}


@pytest.mark.parametrize("layers,variant", [(2, v) for v in REGION_VARIANTS] + [(24, "auto"), (24, "v1")])
def test_regions_parity(layers, variant, monkeypatch):
    for k in ("MAGIS_VARIANT", "MAGIS_P", "MAGIS_TEAMS", "MAGIS_TIER", "MAGIS_KERNELB"):
        monkeypatch.delenv(k, raising=False)
    for k, v in REGION_VARIANTS[variant].items():
        monkeypatch.setenv(k, v)
    wl = build_workload("c3f", layers=layers)
    g = Graph.from_workload(wl, device=0)
    assert g.F == wl.F > 0
    assert (g.info["variant"] in (0, 1)) if variant == "v1" else g.info["variant"] == 2
    o = OracleGraph.from_workload(wl)
    K = 1000 if layers == 2 else 300
    P, D = CandidateGenerator(wl, CandidateSpec(seed=11)).generate(0, K)
    D[3, wl.R] = 3                    # variant index out of range -> bad decision
    D[4, wl.R + 1] = 2                # ordinary
    st_g, pk_g, lt_g = gpu_eval(g, P, D)
    st_o, pk_o, lt_o = o.eval_batch(P, D)
    assert st_o[3] == 4
    assert (st_o == 0).sum() > K // 2
    assert_parity(st_g, pk_g, lt_g, st_o, pk_o, lt_o)
    # the same through the host-buffer (end-to-end) call
    hs, hp, hl = g.eval_schedules_host(P, D)
    assert_parity(hs, hp, hl, st_o, pk_o, lt_o)


def test_regions_front_and_unsupported_paths():
    wl = build_workload("c3f", layers=2)
    g = Graph.from_workload(wl, device=0)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=12)).generate(0, 2048)
    Pd, Dd = torch.from_numpy(P).to(DEV), torch.from_numpy(D).to(DEV)
    st, pk, lt = g.eval_schedules(Pd, Dd)
    fr = pareto_merge(pk, lt, st, cap=1024)
    torch.cuda.synchronize()
    import oracle
    ref = oracle.pareto(pk.cpu().numpy(), lt.cpu().numpy(), st.cpu().numpy())
    n = int(fr["front_n"].item())
    assert n == len(ref) and (fr["front_id"][:n].cpu().numpy() == ref).all()
    # the variant choice moves the (peak, latency) trade-off: the front mixes variants
    assert len(set(map(tuple, D[ref][:, wl.R:]))) > 1
    for call in (lambda: g.generate_candidates(0, 4), lambda: g.hotspots(Pd[:2], Dd[:2, :wl.R].contiguous())):
        with pytest.raises(MagisError):
            call()
