"""a7's optional output: the first step whose allocation
brings M_i to M_peak, emitted by the batch call
magis_eval_schedules_argmax, against the oracle's first argmax (reading
P10: ties go to the first step).  The GPU reports the index into the
candidate's permutation; the oracle counts active steps only, so the test
maps one to the other with the candidate's active set (Fig. 8 rules)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402
from tests.test_oracle_pins import random_case, random_valid_perm  # noqa: E402
from tests.test_parity_gpu import DEV, VARIANTS, both  # noqa: E402


def compacted(perm, dec, n, R, a):
    """Active steps before permutation index a (clone iff dec 1, Store /
    Load iff dec 2)."""
    if a < 0:
        return -1
    c = 0
    for v in perm[:a]:
        if v < n:
            c += 1
        else:
            r, k = divmod(int(v) - n, 3)
            c += int(dec[r] == (1 if k == 0 else 2))
    return c


def check(g, o, P, D, n, R):
    Pt = torch.from_numpy(np.ascontiguousarray(P, np.int32)).to(DEV)
    Dt = torch.from_numpy(np.ascontiguousarray(D, np.uint8)).to(DEV) if R else None
    st, pk, lt, am = g.eval_schedules(Pt, Dt, argmax=True)
    st2, pk2, lt2 = g.eval_schedules(Pt, Dt)
    torch.cuda.synchronize()
    st, pk, lt, am = st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy(), am.cpu().numpy()
    assert np.array_equal(st, st2.cpu().numpy()) and np.array_equal(pk, pk2.cpu().numpy())
    assert np.array_equal(lt, lt2.cpu().numpy())
    nval = 0
    for k in range(len(P)):
        ost, opk, olt, oam = o.eval(P[k], D[k] if R else None)
        assert st[k] == ost and pk[k] == opk
        if ost:
            assert am[k] == -1
            continue
        nval += 1
        v = int(P[k][am[k]])
        assert v < n or D[k][(v - n) // 3] == (1 if (v - n) % 3 == 0 else 2)   # an active node
        assert compacted(P[k], D[k] if R else None, n, R, int(am[k])) == oam
    return nval


@pytest.fixture(params=["auto", "p2", "tier1p4", "tier2p1", "tier3p2"])
def variant(request, monkeypatch):
    for k in ("MAGIS_VARIANT", "MAGIS_P", "MAGIS_TEAMS", "MAGIS_TIER", "MAGIS_KERNELB"):
        monkeypatch.delenv(k, raising=False)
    for k, v in VARIANTS[request.param].items():
        monkeypatch.setenv(k, v)
    return request.param


@pytest.mark.parametrize("cfg", ["c2", "c5", "c3"])
def test_argmax_workloads(cfg, variant):
    wl = build_workload(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=23)).generate(0, 600)
    g = Graph.from_workload(wl)
    if g.info["variant"] != 2:
        pytest.skip("the forced plan does not fit: the graph fell back to the simple kernel")
    o = OracleGraph.from_workload(wl)
    assert check(g, o, P, D, wl.n, wl.R) > 500


def test_argmax_small_graphs_with_ties(variant):
    """Random DAGs with small integer sizes (many steps tie at the peak)."""
    rng = np.random.default_rng(31)
    for trial in range(60):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        size = [int(s) % 4 * 512 for s in size]            # ties at the peak
        o, g = both(n, edges, size, outs, cost=cost, elig=elig, U=U)
        if g.info["variant"] != 2:
            continue
        R = len(elig)
        perms, decs = [], []
        for j in range(16):
            d = rng.integers(0, 3, R).astype(np.uint8)
            p, _, _ = random_valid_perm(rng, n, edges, elig, U, d)
            perms.append(p)
            decs.append(d)
        P = np.array(perms, np.int32)
        D = np.array(decs, np.uint8).reshape(len(perms), max(R, 1))[:, :R] if R else np.zeros((len(perms), 1), np.uint8)
        check(g, o, P, D, n, R)


def test_argmax_unsupported_on_the_simple_kernel(monkeypatch):
    monkeypatch.setenv("MAGIS_VARIANT", "1")
    wl = build_workload("c2")
    g = Graph.from_workload(wl)
    assert g.info["variant"] in (0, 1)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=2)).generate(0, 4)
    from paper_conf_asplos_chend0zll024_b200 import MagisError
    with pytest.raises(MagisError):
        g.eval_schedules(torch.from_numpy(P).to(DEV), torch.from_numpy(D).to(DEV), argmax=True)

