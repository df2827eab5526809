"""Parity at the sizes and launch configurations the bench times (VERDICT r1
"parity at benchmarked sizes"), plus regression tests for paths the
small-K tests never reach:

* many groups per CTA (K >> grid x P), so the double-buffered hand-off, the
  EMPTY-barrier path and the reuse of the per-CTA state run repeatedly;
* bad permutations early in a launch followed by valid candidates on the
  same CTA lane (an id in [NT, NTX) must not leak into the pos
  slots the later groups read);
* the global event-overflow path (more swap-event steps than the shared
  event slots hold);
* full bench sizes (C2 65,536 / C3 262,144 / C4 65,536), checked on a
  sample spread over the whole launch.

Expected values come only from oracle/ on host-generated inputs.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

from magis_inputs import CandidateGenerator, CandidateSpec, build_workload, models  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402
from tests import _defn  # noqa: E402
from tests._opool import eval_parallel  # noqa: E402
from tests.test_parity_gpu import VARIANTS, assert_parity, gpu_eval  # noqa: E402

_WL = {}


def wl_of(name):
    if name not in _WL:
        _WL[name] = build_workload(name)
    return _WL[name]


@pytest.fixture(params=["auto", "p2", "tier1p4", "tier2p1", "tier2p4", "tier3p2", "kb"])
def variant(request, monkeypatch):
    for k in ("MAGIS_VARIANT", "MAGIS_P", "MAGIS_TEAMS", "MAGIS_TIER", "MAGIS_KERNELB"):
        monkeypatch.delenv(k, raising=False)
    for k, v in VARIANTS[request.param].items():
        monkeypatch.setenv(k, v)
    return request.param


@pytest.mark.parametrize("cfg", ["c2", "c5"])
def test_bad_ids_do_not_leak_into_later_groups(cfg, variant):
    """The first grid x P candidates of the launch each carry one id in
    [NT, NT + |U|] (a virtual late-user slot or the dummy slot the row padding
    reads); 5 more rounds of valid candidates follow on the same CTAs."""
    wl = wl_of(cfg)
    g = Graph.from_workload(wl)
    o = OracleGraph.from_workload(wl)
    NT = wl.n_total
    nU = int(wl.U_arrays()[0][-1]) if wl.R else 0
    first = g.info["grid"] * max(1, g.info["pack"])
    K = first * 6
    P, D = CandidateGenerator(wl, CandidateSpec(seed=21)).generate(0, K)
    rng = np.random.default_rng(5)
    bad_ids = np.array([NT, NT + nU, NT + nU - 1 if nU else NT, NT + nU + 1], np.int64)
    for k in range(first):
        P[k, int(rng.integers(0, NT))] = int(bad_ids[k % len(bad_ids)])
    res = gpu_eval(g, P, D)
    ref = eval_parallel(o, P, D)
    assert (ref[0][:first] & 1).all()
    assert (ref[0][first:] == 0).mean() > 0.95
    assert_parity(*res, *ref)


def test_bad_ids_without_eligible_tensors(variant):
    """R = 0 (C1 diamond): the dummy slot is exactly NT, so an off-by-one id
    == n_total must go to the trash slot too."""
    wl = models.diamond([4, 4], seed=1)
    edges = list(zip(wl.src.tolist(), wl.dst.tolist()))
    orders = np.array(_defn.all_topo_orders(wl.n, edges), np.int32)
    g = Graph.from_workload(wl)
    o = OracleGraph.from_workload(wl)
    first = g.info["grid"] * max(1, g.info["pack"])
    K = first * 5
    P = orders[np.arange(K) % len(orders)].copy()
    P[:first, 3] = wl.n_total                      # id == n_total in every early candidate
    res = gpu_eval(g, P, None)
    ref = o.eval_batch(P)
    assert (ref[0][:first] == 1).all() and (ref[0][first:] == 0).all()
    assert_parity(*res, *ref)


@pytest.mark.parametrize("cfg,K", [("c4", 1024), ("c3", 4096)])
def test_large_graph_many_groups_per_cta(cfg, K, variant):
    """C4 (tier 2, one candidate per group: ~7 groups per CTA) and C3 (tier 1,
    P = 2: ~14 groups per CTA) through every tier, element by element."""
    wl = wl_of(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=31)).generate(0, K)
    g = Graph.from_workload(wl)
    res = gpu_eval(g, P, D)
    ref = eval_parallel(OracleGraph.from_workload(wl), P, D)
    assert (ref[0] == 0).mean() > 0.95
    assert_parity(*res, *ref)


@pytest.mark.parametrize("cfg,K", [("c2", 2048), ("c5", 2048), ("c4", 512)])
def test_event_overflow_path(cfg, K, variant):
    """P(swap) = 50%: every swapping candidate raises far more event steps
    than the shared-memory event slots hold (<= 128), so its events go to the
    global overflow region."""
    wl = wl_of(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=41, p_swap=5000, p_remat=1000)).generate(0, K)
    assert ((D[:, :wl.R] == 2).sum(axis=1) * 3 > 128).mean() > 0.99
    g = Graph.from_workload(wl)
    res = gpu_eval(g, P, D)
    ref = eval_parallel(OracleGraph.from_workload(wl), P, D)
    assert (ref[0] == 0).mean() > 0.9
    assert_parity(*res, *ref)


@pytest.mark.parametrize("cfg", ["c2", "c3", "c4", "c5"])
def test_full_bench_size_sampled_parity(cfg):
    """The bench's launch: the config's full K generated on the device (a1),
    scored in one call; 768 candidates spread over the launch (every CTA,
    early and late groups) are regenerated on the HOST (candgen.c) and scored
    by the oracle.  The device rows must equal the host rows (the generator
    is byte-identical), so the oracle input never comes from the CUDA path."""
    from magis_inputs import CONFIGS
    wl = wl_of(cfg)
    K = CONFIGS[cfg]["K"]
    g = Graph.from_workload(wl)
    Pd, Dd = g.generate_candidates(0, K, seed=1)
    st, pk, lt = g.eval_schedules(Pd, Dd if g.dec_len else None)
    torch.cuda.synchronize()
    rng = np.random.default_rng(7)
    ids = np.unique(np.concatenate([np.arange(0, 256), np.arange(K - 256, K), rng.integers(0, K, 256)]))
    gen = CandidateGenerator(wl, CandidateSpec(seed=1))
    Ph = np.empty((len(ids), wl.n_total), np.int32)
    Dh = np.zeros((len(ids), max(wl.R, 1)), np.uint8)
    for j, k in enumerate(ids):
        p, d = gen.generate(int(k), 1)
        Ph[j], Dh[j] = p[0], d[0]
    idt = torch.from_numpy(ids).cuda()
    assert np.array_equal(Pd[idt].cpu().numpy(), Ph)
    if wl.R:
        assert np.array_equal(Dd[idt, :wl.R].cpu().numpy(), Dh[:, :wl.R])
    ref = eval_parallel(OracleGraph.from_workload(wl), Ph, Dh)
    assert_parity(st[idt].cpu().numpy(), pk[idt].cpu().numpy(), lt[idt].cpu().numpy(), *ref)


def test_c3f_full_size_sampled_parity():
    """C3f (F-Trans variant regions, NEXT-4) at the bench's K = 65,536 on the
    packed kernel: the host generator's candidates (the device generator does
    not cover regions), 512 of them spread over the launch checked by the
    oracle."""
    from magis_inputs import CONFIGS
    wl = wl_of("c3f")
    K = CONFIGS["c3f"]["K"]
    P, D = CandidateGenerator(wl, CandidateSpec(seed=1)).generate(0, K)
    g = Graph.from_workload(wl)
    assert g.info["variant"] == 2
    Dd = torch.from_numpy(np.ascontiguousarray(D[:, :g.dec_len])).cuda()
    st, pk, lt = (t.cpu().numpy() for t in g.eval_schedules(torch.from_numpy(P).cuda(), Dd))
    rng = np.random.default_rng(3)
    ids = np.unique(np.concatenate([np.arange(0, 128), np.arange(K - 128, K), rng.integers(0, K, 256)]))
    ref = eval_parallel(OracleGraph.from_workload(wl), P[ids], D[ids])
    assert (ref[0] == 0).mean() > 0.9
    assert_parity(st[ids], pk[ids], lt[ids], *ref)

