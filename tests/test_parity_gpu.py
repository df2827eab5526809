"""Parity of the sm_100a path (through the C ABI) with the CPU oracle.

Bar (BASELINE.json north_star): status and peak bit-exact (int64), latency
within 1e-9 relative.  Inputs come only from magis_inputs (seeded) and the
tests' own constructions; expected values come only from oracle/.
"""
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from magis_inputs import CandidateGenerator, CandidateSpec, build_workload, models  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph, pareto_merge  # noqa: E402
from tests import _defn  # noqa: E402
from tests.test_oracle_pins import T1_EDGES, T2_EDGES, fig2a_graph, random_case, random_valid_perm  # noqa: E402

LAT_RTOL = 1e-9
DEV = "cuda:0"

# kernel variants: magis_eval.cu (v1, global state) and magis_eval2.cu with
# P = 1 / 2 / 4 packed candidates; "auto" is what the loader picks.
VARIANTS = {"auto": {}, "v1": {"MAGIS_VARIANT": "1"}, "p1": {"MAGIS_P": "1", "MAGIS_TEAMS": "1"},
            "p2": {"MAGIS_P": "2", "MAGIS_TEAMS": "1"}, "p4": {"MAGIS_P": "4", "MAGIS_TEAMS": "1"},
            "t2p1": {"MAGIS_P": "1", "MAGIS_TEAMS": "2"}, "t2p2": {"MAGIS_P": "2", "MAGIS_TEAMS": "2"},
            # plan tiers: 1 tables in global, 2 + int32 delta slots, 3 slots in global
            "tier1p4": {"MAGIS_TIER": "1", "MAGIS_P": "4", "MAGIS_TEAMS": "1"},
            "tier2p1": {"MAGIS_TIER": "2", "MAGIS_P": "1", "MAGIS_TEAMS": "1"},
            "tier2p4": {"MAGIS_TIER": "2", "MAGIS_P": "4", "MAGIS_TEAMS": "1"},
            "tier3p2": {"MAGIS_TIER": "3", "MAGIS_P": "2", "MAGIS_TEAMS": "1"},
            # kernel B: one candidate per two-CTA cluster (magis_evalb.cu)
            "kb": {"MAGIS_KERNELB": "1"}}


@pytest.fixture(params=list(VARIANTS))
def variant(request, monkeypatch):
    for k in ("MAGIS_VARIANT", "MAGIS_P", "MAGIS_TEAMS", "MAGIS_TIER", "MAGIS_KERNELB"):
        monkeypatch.delenv(k, raising=False)
    for k, v in VARIANTS[request.param].items():
        monkeypatch.setenv(k, v)
    return request.param


def gpu_eval(g: Graph, perms: np.ndarray, decs) -> tuple:
    P = torch.from_numpy(np.ascontiguousarray(perms, np.int32)).to(DEV)
    D = None
    if g.R:
        D = torch.from_numpy(np.ascontiguousarray(decs, np.uint8).reshape(len(perms), g.R)).to(DEV)
    st, pk, lt = g.eval_schedules(P, D)
    torch.cuda.synchronize()
    return st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy()


def assert_parity(st_g, pk_g, lt_g, st_o, pk_o, lt_o):
    np.testing.assert_array_equal(st_g, st_o)
    np.testing.assert_array_equal(pk_g, pk_o)
    ok = st_o == 0
    assert np.all(np.isinf(lt_g[~ok])) and np.all(pk_g[~ok] == -1)
    rel = np.abs(lt_g[ok] - lt_o[ok]) / np.maximum(np.abs(lt_o[ok]), 1e-300)
    assert rel.size == 0 or rel.max() <= LAT_RTOL, rel.max()


def both(n, edges, size, outputs, cost=None, elig=(), U=(), B=25e9, lam=1e-5):
    iso = np.zeros(n, np.uint8)
    iso[list(outputs)] = 1
    cost = [0.0] * n if cost is None else cost
    src = [u for u, _ in edges]
    dst = [v for _, v in edges]
    o = OracleGraph(list(size), cost, iso, src, dst, list(elig), [list(u) for u in U], B, lam)
    g = Graph(list(size), cost, iso, src, dst, list(elig), [list(u) for u in U], B, lam, device=0)
    return o, g


def test_paper_examples_on_gpu(variant):
    n, edges, size, outs, f, b = fig2a_graph()
    o, g = both(n, edges, size, outs)
    st, pk, lt = gpu_eval(g, np.arange(64)[None], None)
    assert (st[0], pk[0]) == (0, 1056)                 # Fig. 2(a)
    elig = [f(i) for i in range(1, 32)]
    U = [[b(33 - i)] for i in range(1, 32)]
    o, g = both(n, edges, size, outs, elig=elig, U=U)
    order = []
    for i in range(1, 32):
        order += [f(i), n + 3 * (i - 1) + 1]
    order += [f(32), b(1)]
    for k in range(2, 33):
        order += [n + 3 * (32 - k) + 2, b(k)]
    order += [n + 3 * (i - 1) for i in range(1, 32)]
    st, pk, lt = gpu_eval(g, np.array([order]), np.full((1, 31), 2, np.uint8))
    assert (st[0], pk[0]) == (0, 96)                   # Fig. 2(b)


@pytest.mark.parametrize("rows,B", [
    ([([0, 1, 2, 3, 4, 5, 6], 0), ([0, 5, 1, 2, 6, 3, 4], 2), ([0, 5, 1, 6, 2, 3, 4], 2),
      ([0, 6, 5, 1, 2, 3, 4], 2)], 50.0),
    ([([0, 5, 1, 2, 6, 3, 4], 2)], 100.0),
])
def test_T1_toy_on_gpu(rows, B, variant):
    o, g = both(4, T1_EDGES, [100, 200, 200, 10], [3], cost=[1.0] * 4, elig=[0], U=[[3]], B=B, lam=0.0)
    perms = np.array([r[0] for r in rows])
    decs = np.array([[r[1]] for r in rows], np.uint8)
    assert_parity(*gpu_eval(g, perms, decs), *o.eval_batch(perms, decs))


def test_T2_toy_on_gpu(variant):
    o, g = both(5, T2_EDGES, [10, 100, 200, 200, 10], [4], cost=[0.0, 2.0, 1.0, 1.0, 1.0], elig=[1], U=[[4]])
    perms = np.array([[0, 1, 2, 3, 4, 5, 6, 7], [0, 1, 2, 3, 5, 4, 6, 7], [0, 1, 5, 2, 3, 4, 6, 7]])
    decs = np.array([[0], [1], [1]], np.uint8)
    st, pk, lt = gpu_eval(g, perms, decs)
    assert list(pk) == [500, 410, 500] and list(lt) == [5.0, 7.0, 7.0]
    assert_parity(st, pk, lt, *o.eval_batch(perms, decs))


@pytest.mark.parametrize("branches", [[4, 4], [3, 3, 2], [2, 2, 2, 2], [2, 2, 2, 1, 1]])
def test_c1_diamonds_all_orders(branches, variant):
    """C1: every topological order of a 10-op diamond (70..5040 orders)."""
    wl = models.diamond(branches, seed=1)
    edges = list(zip(wl.src.tolist(), wl.dst.tolist()))
    o, g = both(wl.n, edges, wl.size.tolist(), [wl.n - 1], cost=wl.cost.tolist())
    orders = np.array(_defn.all_topo_orders(wl.n, edges), np.int32)
    res = gpu_eval(g, orders, None)
    ref = o.eval_batch(orders)
    assert_parity(*res, *ref)
    assert res[1].min() == ref[1].min()   # brute-force optimum


def test_random_small_graphs_with_decisions(variant):
    """Random DAGs of <= 11 ops with random eligible sets and decisions: valid
    orders, random shuffles (mostly invalid), duplicates, bad decisions."""
    rng = np.random.default_rng(2024)
    for trial in range(150):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        o, g = both(n, edges, size, outs, cost=cost, elig=elig, U=U, B=float(rng.integers(1, 100)) * 1e3,
                    lam=float(rng.random()))
        R = len(elig)
        NT = n + 3 * R
        perms, decs = [], []
        for j in range(24):
            d = rng.integers(0, 3, R).astype(np.uint8)
            p, _, _ = random_valid_perm(rng, n, edges, elig, U, d)
            perms.append(p)
            decs.append(d)
        for j in range(6):
            perms.append(rng.permutation(NT).tolist())
            decs.append(rng.integers(0, 3, R).astype(np.uint8))
        p = list(perms[0])
        p[0] = p[-1]
        perms.append(p)
        decs.append(decs[0])                              # duplicate -> bit0
        p = list(perms[1])
        p[int(rng.integers(0, NT))] = NT + 3                # out of range -> bit0
        perms.append(p)
        decs.append(decs[1])
        if R:
            d = decs[2].copy()
            d[int(rng.integers(0, R))] = 3                  # bad decision -> bit2
            perms.append(perms[2])
            decs.append(d)
        P = np.array(perms, np.int32)
        D = np.array(decs, np.uint8).reshape(len(perms), max(R, 1))[:, :R] if R else None
        ref = o.eval_batch(P, D if R else None)
        assert_parity(*gpu_eval(g, P, D), *ref)


@pytest.fixture(scope="module", params=["c2", "c3", "c5"])
def workload(request):
    return build_workload(request.param)


def test_workload_parity(workload, variant):
    """C2 / C3 / C5 at K=2048 seeded candidates (75% random orders, 24% local
    moves, 1% transpositions; 5%/5% remat/swap), element by element."""
    wl = workload
    gen = CandidateGenerator(wl, CandidateSpec(seed=11))
    P, D = gen.generate(0, 2048)
    g = Graph.from_workload(wl)
    o = OracleGraph.from_workload(wl)
    if variant in ("p1", "p2", "p4") and g.info["variant"] == 2:
        assert g.info["pack"] == int(variant[1])
    if variant == "v1":
        assert g.info["variant"] in (0, 1)
    if variant == "kb":
        assert g.info["variant"] == 3
    res = gpu_eval(g, P, D)
    ref = o.eval_batch(P, D)
    assert_parity(*res, *ref)
    assert (ref[0] == 0).mean() > 0.95 and (ref[0] == 2).any()


def test_c4_large_graph_parity(variant):
    """C4 (~23.5k super-graph nodes): the global-state variant."""
    wl = build_workload("c4")
    gen = CandidateGenerator(wl, CandidateSpec(seed=3))
    P, D = gen.generate(0, 96)
    g = Graph.from_workload(wl)
    assert g.info["variant"] in (1, 2, 3)
    o = OracleGraph.from_workload(wl)
    assert_parity(*gpu_eval(g, P, D), *o.eval_batch(P, D))


def test_c2_full_size_sampled(variant):
    """BASELINE configs[1] at full size (64k candidates, the bench's launch):
    every candidate's status and sampled candidates against the oracle."""
    wl = build_workload("c2")
    K = 65536
    gen = CandidateGenerator(wl, CandidateSpec(seed=1))
    P, D = gen.generate(0, K)
    g = Graph.from_workload(wl)
    st, pk, lt = gpu_eval(g, P, D)
    rng = np.random.default_rng(0)
    idx = np.sort(rng.choice(K, 1500, replace=False))
    o = OracleGraph.from_workload(wl)
    ref = o.eval_batch(P[idx], D[idx])
    assert_parity(st[idx], pk[idx], lt[idx], *ref)
    ok = st == 0
    assert set(np.unique(st).tolist()) <= {0, 2}
    assert (pk[ok] > 0).all() and (lt[ok] >= wl.cost.sum() * (1 - 1e-12)).all()
    assert (pk[ok] <= int(wl.size.sum()) + sum(int(wl.size[t]) for t in wl.elig) * 2).all()


def test_host_path_matches_device_path():
    wl = build_workload("c5")
    P, D = CandidateGenerator(wl, CandidateSpec(seed=5)).generate(0, 3000)
    g = Graph.from_workload(wl)
    dev = gpu_eval(g, P, D)
    Pp = torch.from_numpy(P).pin_memory()
    Dp = torch.from_numpy(D).pin_memory()
    host = g.eval_schedules_host(Pp, Dp)
    for a, b in zip(dev, host):
        np.testing.assert_array_equal(a, b)
    # compact uint16 wire format (magis_eval_schedules_host_u16), pageable and pinned
    host16 = g.eval_schedules_host(P.astype(np.uint16), D)
    for a, b in zip(dev, host16):
        np.testing.assert_array_equal(a, b)
    host16p = g.eval_schedules_host(torch.from_numpy(P.astype(np.uint16)).pin_memory(), Dp)
    for a, b in zip(dev, host16p):
        np.testing.assert_array_equal(a, b)


def test_k_zero_and_one_and_ragged(variant):
    wl = models.diamond([3, 2], seed=3)           # NT = 7: rows not 16-byte aligned
    edges = list(zip(wl.src.tolist(), wl.dst.tolist()))
    o, g = both(wl.n, edges, wl.size.tolist(), [wl.n - 1])
    st, pk, lt = g.eval_schedules(torch.empty((0, wl.n), dtype=torch.int32, device=DEV), None)
    assert st.numel() == 0
    orders = np.array(_defn.all_topo_orders(wl.n, edges), np.int32)
    for k in (1, 3, len(orders)):
        assert_parity(*gpu_eval(g, orders[:k], None), *o.eval_batch(orders[:k]))


# ------------------------------------------------------------------ Pareto --

def gpu_front(peak, lat, status, ids=None, cap=8192, M=-1, L=-1.0):
    t = lambda a, dt: torch.from_numpy(np.ascontiguousarray(a, dt)).to(DEV)
    out = pareto_merge(t(peak, np.int64), t(lat, np.float64), None if status is None else t(status, np.uint8),
                       ids=None if ids is None else t(ids, np.int64), cap=cap, mem_limit=M, lat_limit=L)
    torch.cuda.synchronize()
    nf = int(out["front_n"].item())
    k = min(nf, cap)
    return (nf, out["front_id"][:k].cpu().numpy(), out["front_peak"][:k].cpu().numpy(),
            out["front_lat"][:k].cpu().numpy(), out["best"].cpu().numpy(), out)


@pytest.mark.parametrize("n", [0, 1, 17, 4096, 3 * 4096 + 17])
def test_pareto_matches_oracle(n):
    rng = np.random.default_rng(n)
    peak = rng.integers(0, 300, n).astype(np.int64)
    lat = rng.integers(0, 300, n).astype(np.float64) * 0.5
    status = (rng.random(n) < 0.1).astype(np.uint8)
    ids = np.arange(n, dtype=np.int64)
    M, L = 150, 40.0
    nf, fid, fpk, flt, best, _ = gpu_front(peak, lat, status, M=M, L=L)
    ref = oracle.pareto(peak, lat, status, ids)
    assert nf == len(ref)
    np.testing.assert_array_equal(fid, ids[ref])
    np.testing.assert_array_equal(fpk, peak[ref])
    np.testing.assert_array_equal(flt, lat[ref])
    assert best[0] == oracle.best_under_memory(peak, lat, status, M, ids)
    assert best[1] == oracle.best_under_latency(peak, lat, status, L, ids)


def test_pareto_all_on_front_and_capacity():
    n = 10000
    peak = np.arange(n, dtype=np.int64)
    lat = (n - np.arange(n)).astype(np.float64)            # every point on the front
    nf, fid, fpk, flt, best, out = gpu_front(peak, lat, None, cap=256)
    assert nf == n and (fpk == np.arange(256)).all()
    assert (out["front_id"][:256].cpu().numpy() == np.arange(256)).all()


def test_pareto_shard_merge_identical_to_single():
    """P local fronts (padded, all-gathered) merged == 1-shard front."""
    wl = build_workload("c2")
    P, D = CandidateGenerator(wl, CandidateSpec(seed=9)).generate(0, 12000)
    g = Graph.from_workload(wl)
    st, pk, lt = gpu_eval(g, P, D)
    cap = 2048
    single = gpu_front(pk, lt, st, cap=cap, M=int(np.median(pk[st == 0])), L=float(np.median(lt[st == 0])))
    for nr in (2, 4, 8):
        parts = np.array_split(np.arange(len(pk)), nr)
        gi, gp, gl = [], [], []
        for p in parts:
            nf, fid, fpk, flt, best, out = gpu_front(pk[p], lt[p], st[p], ids=p, cap=cap)
            gi.append(out["front_id"].cpu().numpy())
            gp.append(out["front_peak"].cpu().numpy())
            gl.append(out["front_lat"].cpu().numpy())
        merged = gpu_front(np.concatenate(gp), np.concatenate(gl), None, ids=np.concatenate(gi), cap=cap,
                           M=int(np.median(pk[st == 0])), L=float(np.median(lt[st == 0])))
        assert merged[0] == single[0]
        for a, b in zip(merged[1:5], single[1:5]):
            np.testing.assert_array_equal(a, b)
    # and the GPU front equals the oracle's front of the GPU values
    ref = oracle.pareto(pk, lt, st)
    np.testing.assert_array_equal(single[1], ref)


# --------------------------------------------------- device generator (a1) --

@pytest.mark.parametrize("cfg", ["c1", "c2", "c3", "c4", "c5"])
def test_device_generator_bit_exact(cfg):
    """magis_generate_candidates == the CPU generator (magis_inputs) byte for
    byte, on a shard that does not start at id 0."""
    wl = build_workload(cfg)
    spec = CandidateSpec(seed=17)
    Pc, Dc = CandidateGenerator(wl, spec).generate(1000, 700)
    g = Graph.from_workload(wl)
    Pg, Dg = g.generate_candidates(1000, 700, seed=17)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(Pg.cpu().numpy(), Pc)
    np.testing.assert_array_equal(Dg.cpu().numpy(), Dc)


def _gen_both(wl, spec, id0, K):
    Pc, Dc = CandidateGenerator(wl, spec).generate(id0, K)
    g = Graph.from_workload(wl)
    Pg, Dg = g.generate_candidates(id0, K, seed=spec.seed, pct_random=spec.pct_random, pct_local=spec.pct_local,
                                   p_remat=spec.p_remat, p_swap=spec.p_swap, wmax=spec.wmax, slack=spec.slack)
    torch.cuda.synchronize()
    return Pc, Dc, Pg.cpu().numpy(), Dg.cpu().numpy()


def test_device_generator_sequential_kernel(monkeypatch):
    """MAGIS_GEN_SEQ=1 forces the sequential kernel (the fast kernel's re-run
    path) for the whole call: the same bytes as the CPU generator."""
    monkeypatch.setenv("MAGIS_GEN_SEQ", "1")
    wl = build_workload("c2")
    Pc, Dc, Pg, Dg = _gen_both(wl, CandidateSpec(seed=5), 300, 400)
    np.testing.assert_array_equal(Pg, Pc)
    np.testing.assert_array_equal(Dg, Dc)


def test_device_generator_heap_overflow_rerun():
    """A fan-out wider than the fast kernel's on-chip heap (150 nodes ready at
    once; 64 entries on chip for n <= 3,072): every random-order candidate is
    flagged and re-generated by the sequential kernel, windows longer than the
    heap too, and the result is still the CPU generator's, byte for byte; mixed
    with candidates that stay on the fast kernel in the same launch."""
    from magis_inputs.graph import Workload
    rng = np.random.default_rng(3)
    fan = 150
    n = fan + 12
    edges = [(0, i) for i in range(1, fan + 1)] + [(i, fan + 1) for i in range(1, fan + 1)]
    edges += [(v, v + 1) for v in range(fan + 1, n - 1)]
    edges += [(v, v + 2) for v in range(fan + 1, n - 2)]
    size = (rng.integers(1, 1 << 12, n) * 512).astype(np.int64)
    elig = [fan + 2, fan + 4]
    U = [[fan + 4], [fan + 6]]
    wl = Workload("fan", size, rng.uniform(1e-6, 1e-4, n), np.eye(1, n, n - 1, dtype=np.uint8)[0],
                  np.asarray([u for u, _ in edges], np.int32), np.asarray([v for _, v in edges], np.int32),
                  [""] * n, ["op"] * n, np.asarray(elig, np.int32), U)
    for spec in (CandidateSpec(seed=11, p_remat=3000, p_swap=3000),
                 CandidateSpec(seed=12, pct_random=0, pct_local=100, wmax=n),
                 CandidateSpec(seed=13, pct_random=50, pct_local=20, wmax=40)):
        Pc, Dc, Pg, Dg = _gen_both(wl, spec, 7, 3000)
        np.testing.assert_array_equal(Pg, Pc)
        np.testing.assert_array_equal(Dg, Dc)


def test_device_generator_small_graphs():
    rng = np.random.default_rng(8)
    for trial in range(30):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        o, g = both(n, edges, size, outs, cost=cost, elig=elig, U=U)
        from magis_inputs.graph import Workload
        wl = Workload("rand", np.asarray(size, np.int64), np.asarray(cost), np.zeros(n, np.uint8),
                      np.asarray([u for u, _ in edges], np.int32), np.asarray([v for _, v in edges], np.int32),
                      [""] * n, ["op"] * n, np.asarray(elig, np.int32), [list(u) for u in U])
        for spec in (CandidateSpec(seed=trial, p_remat=3000, p_swap=3000, wmax=4, slack=2),
                     CandidateSpec(seed=trial + 100, pct_random=0, pct_local=50)):
            Pc, Dc = CandidateGenerator(wl, spec).generate(5, 64)
            Pg, Dg = g.generate_candidates(5, 64, seed=spec.seed, pct_random=spec.pct_random,
                                           pct_local=spec.pct_local, p_remat=spec.p_remat, p_swap=spec.p_swap,
                                           wmax=spec.wmax, slack=spec.slack)
            torch.cuda.synchronize()
            np.testing.assert_array_equal(Pg.cpu().numpy(), Pc)
            np.testing.assert_array_equal(Dg.cpu().numpy()[:, :len(elig)], Dc[:, :len(elig)])
            # and the generated candidates evaluate identically on both sides
            R = len(elig)
            assert_parity(*gpu_eval(g, Pc, Dc[:, :R] if R else None), *o.eval_batch(Pc, Dc[:, :R] if R else None))


@pytest.mark.parametrize("cfg", ["c2", "c5"])
def test_delta4_wire_matches_device_path(cfg):
    """End-to-end delta4 call (magis_eval_schedules_host_delta4): several
    chunks, escapes at the row start, out-of-range ids, odd and even rows."""
    from paper_conf_asplos_chend0zll024_b200 import encode_delta4
    wl = build_workload(cfg)
    g = Graph.from_workload(wl, device=0)
    K = 20011
    P, D = CandidateGenerator(wl, CandidateSpec(seed=22)).generate(0, K)
    P[5, 0] = wl.n_total - 1
    P[6, 3] = -1
    P[7, 9] = 70000
    st_d, pk_d, lt_d = gpu_eval(g, P, D[:, :wl.R])
    st_w, pk_w, lt_w = g.eval_schedules_host(encode_delta4(P), np.ascontiguousarray(D[:, :wl.R]))
    np.testing.assert_array_equal(st_w, st_d)
    np.testing.assert_array_equal(pk_w, pk_d)
    np.testing.assert_array_equal(lt_w, lt_d)
    assert st_w[6] & 1 and st_w[7] & 1
    o = OracleGraph.from_workload(wl)
    idx = np.array([0, 5, 6, 7, 9000, K - 1])
    assert_parity(st_w[idx], pk_w[idx], lt_w[idx], *o.eval_batch(P[idx], D[idx, :wl.R]))


@pytest.mark.parametrize("cfg", ["c2", "c5"])
def test_delta8_wire_matches_device_path(cfg):
    """End-to-end delta8 call (magis_eval_schedules_host_delta8): several
    chunks, rows with exceptions at the start, out-of-range ids."""
    from paper_conf_asplos_chend0zll024_b200 import encode_delta8
    wl = build_workload(cfg)
    g = Graph.from_workload(wl, device=0)
    K = 20011
    P, D = CandidateGenerator(wl, CandidateSpec(seed=21)).generate(0, K)
    P[5, 0] = wl.n_total - 1
    P[6, 3] = -1
    P[7, 9] = 70000
    st_d, pk_d, lt_d = gpu_eval(g, P, D[:, :wl.R])
    st_w, pk_w, lt_w = g.eval_schedules_host(encode_delta8(P), np.ascontiguousarray(D[:, :wl.R]))
    np.testing.assert_array_equal(st_w, st_d)
    np.testing.assert_array_equal(pk_w, pk_d)
    np.testing.assert_array_equal(lt_w, lt_d)
    assert st_w[6] & 1 and st_w[7] & 1
    o = OracleGraph.from_workload(wl)
    idx = np.array([0, 5, 6, 7, 9000, K - 1])
    assert_parity(st_w[idx], pk_w[idx], lt_w[idx], *o.eval_batch(P[idx], D[idx, :wl.R]))
