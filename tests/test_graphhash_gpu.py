"""NEXT-2 parity: batched GraphHash and the duplicate filter on the B200
(through the C ABI) against the CPU oracle (Alg. 3 lines 3-6 / 10-12,
readings G1-G4).  Bar: status and hash bit-exact (integer work); the filter's
new-flags bit-exact against oracle.hash_filter over successive batches.
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from magis_inputs.labels import node_labels  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph, GraphHasher, HashSet  # noqa: E402
from tests.test_graphhash_oracle import _random_case  # noqa: E402

DEV = "cuda:0"


def u64(t):
    return t.cpu().numpy().view(np.uint64)


def gpu_hash(hz: GraphHasher, D: np.ndarray):
    d = torch.from_numpy(np.ascontiguousarray(D, np.uint8)).to(DEV)
    st, h = hz.hash(d)
    torch.cuda.synchronize()
    return st.cpu().numpy(), u64(h)


def _pair(n, edges, elig, U):
    size = np.ones(n, np.int64)
    iso = np.zeros(n, np.uint8)
    iso[n - 1] = 1
    src = [u for u, _ in edges]
    dst = [v for _, v in edges]
    o = OracleGraph(size, np.zeros(n), iso, src, dst, list(elig), [list(u) for u in U])
    g = Graph(size, np.zeros(n), iso, src, dst, list(elig), [list(u) for u in U], device=0)
    return o, g


def test_random_small_graphs_bit_exact():
    rng = np.random.default_rng(31)
    for trial in range(60):
        n, edges, label, elig, U, dec = _random_case(rng, nmax=14, nlab=3)
        if not edges:
            continue
        o, g = _pair(n, edges, elig, U)
        hz = GraphHasher(g, label)
        K = int(rng.integers(1, 100))
        R = len(elig)
        D = rng.integers(0, 3, (K, max(R, 1))).astype(np.uint8)
        if R:
            D[rng.random(K) < 0.05, 0] = 7          # bad decision
        st_o, h_o = o.graph_hash_batch(label, D[:, :R] if R else D)
        st_g, h_g = gpu_hash(hz, D[:, :R] if R else D)
        np.testing.assert_array_equal(st_g, st_o)
        np.testing.assert_array_equal(h_g, h_o)


def test_wide_merges_use_every_sort_path():
    """In-degrees 1..40 (register networks of 4 / 8 / 32 and the rank sort
    beyond 32) with duplicate predecessor values (equal labels, no preds)."""
    rng = np.random.default_rng(32)
    n_src = 40
    edges, label = [], []
    for v in range(n_src):
        label.append(int(rng.integers(1, 4)))
    nid = n_src
    for deg in list(range(1, 41)) + [33, 37]:
        for u in rng.choice(nid, size=min(deg, nid), replace=False):
            edges.append((int(u), nid))
        label.append(int(rng.integers(1, 4)))
        nid += 1
    label = np.array(label, np.uint64)
    o, g = _pair(nid, edges, [], [])
    hz = GraphHasher(g, label)
    st_o, h_o = o.graph_hash_batch(label, np.zeros((37, 1), np.uint8))
    st_g, h_g = gpu_hash(hz, np.zeros((37, 1), np.uint8))
    np.testing.assert_array_equal(h_g, h_o)
    assert len(set(h_g.tolist())) == 1


@pytest.mark.parametrize("cfg", ["c2", "c5", "c3"])
def test_configs_sampled_and_consistent(cfg):
    wl = build_workload(cfg)
    label = node_labels(wl)
    g = Graph.from_workload(wl, device=0)
    hz = GraphHasher(g, label)
    o = OracleGraph.from_workload(wl)
    K = 4099                                     # ragged tail of a 32-candidate warp
    _, D = CandidateGenerator(wl, CandidateSpec(seed=3)).generate(0, K)
    D = np.ascontiguousarray(D[:, :wl.R])
    D[5] = 0                                     # duplicates of the all-keep graph
    D[77] = 0
    D[900] = D[901]
    D[11, 3] = 9                                 # bad decision
    st_g, h_g = gpu_hash(hz, D)
    idx = np.array([0, 5, 11, 77, 900, 901, K - 1] + list(range(1000, 1000 + (12 if cfg == "c3" else 40))))
    st_o, h_o = o.graph_hash_batch(label, D[idx])
    np.testing.assert_array_equal(st_g[idx], st_o)
    np.testing.assert_array_equal(h_g[idx], h_o)
    # properties at full size: equal decisions <=> equal graphs => equal hashes
    _, first = np.unique(D, axis=0, return_index=True)
    rows = {}
    for k in range(K):
        key = D[k].tobytes()
        if key in rows:
            assert h_g[k] == h_g[rows[key]]
        else:
            rows[key] = k
    assert st_g[11] == 4 and h_g[11] == 0
    assert h_g[5] == h_g[77] and h_g[900] == h_g[901]


def test_full_c2_batch_and_misaligned_decisions():
    """K = 65,536 at C2 (the bench workload) in the bench's launch shape, plus
    the byte-load path (rows not 16-byte aligned)."""
    wl = build_workload("c2")
    label = node_labels(wl)
    g = Graph.from_workload(wl, device=0)
    hz = GraphHasher(g, label)
    o = OracleGraph.from_workload(wl)
    K = 65536
    _, D = CandidateGenerator(wl, CandidateSpec(seed=4)).generate(0, K)
    D = np.ascontiguousarray(D[:, :wl.R])
    st_g, h_g = gpu_hash(hz, D)
    samp = np.random.default_rng(5).choice(K, 48, replace=False)
    st_o, h_o = o.graph_hash_batch(label, D[samp])
    np.testing.assert_array_equal(h_g[samp], h_o)
    # misaligned rows: the same decisions at an odd byte offset
    buf = torch.zeros(K * wl.R + 1, dtype=torch.uint8, device=DEV)
    buf[1:] = torch.from_numpy(D.reshape(-1)).to(DEV)
    dmis = buf[1:].view(K, wl.R)
    st2, h2 = hz.hash(dmis)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(u64(h2), h_g)


def test_no_eligible_graph_and_empty_batch():
    wl = build_workload("c1")
    label = np.arange(1, wl.n + 1, dtype=np.uint64)
    g = Graph.from_workload(wl, device=0)
    hz = GraphHasher(g, label)
    o = OracleGraph.from_workload(wl)
    st, h = hz.hash(40)
    torch.cuda.synchronize()
    _, ho = o.graph_hash_batch(label, np.zeros((1, 1), np.uint8))
    assert (u64(h) == ho[0]).all() and (st.cpu().numpy() == 0).all()
    st, h = hz.hash(torch.zeros((0, 1), dtype=torch.uint8, device=DEV))
    assert st.numel() == 0


def test_filter_matches_oracle_over_batches():
    rng = np.random.default_rng(33)
    hs = HashSet(1 << 12)
    X = set()
    for b in range(6):
        K = int(rng.integers(1, 3000))
        hv = rng.integers(0, 500, K).astype(np.uint64) * np.uint64(0x9E3779B97F4A7C15)
        hv[rng.random(K) < 0.02] = 0
        stv = ((rng.random(K) < 0.1) * 4).astype(np.uint8)
        new_o, X = oracle.hash_filter(hv, stv, X)
        new_g = hs.filter(torch.from_numpy(hv.view(np.int64)).to(DEV), torch.from_numpy(stv).to(DEV))
        torch.cuda.synchronize()
        np.testing.assert_array_equal(new_g.cpu().numpy(), new_o)
        assert hs.stats() == (len(X), 0)
    hs.clear()
    new_g = hs.filter(torch.from_numpy(hv.view(np.int64)).to(DEV), None)
    new_o, _ = oracle.hash_filter(hv, np.zeros(len(hv), np.uint8), set())
    np.testing.assert_array_equal(new_g.cpu().numpy(), new_o)


def test_filter_overflow_keeps_candidates_new():
    hs = HashSet(4)
    hv = np.arange(1, 11, dtype=np.uint64)
    new = hs.filter(torch.from_numpy(hv.view(np.int64)).to(DEV), None).cpu().numpy()
    assert new.all()
    n, ov = hs.stats()
    assert n == 4 and ov == 6


def test_graph_hash_then_filter_pipeline():
    """Alg. 3 lines 10-12 over GPU hashes of C5 candidates: duplicates of
    earlier decision vectors are filtered, exactly as the oracle's filter on
    the oracle's hashes of the same candidates."""
    wl = build_workload("c5")
    label = node_labels(wl)
    g = Graph.from_workload(wl, device=0)
    hz = GraphHasher(g, label)
    o = OracleGraph.from_workload(wl)
    K = 256
    _, D = CandidateGenerator(wl, CandidateSpec(seed=6, p_remat=20, p_swap=20)).generate(0, K)
    D = np.ascontiguousarray(D[:, :wl.R])
    st, h = hz.hash(torch.from_numpy(D).to(DEV))
    hs = HashSet(1 << 10)
    new = hs.filter(h, st).cpu().numpy()
    st_o, h_o = o.graph_hash_batch(label, D)
    new_o, _ = oracle.hash_filter(h_o, st_o, set())
    np.testing.assert_array_equal(new, new_o)
    assert 0 < new.sum() < K
