"""NEXT-2 pins of the oracle's GraphHash and hash filter (Alg. 3 lines 3-6
and 10-12; WL test P:1776-1778; readings G1-G4 in DESIGN.md).

* mix64 is the SplitMix64 output function: its values at k * GAMMA are the
  published first outputs of SplitMix64 seeded with 0.
* x_v is a hash of v's unfolding (ancestor) tree: on random DAGs with few
  labels (many coincidences) x_u == x_v exactly when brute-force canonical
  unfolding trees are equal, and two graphs hash alike exactly when the
  multisets of canonical trees agree (so a dropped term, a wrong
  predecessor set or an order dependence fails here).
* Relabelling node ids and re-ordering the eligible list leave the hash
  unchanged; the hash of a candidate equals the hash of its explicitly
  materialised Fig. 8 graph (tests/_defn.py) with all decisions 0.
* The filter equals the O(K^2) first-occurrence definition.
"""
import collections

import numpy as np

import oracle
from oracle import OracleGraph
from tests import _defn
from tests.test_oracle_pins import random_dag

GAMMA = 0x9E3779B97F4A7C15
TAG_STORE = 0x45524F5453     # reading G3
TAG_LOAD = 0x44414F4C
M64 = (1 << 64) - 1


def test_mix64_is_splitmix64():
    # SplitMix64 (Steele, Lea, Flood, OOPSLA '14), state 0: the first three
    # outputs are mix64(GAMMA), mix64(2 GAMMA), mix64(3 GAMMA)
    want = [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]
    assert [oracle.mix64(k * GAMMA & M64) for k in (1, 2, 3)] == want


def test_hash_words_is_order_and_length_sensitive():
    a, b = 0x1234, 0xABCDEF
    assert oracle.hash_words([a, b]) != oracle.hash_words([b, a])
    assert oracle.hash_words([0]) != oracle.hash_words([0, 0])
    assert oracle.hash_words([]) != oracle.hash_words([0])


def _graph(n, edges, elig=(), U=()):
    size = [1] * n
    iso = np.zeros(n, np.uint8)
    iso[n - 1] = 1
    return OracleGraph(size, [0.0] * n, iso, [u for u, _ in edges], [v for _, v in edges],
                       list(elig), [list(u) for u in U])


def _random_case(rng, nmax=12, nlab=3):
    n = int(rng.integers(3, nmax + 1))
    edges = random_dag(rng, n)
    label = rng.integers(1, nlab + 1, n).astype(np.uint64)
    cons = {u: sorted({v for (a, v) in edges if a == u}) for u in range(n)}
    has_in = {v for (_, v) in edges}
    cand = [u for u in range(n - 1) if cons[u] and u in has_in]
    rng.shuffle(cand)
    elig = cand[: int(rng.integers(0, len(cand) + 1))]
    U = [sorted(rng.choice(cons[t], size=int(rng.integers(1, len(cons[t]) + 1)), replace=False).tolist())
         for t in elig]
    dec = rng.integers(0, 3, len(elig)).astype(np.uint8)
    return n, edges, label, elig, U, dec


def _canon(n, edges, label, elig, U, dec):
    """Brute-force canonical unfolding trees of the transformed graph's active
    nodes: canon(v) = (label(v), sorted canon(u) over pre(v))."""
    active, te = _defn.transformed(n, edges, elig, U, list(dec))
    pre = collections.defaultdict(list)
    for u, v in te:
        pre[v].append(u)

    def lab(v):
        if v < n:
            return int(label[v])
        r, k = divmod(v - n, 3)
        return int(label[elig[r]]) if k == 0 else (TAG_STORE if k == 1 else TAG_LOAD)

    memo = {}

    def canon(v):
        if v not in memo:
            memo[v] = (lab(v), tuple(sorted(canon(u) for u in pre[v])))
        return memo[v]

    return {v: canon(v) for v in active}


def test_node_hash_equals_unfolding_tree_equivalence():
    rng = np.random.default_rng(21)
    pairs_eq = pairs = 0
    for trial in range(250):
        n, edges, label, elig, U, dec = _random_case(rng)
        g = _graph(n, edges, elig, U)
        st, h, x = g.graph_hash(label, dec if len(elig) else None)
        assert st == 0
        cz = _canon(n, edges, label, elig, U, dec)
        for v in range(g.n_total):
            if v not in cz:
                assert x[v] == 0, (trial, v)
        act = sorted(cz)
        for i, u in enumerate(act):
            for v in act[i + 1:]:
                pairs += 1
                same = cz[u] == cz[v]
                pairs_eq += same
                assert (int(x[u]) == int(x[v])) == same, (trial, u, v)
    assert pairs_eq > 100 and pairs > 5 * pairs_eq   # the pin sees both outcomes


def test_graph_hash_equals_multiset_of_unfolding_trees():
    """Pairs of graphs: equal hashes iff equal multisets of canonical trees
    (line 6 sums x_v over all nodes)."""
    rng = np.random.default_rng(22)
    eq = 0
    cases = [_random_case(rng, nmax=7, nlab=2) for _ in range(120)]
    sig, hs = [], []
    for n, edges, label, elig, U, dec in cases:
        g = _graph(n, edges, elig, U)
        st, h, _ = g.graph_hash(label, dec if len(elig) else None)
        assert st == 0
        sig.append(collections.Counter(_canon(n, edges, label, elig, U, dec).values()))
        hs.append(h)
    for i in range(len(cases)):
        for j in range(i + 1, len(cases)):
            same = sig[i] == sig[j]
            eq += same
            assert (hs[i] == hs[j]) == same, (i, j)
    assert eq > 0


def test_hash_invariant_under_relabelling():
    rng = np.random.default_rng(23)
    for trial in range(200):
        n, edges, label, elig, U, dec = _random_case(rng, nlab=4)
        g = _graph(n, edges, elig, U)
        _, h0, _ = g.graph_hash(label, dec if len(elig) else None)
        # a random relabelling of the ops (keep the output last for _graph)
        p = np.concatenate([rng.permutation(n - 1), [n - 1]])
        e2 = [(int(p[u]), int(p[v])) for u, v in edges]
        lab2 = np.zeros(n, np.uint64)
        lab2[p] = label
        ro = rng.permutation(len(elig))
        el2 = [int(p[elig[r]]) for r in ro]
        U2 = [sorted(int(p[b]) for b in U[r]) for r in ro]
        dec2 = np.array([dec[r] for r in ro], np.uint8)
        g2 = _graph(n, e2, el2, U2)
        _, h1, _ = g2.graph_hash(lab2, dec2 if len(elig) else None)
        assert h0 == h1, trial


def test_hash_equals_hash_of_materialised_transform():
    """Fig. 8 applied by hand (tests/_defn.transformed) to a plain graph with
    the G3 labels for clone / Store / Load: same hash as the decisions."""
    rng = np.random.default_rng(24)
    for trial in range(200):
        n, edges, label, elig, U, dec = _random_case(rng, nlab=5)
        if not len(elig):
            continue
        g = _graph(n, edges, elig, U)
        _, h0, _ = g.graph_hash(label, dec)
        active, te = _defn.transformed(n, edges, elig, U, list(dec))
        ids = {v: i for i, v in enumerate(sorted(active, key=lambda v: (v != n - 1, v)))}
        m = len(ids)
        lab = np.zeros(m, np.uint64)
        for v, i in ids.items():
            if v < n:
                lab[i] = label[v]
            else:
                r, k = divmod(v - n, 3)
                lab[i] = label[elig[r]] if k == 0 else (TAG_STORE if k == 1 else TAG_LOAD)
        e2 = [(ids[u], ids[v]) for u, v in te]
        g2 = _graph(m, e2) if e2 else None
        if g2 is None:
            continue
        # _graph marks the last id as output; outputs do not enter the hash
        order = sorted(ids, key=lambda v: ids[v])
        perm_out = [ids[v] for v in order]
        assert perm_out == list(range(m))
        _, h1, _ = g2.graph_hash(lab)
        assert h0 == h1, trial


def test_hash_sensitive_to_edges_labels_and_decisions():
    rng = np.random.default_rng(25)
    for trial in range(200):
        n, edges, label, elig, U, dec = _random_case(rng, nlab=1000)
        g = _graph(n, edges, elig, U)
        _, h0, _ = g.graph_hash(label, dec if len(elig) else None)
        lab2 = label.copy()
        v = int(rng.integers(0, n))
        lab2[v] = np.uint64(int(label[v]) + 1000)
        assert g.graph_hash(lab2, dec if len(elig) else None)[1] != h0
        missing = [(u, v) for u in range(n) for v in range(u + 1, n) if (u, v) not in set(edges)]
        if missing:
            e2 = edges + [missing[int(rng.integers(0, len(missing)))]]
            assert _graph(n, e2).graph_hash(label)[1] != _graph(n, edges).graph_hash(label)[1]
        if len(elig):
            d2 = dec.copy()
            d2[0] = (d2[0] + 1) % 3
            assert g.graph_hash(label, d2)[1] != h0


def test_clone_hashes_like_its_original():
    """A' is the same op on the same inputs: equal unfolding
    trees, so x(A') = x(A)."""
    rng = np.random.default_rng(26)
    seen = 0
    for trial in range(100):
        n, edges, label, elig, U, dec = _random_case(rng)
        if not len(elig):
            continue
        dec[:] = 1
        g = _graph(n, edges, elig, U)
        st, h, x = g.graph_hash(label, dec)
        for r, t in enumerate(elig):
            assert x[n + 3 * r] == x[t]
            seen += 1
    assert seen > 20


def test_bad_decisions_and_batch():
    rng = np.random.default_rng(27)
    n, edges, label, elig, U, dec = _random_case(rng, nmax=12)
    while not len(elig):
        n, edges, label, elig, U, dec = _random_case(rng, nmax=12)
    g = _graph(n, edges, elig, U)
    D = rng.integers(0, 3, (50, len(elig))).astype(np.uint8)
    D[7, 0] = 3
    st, hs = g.graph_hash_batch(label, D)
    assert st[7] == 4 and hs[7] == 0
    for k in range(50):
        s1, h1, _ = g.graph_hash(label, D[k])
        assert (s1, h1) == (st[k], hs[k])


def _filter_defn(hashes, status, X):
    """Candidate k is new iff valid, its hash not in X and no earlier valid
    candidate j < k has the same hash (Alg. 3 lines 10-12 in id order)."""
    K = len(hashes)
    return np.array([int(status[k] == 0 and int(hashes[k]) not in X and
                         not any(status[j] == 0 and hashes[j] == hashes[k] for j in range(k)))
                     for k in range(K)], np.uint8)


def test_filter_matches_first_occurrence_definition():
    rng = np.random.default_rng(28)
    for trial in range(30):
        K = int(rng.integers(0, 200))
        hashes = rng.integers(0, 40, K).astype(np.uint64)
        hashes[rng.random(K) < 0.05] = 0          # hash value 0 is an ordinary key
        status = (rng.random(K) < 0.1).astype(np.uint8) * 4
        X = set(int(h) for h in rng.integers(0, 40, 5))
        new, X2 = oracle.hash_filter(hashes, status, X)
        assert (new == _filter_defn(hashes, status, X)).all()
        assert X2 == X | {int(h) for h, s in zip(hashes, status) if s == 0}
