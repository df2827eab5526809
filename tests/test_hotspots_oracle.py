"""NEXT-3 pins of the oracle's hot-spots and heat / score (Eq. 3-4).

* Fig. 2(a): the 1056 peak is reached at steps 33 and 34, so the
  hot-spots are f1..f32, b1, b2; the dominator tree and Eq. 3-4 values are
  worked out by hand in the comments below.
* Random DAGs with random decisions: the oracle (C, event lists, dominator
  dataflow) against tests/_defn.py (interval sums, dominators by removal and
  reachability, Eq. 3-4 as set expressions).
"""
import numpy as np

from oracle import OracleGraph
from tests import _defn
from tests.test_oracle_pins import fig2a_graph, make, random_case, random_valid_perm


def test_fig2a_hotspots_dominators_heat_score():
    n, edges, size, outputs, f, b = fig2a_graph()
    g = make(n, edges, size, outputs)
    order = [f(i) for i in range(1, 33)] + [b(i) for i in range(1, 33)]
    st, pk, hot, heat, score = g.hotspots(order, nsplit=2)
    assert st == 0 and pk == 1056
    # step 33 holds f1..f32 + b1, step 34 holds f1..f31 + b1 + b2: both 33 x 32
    assert set(np.flatnonzero(hot)) == {f(i) for i in range(1, 33)} | {b(1), b(2)}
    # dominator tree: f_{i+1} <- f_i; b1 <- f32; b_j <- f_{33-j} (j >= 2)
    idom = g.idom()
    assert idom[f(1)] == -1
    for i in range(1, 32):
        assert idom[f(i + 1)] == f(i)
    assert idom[b(1)] == f(32)
    for j in range(2, 33):
        assert idom[b(j)] == f(33 - j)
    # des(f_k) = f_k..f32, b1, b_j (j <= 33-k); hot among them: f_k..f32, b1, b2 (k <= 31)
    for k in range(1, 33):
        want = 32 * ((33 - k) + 1 + (1 if k <= 31 else 0))
        assert heat[f(k)] == want
        assert score[f(k)] == want / 2          # its only input f_{k-1} is hot
    assert heat[b(1)] == 32 and score[b(1)] == 16.0      # input f32 hot
    assert heat[b(2)] == 32 and score[b(2)] == 16.0      # inputs b1, f31 hot
    assert heat[b(3)] == 0 and score[b(3)] == 0.0        # inputs b2, f30 hot
    for j in range(4, 33):
        assert heat[b(j)] == 0 and score[b(j)] == -32.0  # input b_{j-1} not hot


def test_idom_matches_removal_definition():
    rng = np.random.default_rng(5)
    for trial in range(150):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng, nmax=14)
        g = make(n, edges, size, outs, cost, elig, U)
        assert g.idom().tolist() == _defn.brute_idom(n, edges), trial


def test_hotspots_heat_score_match_definition():
    rng = np.random.default_rng(6)
    checked = 0
    for trial in range(300):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng, nmax=11)
        for r in range(len(elig)):
            if dec[r] == 1 and not any(v == elig[r] for _, v in edges):
                dec[r] = 2
        g = make(n, edges, size, outs, cost, elig, U)
        perm, _, _ = random_valid_perm(rng, n, edges, elig, U, dec)
        nsplit = int(rng.integers(1, 5))
        st, pk, hot, heat, score = g.hotspots(perm, dec if len(elig) else None, nsplit)
        H = _defn.defn_hotspots(n, edges, size, outs, elig, U, list(dec), perm)
        assert st == 0 and H is not None
        assert set(np.flatnonzero(hot)) == H, trial
        h2, s2 = _defn.defn_heat_score(n, edges, size, H, nsplit)
        assert heat.tolist() == h2, trial
        assert score.tolist() == s2, trial
        checked += 1
    assert checked == 300


def test_hotspots_invalid_candidate_is_zeroed():
    n, edges, size, outputs, f, b = fig2a_graph()
    g = make(n, edges, size, outputs)
    order = [f(i) for i in range(1, 33)] + [b(i) for i in range(1, 33)]
    order[0], order[1] = order[1], order[0]
    st, pk, hot, heat, score = g.hotspots(order)
    assert st == 2 and pk == -1 and not hot.any() and not heat.any() and not score.any()
