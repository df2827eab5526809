"""Input generators (magis_inputs): F-Trans byte pins, candidate validity,
determinism, eligible set vs hot-spots.  CPU only."""
import numpy as np
import pytest

from magis_inputs import CandidateGenerator, CandidateSpec, build_workload, ftrans, models
from oracle import OracleGraph


def test_ftrans_parts_shrink_bytes_by_n():
    """F-Trans with factor n (P15, Mutating Rule P:1315-1317):
    every positive-dim part holds |v|/n bytes, the parts sum to |v|, reduce
    partials stay full size, merges restore |v|."""
    for n in (2, 4):
        b = models.bert_large(B=8, S=64, ftrans=n)
        f = ftrans.apply(b, n)
        assert len(f.fission_map) > 0
        for v, parts in f.fission_map.items():
            assert len(parts) == n
            if b.splitdim[v] > 0:
                assert all(f.size[p] * n == b.size[v] for p in parts)
                assert sum(f.size[p] for p in parts) == b.size[v]
            else:
                assert all(f.size[p] == b.size[v] for p in parts)
        # merge nodes restore the full size
        for i, name in enumerate(f.names):
            if name.endswith(".concat") or name.endswith(".addmerge"):
                base = name.rsplit(".", 1)[0]
                j = b.names.index(base)
                assert f.size[i] == b.size[j]


def test_ftrans_slices_and_shared_inputs():
    """Fig. 5: inputs with the split dim are sliced per part,
    weights are shared unsliced; weight gradients are reduce (Add) merges."""
    b = models.bert_large(B=8, S=64, ftrans=2)
    f = ftrans.apply(b, 2)
    slices = [x for x in f.names if ".slice" in x]
    assert slices
    adds = [x for x in f.names if x.endswith(".addmerge")]
    assert any(".dW" in a for a in adds)
    # weights never sliced
    for s in slices:
        base = s.rsplit(".slice", 1)[0]
        assert f.kind[f.names.index(base)] != "weight"


def test_generated_graphs_are_dags_in_natural_order():
    for cfg in ("c2", "c5"):
        wl = build_workload(cfg)
        assert (wl.src < wl.dst).all()
        assert wl.R > 0 and all(len(u) >= 1 for u in wl.U)
        cons = {}
        for u, v in zip(wl.src.tolist(), wl.dst.tolist()):
            cons.setdefault(u, set()).add(v)
        for t, U in zip(wl.elig.tolist(), wl.U):
            assert set(U) <= cons[t] and not wl.is_output[t]


def test_eligible_tensors_are_hot_spots():
    """The hot-spot proxy (reading R-hot) mostly selects tensors that are live
    at the natural order's peak step, checked with the oracle."""
    for cfg, frac in (("c2", 0.8), ("c5", 0.99)):
        wl = build_workload(cfg)
        n = wl.n
        g = OracleGraph(wl.size, wl.cost, wl.is_output, wl.src, wl.dst)
        st, pk, lt, am = g.eval(np.arange(n, dtype=np.int32))
        last = np.arange(n)
        np.maximum.at(last, wl.src, wl.dst)
        last[wl.is_output == 1] = n - 1
        live = (np.arange(n) <= am) & (last >= am)
        assert wl.size[live].sum() == pk
        assert live[wl.elig].mean() >= frac


def test_candidates_deterministic_and_shard_independent():
    wl = build_workload("c2")
    gen = CandidateGenerator(wl, CandidateSpec(seed=7))
    P, D = gen.generate(0, 300)
    P2, D2 = gen.generate(100, 50, nthreads=1)
    assert (P[100:150] == P2).all() and (D[100:150] == D2).all()
    P3, _ = CandidateGenerator(wl, CandidateSpec(seed=8)).generate(0, 300)
    assert (P3 != P).any()


def test_candidates_valid_except_transpositions():
    """F1 / F2 candidates are valid by construction; only the 1% F3
    transpositions may violate an edge (checked with the oracle)."""
    wl = build_workload("c2")
    gen = CandidateGenerator(wl)
    P, D = gen.generate(0, 2000)
    g = OracleGraph.from_workload(wl)
    st, pk, lt = g.eval_batch(P, D)
    assert (np.sort(P, axis=1) == np.arange(wl.n_total)).all()
    assert set(np.unique(st).tolist()) <= {0, 2}
    assert 0 < (st == 2).sum() <= 60
    # decisions ~5% / 5%
    frac = np.bincount(D.ravel(), minlength=3) / D.size
    assert abs(frac[1] - 0.05) < 0.01 and abs(frac[2] - 0.05) < 0.01
    # all-keep candidates have swap-free latency = sum cost
    keep = (D == 0).all(axis=1) & (st == 0)
    if keep.any():
        assert np.allclose(lt[keep], wl.cost.sum(), rtol=1e-12)


@pytest.mark.parametrize("cfg", ["c3", "c4"])
def test_big_graph_sizes(cfg):
    wl = build_workload(cfg)
    s = wl.summary()
    if cfg == "c3":
        assert 5000 <= s["n_total"] <= 8000
    else:
        assert 16384 < s["n_total"] <= 30000       # multi-CTA-sized graph
        assert s["sum_bytes"] > 2 ** 31


def test_random_orders_follow_the_keyed_kahn_recipe():
    """F1 candidates are the keyed Kahn order of the recipe (candgen.c header,
    DESIGN §5): at every step the ready node with the smallest (priority, id),
    priority = the top 16 bits of rnd(seed, k, KEY, v), rnd = three SplitMix64
    mixes.  Written here from the recipe, independently of candgen.c; the
    device generator is held byte-identical to candgen.c by the GPU tests."""
    import heapq
    M = (1 << 64) - 1

    def mix(x):
        x = (x + 0x9E3779B97F4A7C15) & M
        x = ((x ^ (x >> 30)) * 0xBF58476D1CE4E5B9) & M
        x = ((x ^ (x >> 27)) * 0x94D049BB133111EB) & M
        return x ^ (x >> 31)

    def rnd(seed, k, stream, i):
        h = mix((seed + 0x9E3779B97F4A7C15 * (stream + 1)) & M)
        return mix(mix(h ^ k) ^ i)

    wl = build_workload("c2")
    n, seed = wl.n, 21
    spec = CandidateSpec(seed=seed, pct_random=100, pct_local=0, p_remat=0, p_swap=0)
    P, _ = CandidateGenerator(wl, spec).generate(40, 6)
    preds = [[] for _ in range(n)]
    succs = [[] for _ in range(n)]
    for u, v in set(zip(wl.src.tolist(), wl.dst.tolist())):
        preds[v].append(u)
        succs[u].append(v)
    for i in range(6):
        k = 40 + i
        key = [rnd(seed, k, 3, v) >> 48 for v in range(n)]
        indeg = [len(p) for p in preds]
        ready = [(key[v], v) for v in range(n) if indeg[v] == 0]
        heapq.heapify(ready)
        order = []
        while ready:
            _, u = heapq.heappop(ready)
            order.append(u)
            for s in succs[u]:
                indeg[s] -= 1
                if indeg[s] == 0:
                    heapq.heappush(ready, (key[s], s))
        assert P[i, :n].tolist() == order
