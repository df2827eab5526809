"""NEXT-4 pins: F-Trans variant regions (reading F1).

The variant graph holds, per F-Trans group (a region), the unsplit ops and
the splits by n = 2, 4 side by side; a candidate picks one variant per
region in dec[R + i].  The oracle's gated evaluation must equal the plain
evaluation of the graph the F-Trans materialiser builds for the same factors
(§4.2; magis_inputs.ftrans.apply_choice), on the same order of
the same ops -- status, peak and latency exactly.  The materialiser is input
code with none of the method's arithmetic, so this pins the gating (which
nodes and edges exist) to the paper's F-Trans rewrite.
"""
import numpy as np
import pytest

from magis_inputs import eligible, ftrans, models
from oracle import OracleGraph
from tests import _defn

NS = (1, 2, 4)


def small_bert(layers=2):
    return models.bert_large(B=4, S=64, ftrans=4, layers=layers)


def variant_workload(b, R_max=6):
    vb = ftrans.apply_variants(b, NS[1:])
    return eligible.select(vb.finish(), R_max), vb


def materialised(b, choice, tags):
    mb = ftrans.apply_choice(b, {t: NS[c] for t, c in zip(tags, choice)})
    return mb.finish(), mb


def random_order(rng, n, edges):
    """Random-priority Kahn over (n, edges)."""
    pre = [set() for _ in range(n)]
    succ = [[] for _ in range(n)]
    for u, v in edges:
        pre[v].add(u)
        succ[u].append(v)
    indeg = [len(p) for p in pre]
    ready = [v for v in range(n) if indeg[v] == 0]
    out = []
    while ready:
        i = int(rng.integers(0, len(ready)))
        v = ready.pop(i)
        out.append(v)
        for w in succ[v]:
            indeg[w] -= 1
            if indeg[w] == 0:
                ready.append(w)
    assert len(out) == n
    return out


@pytest.mark.parametrize("seed", range(6))
def test_gated_evaluation_equals_materialised_ftrans(seed):
    rng = np.random.default_rng(seed)
    b = small_bert()
    wl, vb = variant_workload(b)
    tags = vb.variant_tags
    F = wl.F
    og = OracleGraph.from_workload(wl)
    assert og.F == F and og.n_total == wl.n + 3 * wl.R
    choice = rng.integers(0, len(NS), F)
    dec = rng.integers(0, 3, wl.R).astype(np.uint8)
    for r in range(wl.R):
        if dec[r] == 1 and not any(d == wl.elig[r] for d in wl.dst):
            dec[r] = 2
    # the materialised graph of the same factors, with the same eligible tensors
    mw, mb = materialised(b, choice, tags)
    mid = {key: i for i, key in mb.prov.items()}
    assert len(mid) == mw.n                       # provenance keys are unique
    act = [v for v in range(wl.n) if wl.regions["node_region"][v] < 0 or
           choice[wl.regions["node_region"][v]] == wl.regions["node_variant"][v]]
    # the present nodes are exactly the ops of the materialised graph
    assert sorted(mid) == sorted(vb.prov[v] for v in act)
    vmap = {v: mid[vb.prov[v]] for v in act}
    for v, m in vmap.items():
        assert wl.size[v] == mw.size[m] and wl.cost[v] == mw.cost[m], (wl.names[v], mw.names[m])
    inv = {m: v for v, m in vmap.items()}
    melig = [vmap[t] for t in wl.elig]
    mU = [[vmap[u] for u in us] for us in wl.U]
    om = OracleGraph(mw.size, mw.cost, mw.is_output, mw.src, mw.dst, melig, mU, mw.swap_Bps, mw.swap_lat)
    for trial in range(3):
        # a valid order of the materialised super-graph (Fig. 8 on its ids)
        medges = list(zip(mw.src.tolist(), mw.dst.tolist()))
        active, te = _defn.transformed(mw.n, medges, melig, mU, list(dec))
        order_m = [v for v in random_order(rng, mw.n + 3 * wl.R, list(te)) if v in active]
        order_m += [v for v in range(mw.n, mw.n + 3 * wl.R) if v not in active]
        # the same order over the variant graph's ids; absent variants go last
        to_v = lambda m: inv[m] if m < mw.n else wl.n + (m - mw.n)
        order_v = [to_v(m) for m in order_m] + [v for v in range(wl.n) if v not in vmap]
        dv = np.concatenate([dec, choice.astype(np.uint8)])
        sv = og.eval(order_v, dv)
        sm = om.eval(order_m, dec if wl.R else None)
        assert sv[0] == sm[0] == 0
        assert sv[1] == sm[1]                 # peak bytes: exact
        assert sv[2] == sm[2]                 # latency: same terms in the same order


def test_all_unsplit_equals_base_graph():
    b = small_bert()
    wl, vb = variant_workload(b)
    base = b.finish()
    og = OracleGraph.from_workload(wl)
    ob = OracleGraph(base.size, base.cost, base.is_output, base.src, base.dst)
    bid = {("op", i): i for i in range(base.n)}
    rng = np.random.default_rng(3)
    order_b = random_order(rng, base.n, list(zip(base.src.tolist(), base.dst.tolist())))
    inv = {bid[vb.prov[v]]: v for v in range(wl.n)
           if wl.regions["node_region"][v] < 0 or wl.regions["node_variant"][v] == 0}
    order_v = [inv[m] for m in order_b] + [v for v in range(wl.n + 3 * wl.R) if v not in set(inv.values())]
    dv = np.zeros(wl.R + wl.F, np.uint8)
    assert og.eval(order_v, dv)[:3] == ob.eval(order_b)[:3]


def test_variant_index_out_of_range_is_bad_decision():
    b = small_bert(layers=1)
    wl, _ = variant_workload(b)
    og = OracleGraph.from_workload(wl)
    dv = np.zeros(wl.R + wl.F, np.uint8)
    dv[wl.R] = len(NS)
    st = og.eval(np.arange(wl.n + 3 * wl.R, dtype=np.int32), dv)[0]
    assert st == 4
