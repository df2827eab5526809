"""Pins for the CPU oracle (oracle/), independent of the CUDA path.

Every expected number here comes from the paper (cited) or from mathematics
(closed forms, brute force over all topological orders, invariants) -- never
from the GPU.  See DESIGN.md §Oracle for the readings (P1..P18).
"""
import itertools
import math

import numpy as np
import pytest

import oracle
from oracle import OracleGraph
from tests import _defn
from tests.golden import PAPER


# ---------------------------------------------------------------- fixtures --

def fig2a_graph():
    """Fig. 2(a): f1..f32 chain, b1..b32 chain, skip
    f_i -> b_{33-i}; every tensor 32; output b32.  ids: f_i = i-1, b_i = 31+i."""
    f = lambda i: i - 1
    b = lambda i: 31 + i
    edges = []
    for i in range(1, 32):
        edges.append((f(i), f(i + 1)))
        edges.append((b(i), b(i + 1)))
    for i in range(1, 33):
        edges.append((f(i), b(33 - i)))
    n = 64
    size = [32] * n
    outputs = [b(32)]
    return n, edges, size, outputs, f, b


def make(n, edges, size, outputs, cost=None, elig=(), U=(), B=25e9, lam=1e-5):
    iso = np.zeros(n, np.uint8)
    iso[list(outputs)] = 1
    src = [u for u, _ in edges]
    dst = [v for _, v in edges]
    cost = [0.0] * n if cost is None else cost
    return OracleGraph(size, cost, iso, src, dst, list(elig), [list(u) for u in U], B, lam)


# ------------------------------------------------------ paper worked examples --

def test_fig2a_peak_is_1056_at_step_33():
    """'a peak memory usage of 1056 since 33 tensors with size 32 are alive
    when computing the 33-th operator'."""
    n, edges, size, outs, f, b = fig2a_graph()
    g = make(n, edges, size, outs)
    order = list(range(64))  # f1..f32, b1..b32
    st, peak, lat, arg = g.eval(order)
    assert st == 0
    assert peak == PAPER["fig2a.peak"] == PAPER["fig2a.live_tensors_at_peak"] * PAPER["fig2a.tensor_size"]
    assert arg == PAPER["fig2a.peak_operator"] - 1     # 0-based step 32 == the 33rd operator
    # the independent interval-sum definition agrees
    pk, a2 = _defn.interval_peak(order, edges, dict(enumerate(size)), set(outs))
    assert (pk, a2) == (PAPER["fig2a.peak"], PAPER["fig2a.peak_operator"] - 1)


def test_fig2a_literal_formula_is_off_by_one():
    """The literal A_i = {v_j | S_j <= i <= F_j} with S_j = j-1
    gives 1088, contradicting the text's 1056 -> reading P1."""
    n, edges, size, outs, f, b = fig2a_graph()
    order = list(range(64))
    assert _defn.literal_peak(order, edges, dict(enumerate(size)), set(outs)) == 1088


def test_fig2b_swapping_peak_is_96():
    """Fig. 2(b): swapping every skip tensor with the
    Store right after its producer and the Load right before its backward
    consumer gives a 96 peak ('4 free memory' under the 100 limit)."""
    n, edges, size, outs, f, b = fig2a_graph()
    elig = [f(i) for i in range(1, 32)]          # f32 -> b1 is not a skip
    U = [[b(33 - i)] for i in range(1, 32)]
    g = make(n, edges, size, outs, elig=elig, U=U)
    R = len(elig)
    store = lambda i: n + 3 * (i - 1) + 1
    load = lambda i: n + 3 * (i - 1) + 2
    clone = lambda i: n + 3 * (i - 1)
    order = []
    for i in range(1, 32):
        order += [f(i), store(i)]
    order += [f(32), b(1)]
    for k in range(2, 33):
        order += [load(33 - k), b(k)]
    order += [clone(i) for i in range(1, 32)]
    assert sorted(order) == list(range(n + 3 * R))
    dec = np.full(R, 2, np.uint8)
    st, peak, lat, arg = g.eval(order, dec)
    assert st == 0 and peak == PAPER["fig2b.peak"] <= PAPER["fig2b.memory_limit"]
    # forward phase alone peaks at 64
    st2, pk2 = _defn.defn_eval(n, edges, size, outs, elig, U, dec, order)
    assert (st2, pk2) == (0, PAPER["fig2b.peak"])


# ------------------------------------------------ hand-computed toy timelines --

T1_EDGES = [(0, 1), (1, 2), (2, 3), (0, 3)]


@pytest.mark.parametrize("order,dec,B,exp", [
    ([0, 1, 2, 3, 4, 5, 6], 0, 100.0, (0, 500, 4.0)),
    ([0, 5, 1, 2, 6, 3, 4], 2, 100.0, (0, 400, 4.0)),   # transfer hidden
    ([0, 5, 1, 2, 6, 3, 4], 2, 50.0, (0, 400, 6.0)),    # d stalls 2 s
    ([0, 5, 1, 6, 2, 3, 4], 2, 50.0, (0, 500, 6.0)),    # load too early
    ([0, 6, 5, 1, 2, 3, 4], 2, 50.0, (2, -1, math.inf)),  # load before store
])
def test_T1_swap_toy(order, dec, B, exp):
    """a->b->c->d + a->d, sizes 100/200/200/10, cost 1,
    eligible (a, U={d}), lambda = 0 (reading P7, worked by hand)."""
    g = make(4, T1_EDGES, [100, 200, 200, 10], [3], cost=[1.0] * 4,
             elig=[0], U=[[3]], B=B, lam=0.0)
    st, peak, lat, _ = g.eval(order, np.array([dec], np.uint8))
    assert (st, peak) == exp[:2]
    assert lat == exp[2]


# T3: two swaps contending on both copy queues.  a->b->c->d->e plus the skips
# a->e, b->e; sizes a=b=100, c=d=10, e=1 (output); costs 1.0; eligible
# r=0: (a, U={e}), r=1: (b, U={e}); B = 50 B/s, lambda = 0.5 s, so every
# transfer takes 0.5 + 100/50 = 2.5 s.  Ids a..e = 0..4, clone0/store0/load0
# = 5/6/7, clone1/store1/load1 = 8/9/10.
T3_EDGES = [(0, 1), (1, 2), (2, 3), (3, 4), (0, 4), (1, 4)]
T3_ARGS = dict(n=5, edges=T3_EDGES, size=[100, 100, 10, 10, 1], outputs=[4], cost=[1.0] * 5,
               elig=[0, 1], U=[[4], [4]], B=50.0, lam=0.5)


@pytest.mark.parametrize("order,dec,exp", [
    # no swap: sum of costs; a, b, c, d all live at step 3 -> 220
    ([0, 1, 2, 3, 4, 5, 6, 7, 8, 9, 10], (0, 0), (0, 220, 5.0)),
    # B: a b St0 St1 c Ld1 d Ld0 e.  compute a[0,1] b[1,2] c[2,3] d[3,4];
    #    St0 = max(Td 0, a 1) -> [1, 3.5];  St1 = max(Td 3.5, b 2) -> [3.5, 6]
    #    (D2H contention: alone it would be [2, 4.5]);
    #    Ld1 = max(Th 0, St1 6) -> [6, 8.5];  Ld0 = max(Th 8.5, St0 3.5) -> [8.5, 11]
    #    (H2D contention: alone it would be [3.5, 6]);
    #    e = max(Tc 4, Ld0 11, Ld1 8.5) -> [11, 12].  Without the D2H queue the
    #    makespan is 10.5, without the H2D queue 9.5, without either 8.0.
    #    Memory: a 0..2, b 1..4, c 4..6, Ld1 5..8, d 6..8, Ld0 7..8, e 8 -> 211.
    ([0, 1, 6, 9, 2, 10, 3, 7, 4, 5, 8], (2, 2), (0, 211, 12.0)),
    # C: a b St0 St1 c d Ld0 Ld1 e: transfer bound, Ld1 = [6, 8.5] either way,
    #    e = [8.5, 9.5]
    ([0, 1, 6, 9, 2, 3, 7, 10, 4, 5, 8], (2, 2), (0, 211, 9.5)),
    # D: only a swapped: St0 [1, 3.5], Ld0 = [3.5, 6] after d [3, 4] -> e [6, 7];
    #    b stays live to e: b + d + Ld0 + e = 211 at the last step
    ([0, 1, 6, 2, 3, 7, 4, 5, 8, 9, 10], (2, 0), (0, 211, 7.0)),
    # E: both swapped, Ld0 issued before St1 finished: a St0 b St1 Ld0 Ld1 c d e
    #    St0 [1, 3.5], St1 [3.5, 6], Ld0 = max(0, 3.5) -> [3.5, 6], Ld1 = max(6, 6)
    #    -> [6, 8.5]; c [2, 3], d [3, 4]; e = [8.5, 9.5].  The Loads come too
    #    early for memory: b (to c), Ld0, Ld1 and c are live at step 6 -> 310
    ([0, 6, 1, 9, 7, 10, 2, 3, 4, 5, 8], (2, 2), (0, 310, 9.5)),
])
def test_T3_two_swap_queue_contention(order, dec, exp):
    """Hand-worked timelines (reading P7): rows B and E need
    both the D2H (Td) and the H2D (Th) serialisation; the event-DAG longest
    path (tests/_defn.py) reproduces every row."""
    a = T3_ARGS
    g = make(a["n"], a["edges"], a["size"], a["outputs"], cost=a["cost"], elig=a["elig"], U=a["U"],
             B=a["B"], lam=a["lam"])
    st, peak, lat, _ = g.eval(order, np.array(dec, np.uint8))
    assert (st, peak) == exp[:2]
    assert lat == exp[2]
    assert _defn.defn_latency(a["n"], a["edges"], a["cost"], a["size"], a["elig"], a["U"], dec, order,
                              a["B"], a["lam"]) == exp[2]
    assert _defn.defn_eval(a["n"], a["edges"], a["size"], a["outputs"], a["elig"], a["U"], dec, order) == exp[:2]


def test_T3_queue_ablation_changes_the_makespan():
    """The two copy queues are what row B measures: dropping the D2H or the
    H2D chain from the event DAG changes its makespan to 10.5 / 9.5 (the
    values worked out in the row's comment), so an oracle without either
    serialisation could not produce 12.0."""
    a = T3_ARGS
    order = [0, 1, 6, 9, 2, 10, 3, 7, 4, 5, 8]
    w, arcs = _defn.event_dag(a["n"], a["edges"], a["cost"], a["size"], a["elig"], a["U"], (2, 2), order,
                              a["B"], a["lam"])
    assert _defn.longest_path_latency(w, arcs) == 12.0
    assert _defn.longest_path_latency(w, arcs - {(6, 9)}) == 10.5          # no D2H queue
    assert _defn.longest_path_latency(w, arcs - {(10, 7)}) == 9.5          # no H2D queue
    assert _defn.longest_path_latency(w, arcs - {(6, 9), (10, 7)}) == 8.0


def test_swap_latency_matches_event_dag_on_random_dags():
    """Random DAGs with swaps (positive lambda, slow links so transfers
    contend): the oracle's three-queue recurrence equals the event-DAG longest
    path within fp64 rounding.  The cases are counted where dropping the D2H
    or the H2D queue chain from the DAG changes the makespan -- there the
    oracle could not match without that serialisation."""
    rng = np.random.default_rng(777)
    nswap = nd2h = nh2d = 0
    for _ in range(8000):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        if len(elig) == 0:
            continue
        dec = np.where(rng.random(len(elig)) < 0.7, 2, dec).astype(np.uint8)
        if not (dec == 2).any():
            continue
        B = float(rng.choice([1.0, 10.0, 1e3]))
        lam = float(rng.random())
        g = make(n, edges, size, outs, cost=cost, elig=elig, U=U, B=B, lam=lam)
        perm, te, active = random_valid_perm(rng, n, edges, elig, U, dec)
        st, pk, lat, _ = g.eval(perm, dec)
        assert st == 0
        w, arcs = _defn.event_dag(n, edges, cost, size, elig, U, dec, perm, B, lam)
        ref = _defn.longest_path_latency(w, arcs)
        assert abs(lat - ref) <= 1e-12 * max(1.0, abs(ref)), (lat, ref)
        order = [v for v in perm if v in w]
        st_q = [x for x in order if x >= n and (x - n) % 3 == 1]
        ld_q = [x for x in order if x >= n and (x - n) % 3 == 2]
        nd2h += _defn.longest_path_latency(w, arcs - set(zip(st_q, st_q[1:]))) != ref
        nh2d += _defn.longest_path_latency(w, arcs - set(zip(ld_q, ld_q[1:]))) != ref
        nswap += 1
        if nswap == 800:
            break
    assert nswap == 800 and nd2h > 50 and nh2d > 50, (nswap, nd2h, nh2d)


T2_EDGES = [(0, 1), (1, 2), (2, 3), (3, 4), (1, 4)]


@pytest.mark.parametrize("order,dec,exp", [
    ([0, 1, 2, 3, 4, 5, 6, 7], 0, (0, 500, 5.0)),
    ([0, 1, 2, 3, 5, 4, 6, 7], 1, (0, 410, 7.0)),   # x held for the clone
    ([0, 1, 5, 2, 3, 4, 6, 7], 1, (0, 500, 7.0)),   # clone too early
])
def test_T2_remat_toy(order, dec, exp):
    """x->a->b->c->d + a->d, sizes 10/100/200/200/10, costs
    0/2/1/1/1; re-materialising a for d adds cost(a) (reading P9)."""
    g = make(5, T2_EDGES, [10, 100, 200, 200, 10], [4], cost=[0.0, 2.0, 1.0, 1.0, 1.0],
             elig=[1], U=[[4]])
    st, peak, lat, _ = g.eval(order, np.array([dec], np.uint8))
    assert (st, peak, lat) == exp


def test_remat_of_input_placeholder_is_bad_decision():
    """A' needs A's inputs: dec=1 on a tensor without inputs is
    flagged bit2; dec=2 on it is fine (T1 uses exactly that)."""
    g = make(4, T1_EDGES, [100, 200, 200, 10], [3], cost=[1.0] * 4, elig=[0], U=[[3]])
    st, pk, lat, _ = g.eval([0, 4, 1, 2, 3, 5, 6], np.array([1], np.uint8))
    assert st == 4 and pk == -1 and lat == math.inf


def test_status_bits():
    g = make(4, T1_EDGES, [100, 200, 200, 10], [3], cost=[1.0] * 4, elig=[0], U=[[3]])
    assert g.eval([0, 1, 2, 3, 4, 5, 5], np.array([0], np.uint8))[0] == 1   # duplicate
    assert g.eval([0, 1, 2, 3, 4, 5, 7], np.array([0], np.uint8))[0] == 1   # out of range
    assert g.eval([0, 1, 2, 3, 4, 5, 6], np.array([3], np.uint8))[0] == 4   # bad decision
    assert g.eval([0, 1, 2, 3, 4, 5, 7], np.array([3], np.uint8))[0] == 5   # both
    assert g.eval([1, 0, 2, 3, 4, 5, 6], np.array([0], np.uint8))[0] == 2   # edge violated


# ----------------------------------------------------------- closed forms --

def test_chain_closed_form():
    rng = np.random.default_rng(7)
    for _ in range(20):
        n = int(rng.integers(2, 30))
        size = [int(x) for x in rng.integers(1, 1 << 40, n)]
        edges = [(i, i + 1) for i in range(n - 1)]
        g = make(n, edges, size, [n - 1])
        exp = max([size[0]] + [size[i - 1] + size[i] for i in range(1, n)])
        assert g.eval(list(range(n)))[1] == exp


def test_U_shape_closed_form():
    """U(k, s): k forward + k backward with skips -> (k+1)*s (Fig. 2(a) at k=32)."""
    for k in range(1, 20):
        for s in (1, 32, 4096):
            n = 2 * k
            edges = [(i, i + 1) for i in range(k - 1)] + [(k + i, k + i + 1) for i in range(k - 1)]
            edges += [(i - 1, k + (k - i)) for i in range(1, k + 1)]
            g = make(n, edges, [s] * n, [n - 1])
            assert g.eval(list(range(n)))[1] == (k + 1) * s


def test_fanout_is_order_invariant():
    """source -> k singletons -> sink: every order has the same peak
    max(|src| + sum|m|, sum|m| + |sink|)."""
    rng = np.random.default_rng(3)
    k = 5
    n = k + 2
    edges = [(0, 1 + j) for j in range(k)] + [(1 + j, k + 1) for j in range(k)]
    size = [int(x) for x in rng.integers(1, 1000, n)]
    g = make(n, edges, size, [k + 1])
    exp = max(size[0] + sum(size[1:k + 1]), sum(size[1:k + 1]) + size[k + 1])
    for mid in itertools.permutations(range(1, k + 1)):
        assert g.eval([0, *mid, k + 1])[1] == exp


# ------------------------------------------------------------ brute force --

def diamond(branches, rng):
    """C1 diamond: source -> chains of given lengths -> sink, sizes 512 B x U[1,2^20)."""
    n = 2 + sum(branches)
    edges = []
    nid = 1
    for L in branches:
        prev = 0
        for _ in range(L):
            edges.append((prev, nid))
            prev = nid
            nid += 1
        edges.append((prev, n - 1))
    size = [512 * int(x) for x in rng.integers(1, 1 << 20, n)]
    return n, edges, size


@pytest.mark.parametrize("branches", [[4, 4], [3, 3, 2], [2, 2, 2, 2]])
def test_bruteforce_all_orders_match_interval_definition(branches):
    """Every topological order of a C1 diamond: the oracle's event simulation
    equals the interval-sum definition, and min/max are the
    brute-force optimum / worst (orders matter)."""
    varied = 0
    for seed in range(4):
        rng = np.random.default_rng(1000 * seed + sum(branches))
        n, edges, size = diamond(branches, rng)
        g = make(n, edges, size, [n - 1])
        orders = _defn.all_topo_orders(n, edges)
        exp_count = math.factorial(sum(branches)) // math.prod(math.factorial(b) for b in branches)
        assert len(orders) == exp_count
        perms = np.array(orders, np.int32)
        st, pk, lt = g.eval_batch(perms)
        assert (st == 0).all()
        ref = [_defn.interval_peak(o, edges, dict(enumerate(size)), {n - 1})[0] for o in orders]
        assert list(pk) == ref
        varied += int(pk.min() < pk.max())
        # order-invariant latency without swaps
        assert np.all(lt == lt[0])
    assert varied >= 2                   # the order matters on these shapes


def random_dag(rng, n, p=0.35):
    edges = [(u, v) for v in range(n) for u in range(v) if rng.random() < p]
    return edges


def random_case(rng, nmax=11):
    n = int(rng.integers(3, nmax + 1))
    edges = random_dag(rng, n)
    size = [int(x) for x in rng.integers(0, 1 << 40, n)]
    cost = [float(x) for x in rng.random(n)]
    outs = [v for v in range(n) if rng.random() < 0.2] or [n - 1]
    cons = {u: sorted({v for (a, v) in edges if a == u}) for u in range(n)}
    has_in = {v for (_, v) in edges}
    cand = [u for u in range(n) if u not in outs and len(cons[u]) >= 2 and u in has_in]
    rng.shuffle(cand)
    elig = cand[: int(rng.integers(0, len(cand) + 1))]
    U = []
    for t in elig:
        c = cons[t]
        k = int(rng.integers(1, len(c)))
        U.append(sorted(rng.choice(c, size=k, replace=False).tolist()))
    dec = rng.integers(0, 3, len(elig)).astype(np.uint8)
    return n, edges, size, cost, outs, elig, U, dec


def random_valid_perm(rng, n, edges, elig, U, dec):
    active, te = _defn.transformed(n, edges, elig, U, list(dec))
    pre = {v: set() for v in active}
    for u, v in te:
        pre[v].add(u)
    order, done = [], set()
    while len(order) < len(active):
        ready = sorted(v for v in active if v not in done and pre[v] <= done)
        v = ready[int(rng.integers(0, len(ready)))]
        order.append(v)
        done.add(v)
    NT = n + 3 * len(elig)
    rest = [v for v in range(NT) if v not in active]
    rng.shuffle(rest)
    # inactive optional nodes may sit anywhere
    for v in rest:
        order.insert(int(rng.integers(0, len(order) + 1)), v)
    return order, te, active


def test_random_dags_match_definition_and_invariants():
    """4000-style random cross-check: interval definition on the
    transformed graph; peak >= max_v(inputs + output); peak <= sum of active
    bytes; swap-free latency = sum cost + sum clone cost."""
    rng = np.random.default_rng(12345)
    checked = 0
    for _ in range(600):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        g = make(n, edges, size, outs, cost=cost, elig=elig, U=U, B=1e3, lam=0.5)
        perm, te, active = random_valid_perm(rng, n, edges, elig, U, dec)
        st, pk, lat, arg = g.eval(perm, dec if len(elig) else None)
        assert st == 0
        st2, pk2 = _defn.defn_eval(n, edges, size, outs, elig, U, dec, perm)
        assert pk == pk2
        R = len(elig)
        byt = {v: size[v] for v in range(n)}
        for r in range(R):
            byt[n + 3 * r] = size[elig[r]]
            byt[n + 3 * r + 1] = 0
            byt[n + 3 * r + 2] = size[elig[r]]
        pre = {}
        for u, v in te:
            pre.setdefault(v, set()).add(u)
        lower = max(byt[v] + sum(byt[u] for u in pre.get(v, ())) for v in active)
        assert lower <= pk <= sum(byt[v] for v in active)
        if not any(d == 2 for d in dec):
            exp = sum(cost) + sum(cost[elig[r]] for r in range(R) if dec[r] == 1)
            assert abs(lat - exp) <= 1e-12 * max(1.0, exp)
        else:
            # swaps can only add stall/transfer time on top of the compute sum
            base = sum(cost) + sum(cost[elig[r]] for r in range(R) if dec[r] == 1)
            assert lat >= base - 1e-12
        checked += 1
    assert checked == 600


def test_relabel_monotone_inactive_invariants():
    rng = np.random.default_rng(99)
    for _ in range(200):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng, 9)
        perm, te, active = random_valid_perm(rng, n, edges, elig, U, dec)
        g = make(n, edges, size, outs, cost=cost, elig=elig, U=U)
        st, pk, lat, _ = g.eval(perm, dec)
        # relabel the original ids with a random bijection
        pi = rng.permutation(n)
        e2 = [(int(pi[u]), int(pi[v])) for u, v in edges]
        s2 = [0] * n
        c2 = [0.0] * n
        for v in range(n):
            s2[pi[v]] = size[v]
            c2[pi[v]] = cost[v]
        g2 = make(n, e2, s2, [int(pi[o]) for o in outs], cost=c2,
                  elig=[int(pi[t]) for t in elig], U=[[int(pi[b]) for b in u] for u in U])
        perm2 = [int(pi[v]) if v < n else v for v in perm]
        st2, pk2, lat2, _ = g2.eval(perm2, dec)
        assert (st2, pk2) == (st, pk)
        assert abs(lat2 - lat) <= 1e-12 * max(1.0, lat)
        # growing one size never lowers the peak
        v = int(rng.integers(0, n))
        s3 = list(size)
        s3[v] += int(rng.integers(1, 1 << 20))
        g3 = make(n, edges, s3, outs, cost=cost, elig=elig, U=U)
        assert g3.eval(perm, dec)[1] >= pk
        # moving an inactive optional node changes nothing
        NT = n + 3 * len(elig)
        inactive = [v for v in range(n, NT) if v not in active]
        if inactive:
            p4 = [v for v in perm if v != inactive[0]]
            p4.insert(int(rng.integers(0, len(p4) + 1)), inactive[0])
            r4 = g.eval(p4, dec)
            assert r4[:2] == (st, pk) and abs(r4[2] - lat) <= 1e-12 * max(1.0, lat)


def test_violating_transposition_is_flagged():
    """Validity: swapping the two ends of any edge in a valid order
    sets bit1."""
    rng = np.random.default_rng(5)
    for _ in range(100):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng, 9)
        perm, te, active = random_valid_perm(rng, n, edges, elig, U, dec)
        if not te:
            continue
        g = make(n, edges, size, outs, cost=cost, elig=elig, U=U)
        u, v = sorted(te)[int(rng.integers(0, len(te)))]
        p = list(perm)
        iu, iv = p.index(u), p.index(v)
        p[iu], p[iv] = p[iv], p[iu]
        assert g.eval(p, dec)[0] == 2


# ------------------------------------------------------------ Eq. (1) pins --

def test_eq1_reproduces_fig2_cde():
    """Fig. 2(c)(d)(e) peaks 98 / 56 / 52 are Eq. (1) values
    (reading P16): 32 + 1056/16, 32 + 96/4, 32 + 8 + 96/8."""
    size = {}
    X = "X"
    size[X] = 32
    hot = [f"h{i}" for i in range(33)]
    for h in hot:
        size[h] = 32
    assert oracle.eq1_estimate(H=hot, S=hot, I=[X], size=size, n=16) == PAPER["fig2c.peak"]
    hot3 = hot[:3]
    assert oracle.eq1_estimate(H=hot3, S=hot3, I=[X], size=size, n=4) == PAPER["fig2d.peak"]
    size["s8"] = 8
    assert oracle.eq1_estimate(H=hot3, S=hot3, I=[X, "s8"], size=size, n=8) == PAPER["fig2e.peak"]
    assert oracle.eq1_m0(hot, size) == PAPER["fig2a.peak"]


# ------------------------------------------------------------------ Pareto --

def pareto_by_sort(peak, lat, status, ids):
    """Independent staircase: sort by (peak, lat, id), keep strict lat drops."""
    idx = [i for i in range(len(peak)) if status[i] == 0]
    idx.sort(key=lambda i: (peak[i], lat[i], ids[i]))
    out, best = [], math.inf
    for i in idx:
        if lat[i] < best:
            out.append(i)
            best = lat[i]
    return out


def test_pareto_front_matches_staircase_and_best_on_front():
    rng = np.random.default_rng(11)
    for trial in range(50):
        n = int(rng.integers(1, 400))
        peak = rng.integers(0, 40, n).astype(np.int64)
        lat = rng.integers(0, 40, n).astype(np.float64) / 4.0
        status = (rng.random(n) < 0.1).astype(np.uint8)
        ids = rng.permutation(10 * n)[:n].astype(np.int64)
        fr = oracle.pareto(peak, lat, status, ids)
        assert list(fr) == pareto_by_sort(peak, lat, status, ids)
        # every valid non-front point is dominated by, or duplicates, a front point
        fs = set(fr.tolist())
        for i in range(n):
            if status[i] or i in fs:
                continue
            assert any(peak[j] <= peak[i] and lat[j] <= lat[i] for j in fs)
        M = int(rng.integers(0, 40))
        b = oracle.best_under_memory(peak, lat, status, M, ids)
        if (status == 0).any():
            key = lambda i: (max(peak[i], M), lat[i], peak[i], ids[i])
            assert b == min((i for i in range(n) if not status[i]), key=key)
            assert b in fs
            L = float(rng.integers(0, 40)) / 4.0
            b2 = oracle.best_under_latency(peak, lat, status, L, ids)
            key2 = lambda i: (max(lat[i], L), peak[i], lat[i], ids[i])
            assert b2 == min((i for i in range(n) if not status[i]), key=key2)
            assert b2 in fs
        else:
            assert b == -1


def test_pareto_shard_merge_equals_single():
    """Merging per-shard fronts gives the single-shard front."""
    rng = np.random.default_rng(2)
    n = 3000
    peak = rng.integers(0, 200, n).astype(np.int64)
    lat = rng.integers(0, 200, n).astype(np.float64)
    status = (rng.random(n) < 0.05).astype(np.uint8)
    ids = np.arange(n, dtype=np.int64)
    full = oracle.pareto(peak, lat, status, ids)
    for P in (2, 3, 8):
        parts = np.array_split(np.arange(n), P)
        gathered = np.concatenate([p[oracle.pareto(peak[p], lat[p], status[p], ids[p])] for p in parts])
        m = oracle.pareto(peak[gathered], lat[gathered], status[gathered], ids[gathered])
        assert list(gathered[m]) == list(full)
