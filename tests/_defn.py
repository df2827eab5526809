"""Independent definitional evaluators used to PIN the oracle (tests only).

These are written from the paper's formulas directly, in a different style
from the C oracle (sets and interval sums instead of event/free lists), so a
plausible slip in either shows up as a mismatch:

* ``interval_peak``: M_i = sum_{u : S_u < i <= F_u} |u| (P:409-424 with the
  1-based S_j = j-1 and the corrected strict inequality, reading P1), written
  as an O(n^2) double loop over steps and tensors.
* ``literal_peak``: the same with the literal, garbled S_j <= i <= F_j
   -- used to show that the text's 1056 needs reading P1.
* ``all_topo_orders``: brute-force enumeration of every topological order.
* ``defn_latency``: the modelled latency as the longest path of an explicit
  event DAG (compute / D2H / H2D queue chains + data edges, reading P7) --
  a different formulation from the oracle's three-queue recurrence.
"""
from __future__ import annotations

import itertools


def succ_map(n, edges):
    s = {v: set() for v in range(n)}
    for u, v in edges:
        s[u].add(v)
    return s


def intervals(order, edges, outputs):
    """1-based S/F per paper: S_j = j-1, F_j = max_{v_k in suc(v_j)} k;
    outputs live to n; no successors -> F_j = j (own step)."""
    n = len(order)
    step = {v: i + 1 for i, v in enumerate(order)}  # 1-based timestamps
    suc = {}
    for u, v in edges:
        suc.setdefault(u, set()).add(v)
    S, F = {}, {}
    for v in order:
        S[v] = step[v] - 1
        if v in outputs:
            F[v] = n
        elif suc.get(v):
            F[v] = max(step[w] for w in suc[v])
        else:
            F[v] = step[v]
    return S, F


def interval_peak(order, edges, size, outputs):
    """max_i sum |u| over u with S_u < i <= F_u  (reading P1)."""
    S, F = intervals(order, edges, outputs)
    n = len(order)
    best, arg = None, None
    for i in range(1, n + 1):
        m = sum(size[u] for u in order if S[u] < i <= F[u])
        if best is None or m > best:
            best, arg = m, i - 1
    return best, arg


def literal_peak(order, edges, size, outputs):
    """Literal P:416 form S_j <= i <= F_j (garbled by one step)."""
    S, F = intervals(order, edges, outputs)
    n = len(order)
    return max(sum(size[u] for u in order if S[u] <= i <= F[u]) for i in range(1, n + 1))


def all_topo_orders(n, edges):
    pre = {v: set() for v in range(n)}
    for u, v in edges:
        pre[v].add(u)
    out = []

    def rec(done, order):
        if len(order) == n:
            out.append(list(order))
            return
        for v in range(n):
            if v not in done and pre[v] <= done:
                done.add(v)
                order.append(v)
                rec(done, order)
                order.pop()
                done.remove(v)

    rec(set(), [])
    return out


def is_topo(order, edges):
    p = {v: i for i, v in enumerate(order)}
    return all(p[u] < p[v] for u, v in edges)


def transformed(n, edges, elig, U, dec):
    """Fig. 8 rule semantics on an explicit edge set (reading P6); returns
    (active node list, edge set, bytes map builder info)."""
    edges = set(map(tuple, edges))
    R = len(elig)
    out = set()
    moved = {}
    for r in range(R):
        for b in U[r]:
            moved[(elig[r], b)] = r
    for (u, v) in edges:
        r = moved.get((u, v))
        if r is not None and dec[r] == 1:
            out.add((n + 3 * r, v))
        elif r is not None and dec[r] == 2:
            out.add((n + 3 * r + 2, v))
        else:
            out.add((u, v))
    for r in range(R):
        t = elig[r]
        if dec[r] == 1:
            for (u, v) in edges:
                if v == t:
                    out.add((u, n + 3 * r))
        elif dec[r] == 2:
            out.add((t, n + 3 * r + 1))
            out.add((n + 3 * r + 1, n + 3 * r + 2))
    active = set(range(n))
    for r in range(R):
        if dec[r] == 1:
            active.add(n + 3 * r)
        if dec[r] == 2:
            active |= {n + 3 * r + 1, n + 3 * r + 2}
    return active, out


def defn_eval(n, edges, size, outputs, elig, U, dec, perm):
    """Interval-sum peak on the transformed graph (no latency)."""
    active, te = transformed(n, edges, elig, U, dec)
    pos = {v: i for i, v in enumerate(perm)}
    if any(pos[u] >= pos[v] for u, v in te):
        return 2, -1
    order = [v for v in perm if v in active]
    sz = {}
    for v in order:
        if v < n:
            sz[v] = size[v]
        else:
            r, k = divmod(v - n, 3)
            sz[v] = 0 if k == 1 else size[elig[r]]
    pk, _ = interval_peak(order, te, sz, set(outputs))
    return 0, pk


# ---- latency as the longest path of an explicit event DAG (reading P7) ----

def event_dag(n, edges, cost, size, elig, U, dec, perm, B, lam):
    """The schedule's execution as a DAG of timed events (P:1784-1789,
    P:1796-1799; reading P7), built from scratch and independent of the
    oracle's queue recurrence:

    * one event per active node, weighted by its duration: a compute op v
      takes cost(v), a clone A' takes cost(t_r) (reading P9), a Store or Load
      of t_r takes lam + |t_r| / B;
    * resource edges: the compute ops (with clones), the Stores and the Loads
      each run on their own in-order queue, so consecutive events of one
      queue in step order are chained;
    * data edges: every edge (u, v) of the transformed graph (Fig. 8) -- in
      particular t_r -> Store_r -> Load_r -> each late user.

    -> (weights {node: duration}, arcs set of (u, v))."""
    active, te = transformed(n, edges, elig, U, list(dec))
    order = [v for v in perm if v in active]

    def kind(v):                     # 'c' compute, 's' Store, 'l' Load
        if v < n:
            return "c"
        return "csl"[(v - n) % 3]

    w = {}
    for v in order:
        if v < n:
            w[v] = cost[v]
        else:
            r, k = divmod(v - n, 3)
            w[v] = cost[elig[r]] if k == 0 else lam + size[elig[r]] / B
    arcs = set(te)
    for q in "csl":
        seq = [v for v in order if kind(v) == q]
        arcs |= set(zip(seq, seq[1:]))
    return w, arcs


def longest_path_latency(w, arcs):
    """Makespan of the event DAG: finish(v) = w(v) + max(finish(p)) over the
    predecessors p of v (0 without any), latency = max finish.  Memoised
    recursion over the predecessor sets -- no step order is used."""
    import sys
    pre = {v: [] for v in w}
    for u, v in arcs:
        pre[v].append(u)
    memo = {}
    sys.setrecursionlimit(max(10000, 4 * len(w) + 100))

    def fin(v):
        if v not in memo:
            memo[v] = w[v] + max((fin(p) for p in pre[v]), default=0.0)
        return memo[v]

    return max((fin(v) for v in w), default=0.0)


def defn_latency(n, edges, cost, size, elig, U, dec, perm, B, lam):
    """Latency of a valid schedule by the event-DAG longest path."""
    return longest_path_latency(*event_dag(n, edges, cost, size, elig, U, dec, perm, B, lam))


# ---- NEXT-3: hot-spots, dominators, heat / score (written from the text) ----

def defn_hotspots(n, edges, size, outputs, elig, U, dec, perm):
    """H = union of A_i over the steps i with M_i = M_peak, A_i = the tensors
    with S_u < i <= F_u (reading P1), on the transformed graph;
    then over the original nodes: a live clone or Load of t_r stands for t_r,
    a Store does not count (reading H1).  -> set of original nodes, or None
    if the schedule violates a dependency."""
    active, te = transformed(n, edges, elig, U, dec)
    pos = {v: i for i, v in enumerate(perm)}
    if any(pos[u] >= pos[v] for u, v in te):
        return None
    order = [v for v in perm if v in active]
    sz = {}
    for v in order:
        if v < n:
            sz[v] = size[v]
        else:
            r, k = divmod(v - n, 3)
            sz[v] = 0 if k == 1 else size[elig[r]]
    S, F = intervals(order, te, set(outputs))
    curve = [sum(sz[u] for u in order if S[u] < i <= F[u]) for i in range(1, len(order) + 1)]
    peak = max(curve)
    Hs = set()
    for i in range(1, len(order) + 1):
        if curve[i - 1] == peak:
            Hs |= {u for u in order if S[u] < i <= F[u]}
    H = {v for v in Hs if v < n}
    for v in Hs:
        if v >= n:
            r, k = divmod(v - n, 3)
            if k != 1:
                H.add(elig[r])
    return H


def brute_dominators(n, edges):
    """dom[u] = set of nodes v that u dominates: u == v, or v cannot be reached
    from any source (node without predecessors) once u is removed."""
    pre = {v: set() for v in range(n)}
    suc = {v: set() for v in range(n)}
    for u, v in edges:
        pre[v].add(u)
        suc[u].add(v)
    sources = [v for v in range(n) if not pre[v]]
    dom = {}
    for u in range(n):
        seen = set()
        stack = [s for s in sources if s != u]
        while stack:
            x = stack.pop()
            if x in seen:
                continue
            seen.add(x)
            stack.extend(y for y in suc[x] if y != u)
        dom[u] = {v for v in range(n) if v == u or v not in seen}
    return dom


def brute_idom(n, edges):
    dom = brute_dominators(n, edges)
    idom = []
    for v in range(n):
        strict = [u for u in range(n) if u != v and v in dom[u]]
        # the strict dominator dominated by every other strict dominator
        best = [u for u in strict if all(u in dom[w] for w in strict)]
        idom.append(best[0] if best else -1)
    return idom


def defn_heat_score(n, edges, size, H, nsplit):
    """Eq. 3 / Eq. 4 literally: heat(v) = sum |w| over w in H and T.des(v);
    score(v) = (1 - 1/nsplit) heat(v) - sum |u| over the inputs of T.des(v)
    (nodes outside it with an edge into it) that are not in H."""
    dom = brute_dominators(n, edges)
    heat, score = [], []
    for v in range(n):
        des = dom[v]
        h = sum(size[w] for w in des if w in H)
        inps = {u for (u, w) in edges if w in des and u not in des}
        inp = sum(size[u] for u in inps if u not in H)
        heat.append(h)
        score.append((1.0 - 1.0 / nsplit) * float(h) - float(inp))
    return heat, score
