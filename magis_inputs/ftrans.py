"""F-Trans materialiser (§4.2, Fig. 5) -- INPUT
GENERATION ONLY.

Given a built graph whose ops carry an F-Trans group tag (the sub-graph S) and
a split-dim sign per op (+1: the op's output has the split dim; -1: a reduce
axis, only on outputs of S -- reading P15), produce the graph after the
F-Trans f = (S, D, n):

* S is copied n times ("split into n parts"; each contiguous run of S in the
  natural order is emitted part after part, so the parts run in sequence);
* every input of S with the split dim gets one Slice node per part
  (|u|/n bytes); shared inputs (weights, explicitly shared activations such
  as K/V of a query-split attention) are read unsliced;
* every output of S gets one merge node: Concat for a positive dim, an n-ary
  Add for a reduce dim (Fig. 5);
* part bytes are |v|/n for positive-dim ops (n divides the dim length, the
  Mutating Rule P:1315-1317), full size for reduce partials.

Part costs use the same cost formula on the smaller shapes, so the launch
term makes fission cost latency.

``apply`` splits every group with one n; ``apply_choice`` takes an n per
group (n = 1 leaves it whole); ``apply_variants`` builds the *variant
graph* of NEXT-4 (reading F1): every group becomes a region holding all its
variants side by side (variant 0 = the unsplit ops, variant j = the split by
ns[j-1]), each node labelled with its (region, variant); a consumer outside a
region reads every variant's version of a region output, and exactly one
variant is present in a candidate, so the graph of a candidate equals
``apply_choice`` with that candidate's factors (names match; tested).
"""
from __future__ import annotations

from typing import Callable, Dict, List, Sequence, Set

from .graph import Builder, op_cost


def _logical_cost(b: Builder, flops: float, size: int, in_sizes: Sequence[int], kind: str, tensor: bool) -> float:
    if kind in ("input", "weight", "label"):
        return 0.0
    return op_cost(flops, size + sum(in_sizes), tensor)


def _materialize(b: Builder, n_of: Callable[[str], int], shared: Dict[str, Set[int]] | None,
                 name: str | None) -> Builder:
    shared = b.shared if shared is None else shared
    N = len(b.names)
    tag = b.tag
    out = Builder(name or b.name)
    out.outputs = set()
    cons = [[] for _ in range(N)]
    for v in range(N):
        for u in b.inputs[v]:
            cons[u].append(v)

    newid = [-1] * N                 # id of the node (or its merge) seen from outside S
    part = {}                        # (v, k) -> id of part copy
    slices = {}                      # (u, k, tag) -> id of slice node
    fmap = {}                        # bookkeeping for tests: v -> [part ids]
    prov = {}                        # node id -> provenance key (tests map graphs by it)

    def is_in(v, t):
        return tag[v] is not None and tag[v] == t

    v = 0
    while v < N:
        t = tag[v]
        n = n_of(t) if t is not None else 1
        if t is None or n <= 1:
            ins = [newid[u] for u in b.inputs[v]]
            assert all(i >= 0 for i in ins)
            nv = out.node(b.names[v], b.size[v], ins, b.flops[v], b.kind[v], b.tensor[v])
            newid[v] = nv
            prov[nv] = ("op", v)
            if v in b.outputs:
                out.outputs.add(nv)
            if v == b.loss_node:
                out.loss_node = nv
            v += 1
            continue
        # maximal contiguous run of the same group
        run = [v]
        w = v + 1
        while w < N and tag[w] == t:
            run.append(w)
            w += 1
        sh = shared.get(t, set())
        for k in range(n):
            for x in run:
                ins = []
                for u in b.inputs[x]:
                    if is_in(u, t):
                        ins.append(part[(u, k)])
                    elif b.kind[u] == "weight" or u in sh:
                        ins.append(newid[u])
                    else:
                        key = (u, k, t)
                        if key not in slices:
                            assert b.size[u] % n == 0, ("slice not divisible", b.names[u], n)
                            su = b.size[u] // n
                            slices[key] = out.node(f"{b.names[u]}.slice{k}", su, [newid[u]],
                                                   flops=float(su), kind="op")
                            prov[slices[key]] = ("slice", u, k, t)
                        ins.append(slices[key])
                sd = b.splitdim[x]
                if sd > 0:
                    assert b.size[x] % n == 0, ("part not divisible", b.names[x], n)
                    sz = b.size[x] // n
                else:
                    sz = b.size[x]
                pid = out.node(f"{b.names[x]}.p{k}", sz, ins, b.flops[x] / n, b.kind[x], b.tensor[x])
                prov[pid] = ("part", x, k)
                part[(x, k)] = pid
                fmap.setdefault(x, []).append(pid)
        for x in run:
            outside = any(not is_in(c, t) for c in cons[x]) or x in b.outputs
            if not outside:
                continue
            parts = [part[(x, k)] for k in range(n)]
            if b.splitdim[x] > 0:
                m = out.node(f"{b.names[x]}.concat", b.size[x], parts, flops=float(b.size[x]))
            else:
                m = out.node(f"{b.names[x]}.addmerge", b.size[x], parts, flops=float(n * b.size[x]))
            prov[m] = ("merge", x)
            newid[x] = m
            if x in b.outputs:
                out.outputs.add(m)
        v = w
    out.fission_map = fmap          # type: ignore[attr-defined]
    out.fission_src = b             # type: ignore[attr-defined]
    out.prov = prov                 # type: ignore[attr-defined]
    return out


def apply(b: Builder, n: int, shared: Dict[str, Set[int]] | None = None,
          name: str | None = None) -> Builder:
    """Return a new Builder with every tagged group split into n parts."""
    if n <= 1:
        return b
    out = _materialize(b, lambda t: n, shared, name)
    out.fission_n = n               # type: ignore[attr-defined]
    return out


def groups(b: Builder) -> List[str]:
    """F-Trans group tags in order of first appearance."""
    seen: Dict[str, None] = {}
    for t in b.tag:
        if t is not None and t not in seen:
            seen[t] = None
    return list(seen)


def apply_choice(b: Builder, nmap: Dict[str, int], shared: Dict[str, Set[int]] | None = None,
                 name: str | None = None) -> Builder:
    """F-Trans with one factor per group (nmap[tag]; missing or 1 = unsplit)."""
    return _materialize(b, lambda t: int(nmap.get(t, 1)), shared, name)


def apply_variants(b: Builder, ns: Sequence[int] = (2, 4), shared: Dict[str, Set[int]] | None = None,
                   name: str | None = None) -> Builder:
    """The variant graph (NEXT-4, reading F1): region i = group i (every run
    of its tag, forward and backward, so parts of the backward read the parts
    of the forward), variants 0 (unsplit) and j = 1..len(ns) (split by
    ns[j-1]).  Node names inside variant j carry the suffix "@n<ns[j-1]>";
    costs are those of the materialised graph (logical inputs), so that a
    consumer reading every variant's version of an input is not charged for
    all of them."""
    shared = b.shared if shared is None else shared
    N = len(b.names)
    tag = b.tag
    tags = groups(b)
    reg = {t: i for i, t in enumerate(tags)}
    V = 1 + len(ns)
    out = Builder(name or b.name + ".variants")
    out.outputs = set()
    out.n_variants = [V] * len(tags)
    cons = [[] for _ in range(N)]
    for v in range(N):
        for u in b.inputs[v]:
            cons[u].append(v)
    alts: List[List[int]] = [[] for _ in range(N)]   # ids standing for v outside its region (one per variant)
    size_seen = b.size

    def is_in(v, t):
        return tag[v] is not None and tag[v] == t

    v = 0
    prov = {}                         # node id -> provenance key, as _materialize's
    id0 = {}                          # variant-0 copy of a region node
    part = {}                         # (x, j, k) -> part id
    slices = {}                       # (u, j, k, t) -> slice id
    while v < N:
        t = tag[v]
        if t is None:
            ins = [i for u in b.inputs[v] for i in alts[u]]
            c = b.cost_of(v)
            nv = out.node(b.names[v], b.size[v], ins, b.flops[v], b.kind[v], b.tensor[v], cost=c)
            prov[nv] = ("op", v)
            alts[v] = [nv]
            if v in b.outputs:
                out.outputs.add(nv)
            if v == b.loss_node:
                out.loss_node = nv
            v += 1
            continue
        run = [v]
        w = v + 1
        while w < N and tag[w] == t:
            run.append(w)
            w += 1
        ri = reg[t]
        sh = shared.get(t, set())
        # variant 0: the unsplit ops
        for x in run:
            ins = []
            for u in b.inputs[x]:
                if is_in(u, t):
                    ins.append(id0[u])
                else:
                    assert len(alts[u]) == 1, ("adjacent F-Trans regions", b.names[u], b.names[x])
                    ins.append(alts[u][0])
            id0[x] = out.node(b.names[x], b.size[x], ins, b.flops[x], b.kind[x], b.tensor[x],
                              cost=b.cost_of(x), region=ri, variant=0)
            prov[id0[x]] = ("op", x)
        # variant j: split by n
        merges = {}
        for j, n in enumerate(ns, start=1):
            sfx = f"@n{n}"
            for k in range(n):
                for x in run:
                    ins, in_sizes = [], []
                    for u in b.inputs[x]:
                        if is_in(u, t):
                            p = part[(u, j, k)]
                            ins.append(p)
                            in_sizes.append(out.size[p])
                        elif b.kind[u] == "weight" or u in sh:
                            assert len(alts[u]) == 1, ("adjacent F-Trans regions", b.names[u], b.names[x])
                            ins.append(alts[u][0])
                            in_sizes.append(b.size[u])
                        else:
                            assert len(alts[u]) == 1, ("adjacent F-Trans regions", b.names[u], b.names[x])
                            key = (u, j, k, t)
                            if key not in slices:
                                assert b.size[u] % n == 0, ("slice not divisible", b.names[u], n)
                                su = b.size[u] // n
                                slices[key] = out.node(f"{b.names[u]}.slice{k}{sfx}", su, [alts[u][0]],
                                                       flops=float(su), kind="op",
                                                       cost=_logical_cost(b, float(su), su, [b.size[u]], "op", False),
                                                       region=ri, variant=j)
                            prov[slices[key]] = ("slice", u, k, t)
                            ins.append(slices[key])
                            in_sizes.append(b.size[u] // n)
                    sz = b.size[x] // n if b.splitdim[x] > 0 else b.size[x]
                    if b.splitdim[x] > 0:
                        assert b.size[x] % n == 0, ("part not divisible", b.names[x], n)
                    c = _logical_cost(b, b.flops[x] / n, sz, in_sizes, b.kind[x], b.tensor[x])
                    part[(x, j, k)] = out.node(f"{b.names[x]}.p{k}{sfx}", sz, ins, b.flops[x] / n, b.kind[x],
                                               b.tensor[x], cost=c, region=ri, variant=j)
                    prov[part[(x, j, k)]] = ("part", x, k)
            for x in run:
                outside = any(not is_in(c2, t) for c2 in cons[x]) or x in b.outputs
                if not outside:
                    continue
                parts = [part[(x, j, k)] for k in range(n)]
                psz = [out.size[p] for p in parts]
                if b.splitdim[x] > 0:
                    m = out.node(f"{b.names[x]}.concat{sfx}", b.size[x], parts, flops=float(b.size[x]),
                                 cost=_logical_cost(b, float(b.size[x]), b.size[x], psz, "op", False),
                                 region=ri, variant=j)
                else:
                    m = out.node(f"{b.names[x]}.addmerge{sfx}", b.size[x], parts, flops=float(n * b.size[x]),
                                 cost=_logical_cost(b, float(n * b.size[x]), b.size[x], psz, "op", False),
                                 region=ri, variant=j)
                prov[m] = ("merge", x)
                merges.setdefault(x, []).append(m)
        for x in run:
            outside = any(not is_in(c2, t) for c2 in cons[x]) or x in b.outputs
            if outside:
                alts[x] = [id0[x]] + merges.get(x, [])
                if x in b.outputs:
                    out.outputs.update(alts[x])
            else:
                alts[x] = [id0[x]]
        v = w
    del size_seen
    out.prov = prov                   # type: ignore[attr-defined]
    out.variant_ns = [1] + list(ns)   # type: ignore[attr-defined]
    out.variant_tags = tags           # type: ignore[attr-defined]
    return out
