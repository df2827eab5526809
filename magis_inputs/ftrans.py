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
"""
from __future__ import annotations

from typing import Dict, Set

from .graph import Builder


def apply(b: Builder, n: int, shared: Dict[str, Set[int]] | None = None,
          name: str | None = None) -> Builder:
    """Return a new Builder with every tagged group split into n parts."""
    if n <= 1:
        return b
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

    def is_in(v, t):
        return tag[v] is not None and tag[v] == t

    v = 0
    while v < N:
        t = tag[v]
        if t is None:
            ins = [newid[u] for u in b.inputs[v]]
            assert all(i >= 0 for i in ins)
            nv = out.node(b.names[v], b.size[v], ins, b.flops[v], b.kind[v], b.tensor[v])
            newid[v] = nv
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
                        ins.append(slices[key])
                sd = b.splitdim[x]
                if sd > 0:
                    assert b.size[x] % n == 0, ("part not divisible", b.names[x], n)
                    sz = b.size[x] // n
                else:
                    sz = b.size[x]
                pid = out.node(f"{b.names[x]}.p{k}", sz, ins, b.flops[x] / n, b.kind[x], b.tensor[x])
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
            newid[x] = m
            if x in b.outputs:
                out.outputs.add(m)
        v = w
    out.fission_map = fmap          # type: ignore[attr-defined]
    out.fission_n = n               # type: ignore[attr-defined]
    out.fission_src = b             # type: ignore[attr-defined]
    return out
