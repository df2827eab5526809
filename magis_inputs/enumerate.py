"""Every topological order of a small DAG -- INPUT GENERATION ONLY.

C1 (BASELINE configs[0]) scores the full set of schedules of a 10-op
diamond: a schedule is a topological order of G, and the
brute-force minimum peak is the minimum over all of them.  This module only
enumerates the orders (iterative depth-first search over the ready sets,
lexicographic by node id); it holds none of the evaluation arithmetic.
"""
from __future__ import annotations

import numpy as np


def topo_orders(n: int, src, dst) -> np.ndarray:
    """-> int32 [count, n]: every topological order of the DAG (n <= 20)."""
    pre = [0] * n
    for u, v in zip(np.asarray(src).tolist(), np.asarray(dst).tolist()):
        pre[v] |= 1 << u
    out = []
    order = []
    # stack of (done mask, candidates still to try at this depth)
    full = (1 << n) - 1

    def ready(done):
        return [v for v in range(n) if not (done >> v) & 1 and (pre[v] & ~done) == 0]

    stack = [(0, ready(0))]
    while stack:
        done, cand = stack[-1]
        if done == full:
            out.append(list(order))
            stack.pop()
            if order:
                order.pop()
            continue
        if not cand:
            stack.pop()
            if order:
                order.pop()
            continue
        v = cand.pop(0)
        order.append(v)
        nd = done | (1 << v)
        stack.append((nd, ready(nd)))
    return np.asarray(out, np.int32).reshape(-1, n)
