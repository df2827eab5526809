"""Eligible-tensor selection (hot-spot filter) -- INPUT
GENERATION ONLY.

The paper applies the re-materialisation and swapping rules only to
sub-graphs containing memory hot-spots.  This module must not simulate
memory (it holds none of the method's arithmetic), so it uses the structural
proxy DESIGN.md reading R-hot describes: in a training graph the hot-spot set
H at the natural order's peak is the set of forward activations saved for the
backward pass, i.e. tensors whose readers straddle the loss.  We keep compute
nodes with >= 1 input, not graph outputs, with >= 2 readers spanning >= 8
steps of the natural order and a reader after the loss, and take the largest
R_max by bytes (ties: smaller id).  U_t = the readers after t's first reader
in the natural order (reading P6).  tests/test_inputs.py checks with the
oracle that the chosen tensors really are in H.
"""
from __future__ import annotations

import numpy as np

from .graph import Workload


def select(wl: Workload, R_max: int, min_span: int = 8) -> Workload:
    n = wl.n
    cons = [[] for _ in range(n)]
    has_in = np.zeros(n, bool)
    for u, v in zip(wl.src.tolist(), wl.dst.tolist()):
        cons[u].append(v)
        has_in[v] = True
    loss = wl.loss_node if wl.loss_node >= 0 else n // 2
    # F-Trans variant graphs (NEXT-4): the Fig. 8 rules stay on the nodes that
    # exist in every variant -- t, its inputs and its late users ungated
    gated = (wl.regions["node_region"] >= 0) if wl.regions is not None else np.zeros(n, bool)
    if gated.any():
        pre_gated = np.zeros(n, bool)
        for u, v in zip(wl.src.tolist(), wl.dst.tolist()):
            if gated[u]:
                pre_gated[v] = True
        cons = [[v for v in cs if not gated[v]] for cs in cons]
    cand = []
    for t in range(n):
        c = sorted(set(cons[t]))
        if wl.kind[t] != "op" or wl.is_output[t] or not has_in[t] or len(c) < 2:
            continue
        if gated[t] or (gated.any() and pre_gated[t]):
            continue
        if c[-1] - c[0] < min_span or c[-1] <= loss:
            continue
        cand.append(t)
    cand.sort(key=lambda t: (-int(wl.size[t]), t))
    chosen = sorted(cand[:R_max])
    wl.elig = np.asarray(chosen, np.int32)
    wl.U = [sorted(set(cons[t]))[1:] for t in chosen]
    return wl
