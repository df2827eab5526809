"""Per-op 64-bit labels for GraphHash -- INPUT GENERATION ONLY.

``hash(v)`` in Alg. 3 line 5 hashes the node itself.  For the
WL-style duplicate test two ops must get the same label iff
they are the same computation: same op type and attributes, same output
shape -- but not the same layer index (the graph structure distinguishes
layers).  The generator's op signature is the node name with layer indices
stripped ("l3.5.bn2.norm.dx" -> "l#.#.bn2.norm.dx"; "h18.proj.dX.p3" ->
"h#.proj.dX.p3": F-Trans part / slice indices are attributes and stay),
together with the node kind, output bytes and cost.  The label is the first
8 bytes of BLAKE2b of that signature (reading G3 in DESIGN.md): a fixed,
seed-free function of the op, so isomorphic sub-graphs hash alike.
"""
from __future__ import annotations

import hashlib
import re

import numpy as np

_LAYER = re.compile(r"^([a-z]+)\d+$")


def op_signature(name: str, kind: str, size: int, cost: float) -> str:
    parts = name.split(".")
    out = []
    for i, p in enumerate(parts):
        if p.isdigit():
            out.append("#")
        elif i == 0 or (i == 1 and parts[0] in ("acc", "update")):
            m = _LAYER.match(p)
            out.append(m.group(1) + "#" if m else p)
        else:
            out.append(p)
    return f"{kind}|{'.'.join(out)}|{int(size)}|{float(cost)!r}"


def label_of(sig: str) -> int:
    return int.from_bytes(hashlib.blake2b(sig.encode(), digest_size=8).digest(), "little")


def node_labels(wl) -> np.ndarray:
    """uint64 [n] labels of a Workload's ops."""
    return np.array([label_of(op_signature(nm, k, s, c))
                     for nm, k, s, c in zip(wl.names, wl.kind, wl.size.tolist(), wl.cost.tolist())],
                    dtype=np.uint64)
