"""Seeded synthetic computation graphs -- INPUT GENERATION ONLY.

This module builds the DNN training graphs the bench and the tests feed to
both the CUDA path and the oracle.  It holds none of the evaluation
arithmetic (no lifetimes, no memory simulation, no latency model beyond the
per-op cost table the paper takes from its operator performance cache,
P:1780-1783).

Graph model (Table 1 / §2.1): every op has several inputs and one
output tensor; inputs, labels and weights are zero-cost nodes (P:392-393,
reading P3); auxiliary outputs (BN statistics, dropout masks) are folded into
the op's single output (reading P4).
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence

import numpy as np

# Synthetic cost model standing in for the paper's measured perf cache
# (P:1780-1783); RTX-3090-like constants so the graphs are "shaped like the
# paper".  cost(v) = launch + max(flops/F, bytes_rw/BW).
LAUNCH_S = 5e-6
F_TENSOR = 71e12     # tf32/bf16 tensor-core rate for matmul / conv
F_SIMT = 35.6e12     # everything else
BW = 936e9           # bytes/s

# swap link (PCIe-4 class): reading P7
SWAP_BPS = 25e9
SWAP_LAT = 1e-5


def op_cost(flops: float, bytes_rw: float, tensor: bool) -> float:
    return LAUNCH_S + max(flops / (F_TENSOR if tensor else F_SIMT), bytes_rw / BW)


@dataclass
class Workload:
    """One graph plus its eligible tensors; the unit both sides load."""
    name: str
    size: np.ndarray          # int64 [n] output bytes |v|
    cost: np.ndarray          # float64 [n] seconds
    is_output: np.ndarray     # uint8 [n]
    src: np.ndarray           # int32 [E]
    dst: np.ndarray           # int32 [E]
    names: List[str]
    kind: List[str]
    elig: np.ndarray = field(default_factory=lambda: np.zeros(0, np.int32))   # int32 [R]
    U: List[List[int]] = field(default_factory=list)                          # late users
    swap_Bps: float = SWAP_BPS
    swap_lat: float = SWAP_LAT
    loss_node: int = -1
    meta: Dict = field(default_factory=dict)
    # F-Trans variant regions (NEXT-4, reading F1): n_variants [F],
    # node_region [n] (-1: present in every variant), node_variant [n]
    regions: Optional[Dict] = None

    @property
    def F(self) -> int:
        return 0 if self.regions is None else len(self.regions["n_variants"])

    @property
    def n(self) -> int:
        return int(self.size.shape[0])

    @property
    def R(self) -> int:
        return int(self.elig.shape[0])

    @property
    def n_total(self) -> int:
        return self.n + 3 * self.R

    @property
    def n_edges(self) -> int:
        return int(self.src.shape[0])

    def U_arrays(self):
        ptr = np.zeros(self.R + 1, np.int64)
        for r, u in enumerate(self.U):
            ptr[r + 1] = ptr[r] + len(u)
        idx = (np.concatenate([np.asarray(u, np.int32) for u in self.U])
               if self.R else np.zeros(0, np.int32)).astype(np.int32)
        return ptr, idx

    def summary(self) -> Dict:
        return {"graph": self.name, "n_nodes": self.n, "n_edges": self.n_edges,
                "R": self.R, "n_total": self.n_total,
                "sum_bytes": int(self.size.sum()), "max_bytes": int(self.size.max(initial=0))}


class Builder:
    """Append-only DAG; node ids are a topological (natural) order."""

    def __init__(self, name: str):
        self.name = name
        self.names: List[str] = []
        self.kind: List[str] = []
        self.size: List[int] = []
        self.flops: List[float] = []
        self.tensor: List[bool] = []
        self.inputs: List[List[int]] = []
        self.outputs: set = set()
        self.tag: List[Optional[str]] = []      # free-form group tag (for F-Trans sets)
        self.splitdim: List[int] = []           # +1 split along the tag's positive dim, -1 reduce, 0 none
        self.loss_node = -1
        self.shared: Dict[str, set] = {}       # F-Trans group -> activations read unsliced
        self.cost_fix: List[Optional[float]] = []   # cost override (variant graphs), else the formula
        self.region: List[int] = []            # F-Trans variant region of the node, -1 = always present
        self.variant: List[int] = []           # variant of that region the node belongs to
        self.n_variants: List[int] = []        # per region

    def node(self, name: str, nbytes: int, inputs: Sequence[int] = (), flops: float = 0.0,
             kind: str = "op", tensor: bool = False, tag: Optional[str] = None,
             splitdim: int = 0, cost: Optional[float] = None, region: int = -1, variant: int = 0) -> int:
        v = len(self.names)
        ins = list(dict.fromkeys(int(u) for u in inputs))
        for u in ins:
            assert 0 <= u < v, (name, u, v)
        assert nbytes >= 0
        self.names.append(name)
        self.kind.append(kind)
        self.size.append(int(nbytes))
        self.flops.append(float(flops))
        self.tensor.append(bool(tensor))
        self.inputs.append(ins)
        self.tag.append(tag)
        self.splitdim.append(int(splitdim))
        self.cost_fix.append(cost)
        self.region.append(int(region))
        self.variant.append(int(variant))
        return v

    def cost_of(self, v: int) -> float:
        if self.cost_fix and self.cost_fix[v] is not None:
            return self.cost_fix[v]
        if self.kind[v] in ("input", "weight", "label"):
            return 0.0
        rw = self.size[v] + sum(self.size[u] for u in self.inputs[v])
        return op_cost(self.flops[v], rw, self.tensor[v])

    def finish(self, elig=None, U=None, meta=None) -> Workload:
        n = len(self.names)
        src, dst = [], []
        for v in range(n):
            for u in self.inputs[v]:
                src.append(u)
                dst.append(v)
        iso = np.zeros(n, np.uint8)
        for o in self.outputs:
            iso[o] = 1
        wl = Workload(
            name=self.name,
            size=np.asarray(self.size, np.int64),
            cost=np.asarray([self.cost_of(v) for v in range(n)], np.float64),
            is_output=iso,
            src=np.asarray(src, np.int32),
            dst=np.asarray(dst, np.int32),
            names=list(self.names),
            kind=list(self.kind),
            loss_node=self.loss_node,
            meta=dict(meta or {}),
        )
        if elig is not None:
            wl.elig = np.asarray(elig, np.int32)
            wl.U = [list(map(int, u)) for u in U]
        if self.n_variants:
            wl.regions = {"n_variants": np.asarray(self.n_variants, np.int32),
                          "node_region": np.asarray(self.region, np.int32),
                          "node_variant": np.asarray(self.variant, np.uint8)}
        return wl


# ---------------------------------------------------------------------------
# A tiny reverse-mode tracer that emits the backward ops of a training step.
# ---------------------------------------------------------------------------

def numel(shape) -> int:
    return int(np.prod(shape, dtype=np.int64))


class T:
    __slots__ = ("id", "shape", "grad", "param")

    def __init__(self, id_: int, shape, grad: bool, param: bool = False):
        self.id = id_
        self.shape = tuple(int(s) for s in shape)
        self.grad = grad
        self.param = param


class AG:
    """Forward ops record a backward closure; ``backward(loss)`` replays the
    tape in reverse, accumulating partial gradients pairwise (as autograd
    does) and emitting one update op per parameter as soon as its gradient is
    final.  Updated parameters and the loss are the graph outputs."""

    def __init__(self, b: Builder, dtype_bytes: int):
        self.b = b
        self.db = dtype_bytes
        self.tape = []           # (out T, inputs [T], bwd fn, tag)
        self.tag: Optional[str] = None   # current F-Trans group tag
        self.params: List[T] = []
        self.uses: Dict[int, int] = {}

    # -- leaves ---------------------------------------------------------------
    def input(self, name, shape, kind="input", dbytes=None) -> T:
        db = self.db if dbytes is None else dbytes
        return T(self.b.node(name, numel(shape) * db, (), kind=kind), shape, grad=False)

    def param(self, name, shape) -> T:
        t = T(self.b.node(name, numel(shape) * self.db, (), kind="weight"), shape, grad=True, param=True)
        self.params.append(t)
        return t

    # -- generic op -----------------------------------------------------------
    def op(self, name, inputs: Sequence[T], shape, flops, bwd=None, tensor=False, dbytes=None,
           splitdim=None) -> T:
        db = self.db if dbytes is None else dbytes
        sd = (1 if self.tag else 0) if splitdim is None else splitdim
        v = self.b.node(name, numel(shape) * db, [t.id for t in inputs], flops=flops,
                        tensor=tensor, tag=self.tag, splitdim=sd)
        need = any(t.grad for t in inputs)
        out = T(v, shape, grad=need)
        for t in inputs:
            self.uses[t.id] = self.uses.get(t.id, 0) + 1
        if need and bwd is not None:
            self.tape.append((out, list(inputs), bwd, self.tag))
        return out

    def _g(self, name, inputs: Sequence[T], like: T, flops, tensor=False, splitdim=None) -> T:
        """Emit a gradient op (no further backward)."""
        sd = (1 if self.tag else 0) if splitdim is None else splitdim
        v = self.b.node(name, numel(like.shape) * self.db, [t.id for t in inputs], flops=flops,
                        tensor=tensor, tag=self.tag, splitdim=sd)
        return T(v, like.shape, grad=False)

    # -- ops with backward rules ------------------------------------------------
    def matmul(self, name, x: T, w: T, out_shape, tensor=True) -> T:
        m = numel(out_shape) // out_shape[-1]
        k = x.shape[-1]
        nn = out_shape[-1]
        fl = 2.0 * m * k * nn

        def bwd(ag, dy, out, ins):
            x_, w_ = ins
            r = []
            if x_.grad:
                r.append((x_, ag._g(name + ".dX", [dy, w_], x_, fl, tensor=True)))
            if w_.grad:
                r.append((w_, ag._g(name + ".dW", [x_, dy], w_, fl, tensor=True,
                                    splitdim=(-1 if ag.tag else 0))))
            return r
        return self.op(name, [x, w], out_shape, fl, bwd, tensor=tensor)

    def bmm(self, name, a: T, bt: T, out_shape, fl, b_shared: bool = False) -> T:
        """Batched matmul.  With b_shared (inside an F-Trans group split along
        a dim the second operand lacks, e.g. K/V of a query-split attention),
        bt is read unsliced and its gradient is a reduce partial (P15)."""
        if b_shared and self.tag:
            self.b.shared.setdefault(self.tag, set()).add(bt.id)

        def bwd(ag, dy, out, ins):
            a_, b_ = ins
            r = []
            if a_.grad:
                r.append((a_, ag._g(name + ".dA", [dy, b_], a_, fl, tensor=True)))
            if b_.grad:
                r.append((b_, ag._g(name + ".dB", [dy, a_], b_, fl, tensor=True,
                                    splitdim=(-1 if (ag.tag and b_shared) else None))))
            return r
        return self.op(name, [a, bt], out_shape, fl, bwd, tensor=True)

    def conv(self, name, x: T, w: T, out_shape) -> T:
        # w shape (Cout, Cin, k, k); flops 2*N*Cout*Ho*Wo*Cin*k*k
        fl = 2.0 * numel(out_shape) * w.shape[1] * w.shape[2] * w.shape[3]

        def bwd(ag, dy, out, ins):
            x_, w_ = ins
            r = []
            if x_.grad:
                r.append((x_, ag._g(name + ".dX", [dy, w_], x_, fl, tensor=True)))
            if w_.grad:
                r.append((w_, ag._g(name + ".dW", [x_, dy], w_, fl, tensor=True,
                                    splitdim=(-1 if ag.tag else 0))))
            return r
        return self.op(name, [x, w], out_shape, fl, bwd, tensor=True)

    def unary(self, name, x: T, save: str = "x", flops_per=1.0, shape=None) -> T:
        """y = f(x); backward reads dy and x (save='x'), y (save='y') or nothing."""
        shape = x.shape if shape is None else shape

        def bwd(ag, dy, out, ins):
            x_, = ins
            reads = [dy] + ([x_] if save == "x" else [out] if save == "y" else [])
            return [(x_, ag._g(name + ".d", reads, x_, flops_per * numel(x_.shape)))]
        return self.op(name, [x], shape, flops_per * numel(shape), bwd)

    def add(self, name, a: T, b: T) -> T:
        """Residual add; gradient passes through (no op)."""
        def bwd(ag, dy, out, ins):
            return [(t, dy) for t in ins if t.grad]
        return self.op(name, [a, b], a.shape, numel(a.shape), bwd)

    def bias(self, name, x: T, bvec: T) -> T:
        def bwd(ag, dy, out, ins):
            x_, b_ = ins
            r = []
            if x_.grad:
                r.append((x_, dy))
            if b_.grad:
                r.append((b_, ag._g(name + ".db", [dy], b_, numel(dy.shape),
                                    splitdim=(-1 if ag.tag else 0))))
            return r
        return self.op(name, [x, bvec], x.shape, numel(x.shape), bwd)

    def binary(self, name, a: T, b: T, shape=None) -> T:
        """y = a * b (gating): da reads dy, b; db reads dy, a."""
        shape = a.shape if shape is None else shape

        def bwd(ag, dy, out, ins):
            a_, b_ = ins
            r = []
            if a_.grad:
                r.append((a_, ag._g(name + ".da", [dy, b_], a_, numel(a_.shape))))
            if b_.grad:
                r.append((b_, ag._g(name + ".db", [dy, a_], b_, numel(b_.shape))))
            return r
        return self.op(name, [a, b], shape, numel(shape), bwd)

    def const_op(self, name, x: T, c: T, save="y") -> T:
        """y = f(x, c) with a non-differentiable constant input (mask)."""
        def bwd(ag, dy, out, ins):
            x_, c_ = ins
            reads = [dy] + ([out] if save == "y" else [c_])
            return [(x_, ag._g(name + ".d", reads, x_, numel(x_.shape)))]
        return self.op(name, [x, c], x.shape, numel(x.shape), bwd)

    def norm(self, name, x: T, gamma: T, beta: T) -> T:
        """Fused LayerNorm-like op (stats folded into the output, reading P4)."""
        def bwd(ag, dy, out, ins):
            x_, g_, b_ = ins
            r = [(x_, ag._g(name + ".dX", [dy, x_, g_], x_, 8.0 * numel(x_.shape)))]
            sd = -1 if ag.tag else 0
            r.append((g_, ag._g(name + ".dg", [dy, x_], g_, 4.0 * numel(x_.shape), splitdim=sd)))
            r.append((b_, ag._g(name + ".db", [dy], b_, numel(x_.shape), splitdim=sd)))
            return r
        return self.op(name, [x, gamma, beta], x.shape, 8.0 * numel(x.shape), bwd)

    def loss(self, name, logits: T, labels: T) -> T:
        def bwd(ag, dy, out, ins):
            lg, lb = ins
            return [(lg, ag._g(name + ".d", [dy, lg, lb], lg, 4.0 * numel(lg.shape)))]
        t = self.op(name, [logits, labels], (1,), 4.0 * numel(logits.shape), bwd, dbytes=4)
        self.b.loss_node = t.id
        return t

    # -- backward -----------------------------------------------------------
    def backward(self, loss: T, update: bool = True):
        b = self.b
        b.outputs.add(loss.id)
        self.tag = None
        grad: Dict[int, T] = {}
        # d(loss)/d(loss): a tiny seed op
        grad[loss.id] = T(b.node("loss.grad_seed", 4, [loss.id], flops=1.0), (1,), False)
        remaining = {p.id: self.uses.get(p.id, 0) for p in self.params}
        pmap = {p.id: p for p in self.params}

        def accumulate(t: T, gt: T):
            old = grad.get(t.id)
            if old is None:
                grad[t.id] = gt
            else:
                self.tag = None
                grad[t.id] = self._g(f"acc.{b.names[t.id]}", [old, gt], t, numel(t.shape), splitdim=0)

        for out, ins, fn, tag in reversed(self.tape):
            dy = grad.pop(out.id, None)
            if dy is None:
                continue
            self.tag = tag
            parts = fn(self, dy, out, ins)
            self.tag = None
            for t, gt in parts:
                accumulate(t, gt)
            for t in ins:
                if t.id in remaining:
                    remaining[t.id] -= 1
                    if remaining[t.id] == 0 and update and t.id in grad:
                        p = pmap[t.id]
                        g = grad.pop(t.id)
                        u = b.node(f"update.{b.names[p.id]}", numel(p.shape) * self.db, [p.id, g.id],
                                   flops=4.0 * numel(p.shape))
                        b.outputs.add(u)
