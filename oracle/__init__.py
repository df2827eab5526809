"""MAGIS schedule-evaluation ORACLE -- TEST INFRASTRUCTURE ONLY.

A plain, slow, single-threaded CPU implementation of what the B200 path
computes (§2.1, §5.2, §6.2, Alg. 3
BetterThan P:1689-1692).  It shares no code with the CUDA path and must only
be imported by ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs.

Pins (tests/test_oracle_*.py): Fig. 2(a) = 1056, Fig. 2(b) = 96
(P:469-476), hand-computed toys T1/T2/T3 (T3: two swaps
contending on both copy queues), closed forms, brute-force enumeration of all
topological orders against an independently written interval formula, the
swap latency against an independent event-DAG longest path (reading P7,
P:1784-1789), invariants, Eq. (1) = 98/56/52.

Parity status per function:
  * peak / status / argmax ....... pinned (paper numbers + brute force)
  * swap-free latency ............ pinned (closed form P:406-408)
  * swap latency (queues) ........ parity unpinned by the paper (reading P7);
                                   pinned only by hand-computed toys T1
  * pareto / best ................ pinned (definition, brute-force dominance)
  * GraphHash (Alg. 3 l.3-6) ..... pinned (SplitMix64 published outputs for
                                   mix64; WL unfolding-tree equivalence by
                                   brute force; relabelling / schedule
                                   invariance; materialised Fig. 8 graphs)
  * hash filter (Alg. 3 l.10-12) . pinned (O(K^2) first-occurrence definition)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "magis_oracle.c")
_LIB = os.path.join(_HERE, "libmagis_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (plain -O2, no vectorisation tricks)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    lib = ctypes.CDLL(_LIB)
    P = ctypes.c_void_p
    lib.orc_graph_new.restype = P
    lib.orc_graph_new.argtypes = [ctypes.c_int32, P, P, P, ctypes.c_int64, P, P, ctypes.c_int32,
                                  P, P, P, ctypes.c_double, ctypes.c_double]
    lib.orc_graph_free.argtypes = [P]
    lib.orc_graph_n_total.restype = ctypes.c_int32
    lib.orc_graph_n_total.argtypes = [P]
    lib.orc_graph_n_edges.restype = ctypes.c_int64
    lib.orc_graph_n_edges.argtypes = [P]
    lib.orc_eval.argtypes = [P, P, P, P, P, P, P]
    lib.orc_eval_batch.argtypes = [P, ctypes.c_int64, P, P, P, P, P]
    lib.orc_idom.restype = ctypes.c_int
    lib.orc_idom.argtypes = [P, P]
    lib.orc_hotspots.restype = ctypes.c_int
    lib.orc_hotspots.argtypes = [P, P, P, ctypes.c_int32, P, P, P, P]
    lib.orc_pareto.restype = ctypes.c_int64
    lib.orc_pareto.argtypes = [ctypes.c_int64, P, P, P, P, P]
    lib.orc_best_mem.restype = ctypes.c_int64
    lib.orc_best_mem.argtypes = [ctypes.c_int64, P, P, P, P, ctypes.c_int64]
    lib.orc_best_lat.restype = ctypes.c_int64
    lib.orc_best_lat.argtypes = [ctypes.c_int64, P, P, P, P, ctypes.c_double]
    lib.orc_graph_set_regions.restype = ctypes.c_int
    lib.orc_graph_set_regions.argtypes = [P, ctypes.c_int32, P, P, P]
    lib.orc_graph_dec_len.restype = ctypes.c_int32
    lib.orc_graph_dec_len.argtypes = [P]
    lib.orc_mix64.restype = ctypes.c_uint64
    lib.orc_mix64.argtypes = [ctypes.c_uint64]
    lib.orc_hash_words.restype = ctypes.c_uint64
    lib.orc_hash_words.argtypes = [P, ctypes.c_int64]
    lib.orc_graph_hash.restype = ctypes.c_int
    lib.orc_graph_hash.argtypes = [P, P, P, P, P]
    lib.orc_graph_hash_batch.argtypes = [P, P, ctypes.c_int64, P, P, P]
    _lib = lib
    return lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


class OracleGraph:
    """Graph G = (V, E) with size(v), cost(v), outs(G) (Table 1),
    plus the eligible tensors t_r with their late-user sets U_r (reading P6)
    and the swap link model (bytes/s, latency; reading P7)."""

    def __init__(self, size, cost, is_output, src, dst, elig=(), U=(),
                 swap_Bps: float = 25e9, swap_lat: float = 1e-5, regions=None):
        self._lib = _load()
        self.size = np.ascontiguousarray(size, dtype=np.int64)
        self.cost = np.ascontiguousarray(cost, dtype=np.float64)
        self.n = int(self.size.shape[0])
        self.is_output = np.ascontiguousarray(is_output, dtype=np.uint8)
        self.src = np.ascontiguousarray(src, dtype=np.int32)
        self.dst = np.ascontiguousarray(dst, dtype=np.int32)
        self.elig = np.ascontiguousarray(elig, dtype=np.int32).reshape(-1)
        self.R = int(self.elig.shape[0])
        U = list(U)
        assert len(U) == self.R
        ptr = np.zeros(self.R + 1, dtype=np.int64)
        for r, u in enumerate(U):
            ptr[r + 1] = ptr[r] + len(u)
        self.U_ptr = ptr
        self.U_idx = np.ascontiguousarray(np.concatenate([np.asarray(u, dtype=np.int32) for u in U])
                                          if self.R else np.zeros(0, np.int32), dtype=np.int32)
        self.swap_Bps = float(swap_Bps)
        self.swap_lat = float(swap_lat)
        h = self._lib.orc_graph_new(self.n, _ptr(self.size), _ptr(self.cost), _ptr(self.is_output),
                                    int(self.src.shape[0]), _ptr(self.src), _ptr(self.dst), self.R,
                                    _ptr(self.elig), _ptr(self.U_ptr), _ptr(self.U_idx),
                                    self.swap_Bps, self.swap_lat)
        if not h:
            raise ValueError("oracle: malformed graph")
        self._h = h
        self.n_total = int(self._lib.orc_graph_n_total(h))
        self.n_edges = int(self._lib.orc_graph_n_edges(h))
        # F-Trans variant regions (NEXT-4, reading F1): dict(n_variants [F],
        # node_region [n] (-1 = in every variant), node_variant [n])
        self.F = 0
        if regions is not None:
            nv = np.ascontiguousarray(regions["n_variants"], dtype=np.int32)
            nr = np.ascontiguousarray(regions["node_region"], dtype=np.int32)
            vn = np.ascontiguousarray(regions["node_variant"], dtype=np.uint8)
            assert nr.shape == (self.n,) and vn.shape == (self.n,)
            self._regions = (nv, nr, vn)
            if self._lib.orc_graph_set_regions(h, int(nv.shape[0]), _ptr(nv), _ptr(nr), _ptr(vn)) != 0:
                raise ValueError("oracle: bad regions")
            self.F = int(nv.shape[0])
        self.dec_len = self.R + self.F

    @classmethod
    def from_workload(cls, wl):
        """Build from a magis_inputs.Workload (input generator output)."""
        return cls(wl.size, wl.cost, wl.is_output, wl.src, wl.dst, wl.elig, wl.U,
                   wl.swap_Bps, wl.swap_lat, getattr(wl, "regions", None))

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            self._lib.orc_graph_free(h)
            self._h = None

    def eval(self, perm, dec=None):
        """-> (status, peak, latency, argmax_step) for one candidate."""
        perm = np.ascontiguousarray(perm, dtype=np.int32)
        assert perm.shape == (self.n_total,)
        if dec is None:
            dec = np.zeros(max(self.dec_len, 1), dtype=np.uint8)
        dec = np.ascontiguousarray(dec, dtype=np.uint8)
        st = np.zeros(1, np.uint8)
        pk = np.zeros(1, np.int64)
        lt = np.zeros(1, np.float64)
        am = np.zeros(1, np.int64)
        self._lib.orc_eval(self._h, _ptr(perm), _ptr(dec), _ptr(st), _ptr(pk), _ptr(lt), _ptr(am))
        return int(st[0]), int(pk[0]), float(lt[0]), int(am[0])

    def eval_batch(self, perms, decs=None):
        """perms: (K, n_total) int32; decs: (K, R) uint8 -> (status, peak, lat) arrays."""
        perms = np.ascontiguousarray(perms, dtype=np.int32)
        K = perms.shape[0]
        assert perms.shape[1] == self.n_total
        if decs is None or self.dec_len == 0:
            decs = np.zeros((K, max(self.dec_len, 1)), dtype=np.uint8)
        decs = np.ascontiguousarray(decs, dtype=np.uint8)
        assert decs.shape[1] >= self.dec_len
        decs = np.ascontiguousarray(decs[:, :max(self.dec_len, 1)])
        st = np.zeros(K, np.uint8)
        pk = np.zeros(K, np.int64)
        lt = np.zeros(K, np.float64)
        self._lib.orc_eval_batch(self._h, K, _ptr(perms), _ptr(decs), _ptr(st), _ptr(pk), _ptr(lt))
        return st, pk, lt

    def idom(self):
        """Immediate dominators of the original graph (-1: only the sources'
        virtual root dominates), from the plain set definition."""
        out = np.zeros(max(self.n, 1), np.int32)
        if self._lib.orc_idom(self._h, _ptr(out)) != 0:
            raise ValueError("oracle: cyclic graph")
        return out[:self.n]

    def hotspots(self, perm, dec=None, nsplit: int = 2):
        """Memory hot-spots H (reading H1) and heat / score
        (Eq. 3-4) -> (status, peak, hot[n] u8, heat[n] int64, score[n] f64)."""
        perm = np.ascontiguousarray(perm, dtype=np.int32)
        assert perm.shape == (self.n_total,)
        if dec is None or self.R == 0:
            dec = np.zeros(max(self.R, 1), dtype=np.uint8)
        dec = np.ascontiguousarray(dec, dtype=np.uint8)
        m = max(self.n, 1)
        hot = np.zeros(m, np.uint8)
        heat = np.zeros(m, np.int64)
        score = np.zeros(m, np.float64)
        pk = np.zeros(1, np.int64)
        st = self._lib.orc_hotspots(self._h, _ptr(perm), _ptr(dec), int(nsplit), _ptr(hot), _ptr(heat),
                                    _ptr(score), _ptr(pk))
        return int(st), int(pk[0]), hot[:self.n], heat[:self.n], score[:self.n]

    def graph_hash(self, label, dec=None):
        """GraphHash of one candidate's transformed graph (Alg. 3 lines 3-6,
        P:1693-1700; readings G1-G4) -> (status, hash, x[n_total]); x_v = 0
        for inactive nodes."""
        label = np.ascontiguousarray(label, dtype=np.uint64)
        assert label.shape == (self.n,)
        if dec is None or self.R == 0:
            dec = np.zeros(max(self.R, 1), dtype=np.uint8)
        dec = np.ascontiguousarray(dec, dtype=np.uint8)
        x = np.zeros(max(self.n_total, 1), np.uint64)
        h = np.zeros(1, np.uint64)
        st = self._lib.orc_graph_hash(self._h, _ptr(label), _ptr(dec), _ptr(x), _ptr(h))
        return int(st), int(h[0]), x[:self.n_total]

    def graph_hash_batch(self, label, decs):
        """decs: (K, R) uint8 -> (status u8[K], hash u64[K])."""
        label = np.ascontiguousarray(label, dtype=np.uint64)
        decs = np.ascontiguousarray(decs, dtype=np.uint8)
        K = decs.shape[0]
        if self.R == 0:
            decs = np.zeros((K, 1), dtype=np.uint8)
        st = np.zeros(K, np.uint8)
        hs = np.zeros(K, np.uint64)
        self._lib.orc_graph_hash_batch(self._h, _ptr(label), K, _ptr(decs), _ptr(st), _ptr(hs))
        return st, hs


def mix64(z: int) -> int:
    """The SplitMix64 output function (reading G1)."""
    return int(_load().orc_mix64(ctypes.c_uint64(z & 0xFFFFFFFFFFFFFFFF)))


def hash_words(words) -> int:
    """hash() of Alg. 3 over the concatenation of 64-bit words (reading G1)."""
    w = np.ascontiguousarray(words, dtype=np.uint64)
    return int(_load().orc_hash_words(_ptr(w), int(w.shape[0])))


def hash_filter(hashes, status, seen=None):
    """Alg. 3 lines 10-12 over a batch in candidate-id order: candidate k is
    new iff it is valid, its hash is not in X (``seen``) and no earlier valid
    candidate of the batch has the same hash; X then takes every valid hash.
    Returns (new u8[K], X)."""
    X = set() if seen is None else set(seen)
    new = np.zeros(len(hashes), np.uint8)
    for k, (h, s) in enumerate(zip(hashes, status)):
        if s:
            continue
        h = int(h)
        if h in X:
            continue
        X.add(h)
        new[k] = 1
    return new, X


def pareto(peak, lat, status, ids=None):
    """Indices of the Pareto front (ascending peak), by brute-force dominance."""
    lib = _load()
    peak = np.ascontiguousarray(peak, dtype=np.int64)
    lat = np.ascontiguousarray(lat, dtype=np.float64)
    status = np.ascontiguousarray(status, dtype=np.uint8)
    n = peak.shape[0]
    ids = np.arange(n, dtype=np.int64) if ids is None else np.ascontiguousarray(ids, dtype=np.int64)
    out = np.zeros(max(n, 1), np.int64)
    nf = lib.orc_pareto(n, _ptr(peak), _ptr(lat), _ptr(status), _ptr(ids), _ptr(out))
    return out[:nf].copy()


def best_under_memory(peak, lat, status, M, ids=None):
    """Alg. 3 BetterThan-best under memory limit M -> index or -1."""
    lib = _load()
    peak = np.ascontiguousarray(peak, dtype=np.int64)
    lat = np.ascontiguousarray(lat, dtype=np.float64)
    status = np.ascontiguousarray(status, dtype=np.uint8)
    n = peak.shape[0]
    ids = np.arange(n, dtype=np.int64) if ids is None else np.ascontiguousarray(ids, dtype=np.int64)
    return int(lib.orc_best_mem(n, _ptr(peak), _ptr(lat), _ptr(status), _ptr(ids), int(M)))


def best_under_latency(peak, lat, status, L, ids=None):
    """Second optimisation mode: best under latency limit L."""
    lib = _load()
    peak = np.ascontiguousarray(peak, dtype=np.int64)
    lat = np.ascontiguousarray(lat, dtype=np.float64)
    status = np.ascontiguousarray(status, dtype=np.uint8)
    n = peak.shape[0]
    ids = np.arange(n, dtype=np.int64) if ids is None else np.ascontiguousarray(ids, dtype=np.int64)
    return int(lib.orc_best_lat(n, _ptr(peak), _ptr(lat), _ptr(status), _ptr(ids), float(L)))


def eq1_estimate(H, S, I, size, n):
    """Eq. (1): M_f ~= sum_{(H\\S) u I} |v| + sum_{H n S} |v| / n.

    H, S, I are collections of node ids; size maps id -> bytes.  Returns a
    float (the paper's estimate; it is an approximation, reading P16)."""
    H, S, I = set(H), set(S), set(I)
    outside = (H - S) | I
    return float(sum(size[v] for v in outside)) + sum(size[v] for v in (H & S)) / float(n)


def eq1_m0(H, size):
    """M_0 = sum_{v in H} |v| (Eq. (1))."""
    return float(sum(size[v] for v in set(H)))
