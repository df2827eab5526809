"""Seeded candidate schedules (perm + decisions) -- INPUT GENERATION ONLY.

Python front end of csrc/candgen.c (recipe in its header and DESIGN.md
§Inputs).  Candidates depend only on (seed, global id), never on sharding.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

from .graph import Workload

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "csrc", "candgen.c")
_LIB = os.path.join(_HERE, "csrc", "libcandgen.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=gnu99", "-shared", "-fPIC", "-o", _LIB, _SRC,
                               "-lpthread"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i32, i64, u64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
        lib.candgen.argtypes = [i32, i32, P, P, P, P, P, P, P, u64, i32, i32, i32, i32, i32, i32,
                                u64, i64, P, P, i32]
        lib.candgen.restype = None
        lib.candgen_regions.argtypes = [i32, i32, P, P, P, P, P, P, P, u64, i32, i32, i32, i32, i32, i32,
                                        u64, i64, P, P, i32, i32, P, P, P]
        lib.candgen_regions.restype = None
        lib.wingen.argtypes = [i32, i32, P, P, P, P, P, P, P, P, P, P, u64, i32, i32, u64, i64, P, P, P]
        lib.wingen.restype = None
        _lib = lib
    return _lib


@dataclass
class CandidateSpec:
    """Candidate mix: 75% random topo orders, 24% local moves,
    1% random transposition; P(remat) = P(swap) = 5% per eligible tensor;
    windows <= 64; Load/clone slack 0-8 steps."""
    seed: int = 1
    pct_random: int = 75
    pct_local: int = 24
    p_remat: int = 500      # per 10000
    p_swap: int = 500       # per 10000
    wmax: int = 64
    slack: int = 8


def csr(n: int, src: np.ndarray, dst: np.ndarray):
    """Deduplicated successor / predecessor CSR (both sorted)."""
    if src.size:
        key = np.unique(src.astype(np.int64) * n + dst.astype(np.int64))
        s = (key // n).astype(np.int32)
        d = (key % n).astype(np.int32)
    else:
        s = d = np.zeros(0, np.int32)
    sp = np.zeros(n + 1, np.int64)
    np.add.at(sp, s.astype(np.int64) + 1, 1)
    sp = np.cumsum(sp)
    order = np.lexsort((s, d))
    pp = np.zeros(n + 1, np.int64)
    np.add.at(pp, d.astype(np.int64) + 1, 1)
    pp = np.cumsum(pp)
    return sp, d.copy(), pp, s[order].copy()


class CandidateGenerator:
    def __init__(self, wl: Workload, spec: CandidateSpec | None = None):
        self.wl = wl
        self.spec = spec or CandidateSpec()
        self.succ_ptr, self.succ_idx, self.pred_ptr, self.pred_idx = csr(wl.n, wl.src, wl.dst)
        self.U_ptr, self.U_idx = wl.U_arrays()
        self.elig = np.ascontiguousarray(wl.elig, np.int32)

    def generate(self, id0: int, K: int, nthreads: int | None = None, out=None):
        """-> (perms int32 [K, n_total], decs uint8 [K, max(R + F, 1)]); with
        F-Trans variant regions (NEXT-4) the last F columns are the chosen
        variants."""
        lib = _load()
        wl, sp = self.wl, self.spec
        NT = wl.n_total
        F = wl.F
        if out is None:
            perms = np.empty((K, NT), np.int32)
            decs = np.zeros((K, max(wl.R + F, 1)), np.uint8)
        else:
            perms, decs = out
        if nthreads is None:
            nthreads = max(1, min(os.cpu_count() or 1, 64))
        p = lambda a: a.ctypes.data_as(ctypes.c_void_p)
        args = [wl.n, wl.R, p(self.succ_ptr), p(self.succ_idx), p(self.pred_ptr), p(self.pred_idx),
                p(self.elig), p(self.U_ptr), p(self.U_idx), ctypes.c_uint64(sp.seed),
                sp.pct_random, sp.pct_local, sp.p_remat, sp.p_swap, sp.wmax, sp.slack,
                ctypes.c_uint64(id0), K, p(perms), p(decs), int(nthreads)]
        if F:
            rg = wl.regions
            self._rk = (np.ascontiguousarray(rg["n_variants"], np.int32),
                        np.ascontiguousarray(rg["node_region"], np.int32),
                        np.ascontiguousarray(rg["node_variant"], np.uint8))
            lib.candgen_regions(*args, F, *(p(a) for a in self._rk))
        else:
            lib.candgen(*args)
        return perms, decs


class WindowGenerator:
    """Local-move candidates over a base schedule (csrc/candgen.c wingen):
    candidate k re-orders base steps [wstart, wstart + wlen) by the keyed Kahn
    over the window's dependencies under the base decisions; pct_bad % get the
    window's two ends swapped (may be invalid)."""

    def __init__(self, wl: Workload, base_perm, base_dec=None, seed: int = 1, wmax: int = 64, pct_bad: int = 1):
        self.wl = wl
        self.NT = wl.n_total
        self.bperm = np.ascontiguousarray(base_perm, np.int32)
        self.bpos = np.empty(self.NT, np.int32)
        self.bpos[self.bperm] = np.arange(self.NT, dtype=np.int32)
        self.bdec = np.ascontiguousarray(base_dec if base_dec is not None else np.zeros(max(wl.R, 1)), np.uint8)
        self.seed, self.wmax, self.pct_bad = seed, wmax, pct_bad
        _, _, self.pred_ptr, self.pred_idx = csr(wl.n, wl.src, wl.dst)
        self.U_ptr, self.U_idx = wl.U_arrays()
        lu = [[] for _ in range(wl.n)]
        for r, us in enumerate(wl.U):
            for b in us:
                lu[b].append(r)
        self.lu_ptr = np.zeros(wl.n + 1, np.int64)
        for v in range(wl.n):
            self.lu_ptr[v + 1] = self.lu_ptr[v] + len(lu[v])
        self.lu_idx = np.ascontiguousarray(np.concatenate([np.asarray(x, np.int32) for x in lu])
                                           if self.lu_ptr[-1] else np.zeros(0, np.int32), np.int32)
        self.elig = np.ascontiguousarray(wl.elig, np.int32)

    def generate(self, id0: int, K: int):
        lib = _load()
        ws = np.empty(K, np.int32)
        wln = np.empty(K, np.int32)
        wp = np.empty((K, self.wmax), np.int32)
        p = lambda a: a.ctypes.data_as(ctypes.c_void_p)
        lib.wingen(self.wl.n, self.wl.R, p(self.pred_ptr), p(self.pred_idx), p(self.elig), p(self.U_ptr),
                   p(self.U_idx), p(self.lu_ptr), p(self.lu_idx), p(self.bperm), p(self.bpos), p(self.bdec),
                   ctypes.c_uint64(self.seed), self.wmax, self.pct_bad, ctypes.c_uint64(id0), K, p(ws), p(wln), p(wp))
        return ws, wln, wp

    def expand(self, ws, wln, wp):
        """Full perms of window candidates (for the oracle)."""
        K = len(ws)
        out = np.repeat(self.bperm[None, :], K, axis=0)
        for k in range(K):
            b, w = int(ws[k]), int(wln[k])
            out[k, b:b + w] = wp[k, :w]
        return out
