"""Thin ctypes binding of libmagis.so (include/magis.h) -- argument marshalling only.

Every step of the evaluation runs in the library's sm_100a kernels; PyTorch
supplies device memory and streams.  There is no fallback: if libmagis.so is
missing or no B200 is visible, the calls raise MagisError.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Sequence

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# MAGIS_LIB: an alternative in-tree build (A/B timing of kernel variants)
LIB_PATH = os.environ.get("MAGIS_LIB") or os.path.join(_PKG, "libmagis.so")

MAGIS_SUCCESS = 0
ERRORS = {-1: "MAGIS_E_INVAL", -2: "MAGIS_E_CYCLE", -3: "MAGIS_E_NOMEM", -4: "MAGIS_E_CUDA",
          -5: "MAGIS_E_UNSUPPORTED", -6: "MAGIS_E_CAPACITY"}
ST_NOT_PERM, ST_EDGE, ST_BAD_DEC = 1, 2, 4

# names declared in include/magis.h (checked by tests/test_abi.py)
EXPORTS = ["magis_graph_load", "magis_graph_free", "magis_graph_info_get", "magis_eval_schedules",
           "magis_eval_schedules_host", "magis_pareto_workspace_size", "magis_pareto_merge",
           "magis_last_error", "magis_abi_version", "magis_device_supported", "magis_generate_candidates",
           "magis_base_create", "magis_base_info", "magis_base_free", "magis_eval_windows", "magis_hotspots",
           "magis_graph_idom", "magis_eval_schedules_host_u16", "magis_ghash_create", "magis_ghash_free",
           "magis_graph_hash", "magis_ghash_info", "magis_hashset_create", "magis_hashset_free",
           "magis_hashset_clear", "magis_hashset_filter", "magis_hashset_stats", "magis_graph_load_regions",
           "magis_eval_schedules_host_delta8", "magis_eval_schedules_host_delta4", "magis_eval_schedules_argmax"]


class MagisError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{ERRORS.get(code, code)}: {msg}")
        self.code = code


class GraphDesc(ctypes.Structure):
    _fields_ = [("n_nodes", ctypes.c_int32), ("out_bytes", ctypes.c_void_p), ("cost", ctypes.c_void_p),
                ("is_output", ctypes.c_void_p), ("n_edges", ctypes.c_int64), ("edge_src", ctypes.c_void_p),
                ("edge_dst", ctypes.c_void_p), ("n_eligible", ctypes.c_int32),
                ("eligible_tensor", ctypes.c_void_p), ("late_user_ptr", ctypes.c_void_p),
                ("late_user_idx", ctypes.c_void_p), ("swap_bytes_per_s", ctypes.c_double),
                ("swap_latency_s", ctypes.c_double)]


class GenSpec(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("pct_random", ctypes.c_int32), ("pct_local", ctypes.c_int32),
                ("p_remat", ctypes.c_int32), ("p_swap", ctypes.c_int32), ("wmax", ctypes.c_int32),
                ("slack", ctypes.c_int32)]


class GraphInfo(ctypes.Structure):
    _fields_ = [("n_nodes", ctypes.c_int32), ("n_eligible", ctypes.c_int32), ("n_total", ctypes.c_int32),
                ("n_edges", ctypes.c_int64), ("n_super_edges", ctypes.c_int64), ("device", ctypes.c_int32),
                ("variant", ctypes.c_int32), ("grid", ctypes.c_int32), ("block", ctypes.c_int32),
                ("smem_bytes", ctypes.c_int64), ("table_bytes", ctypes.c_int64), ("base_cost", ctypes.c_double),
                ("pack", ctypes.c_int32), ("n_regions", ctypes.c_int32)]


class RegionDesc(ctypes.Structure):
    _fields_ = [("n_regions", ctypes.c_int32), ("n_variants", ctypes.c_void_p), ("node_region", ctypes.c_void_p),
                ("node_variant", ctypes.c_void_p)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load libmagis.so (raises if it is not built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise MagisError(-5, f"{LIB_PATH} not built (run __graft_entry__.build()); there is no fallback")
    L = ctypes.CDLL(LIB_PATH)
    P, i32, i64, d = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_double
    L.magis_graph_load.argtypes = [ctypes.POINTER(GraphDesc), ctypes.c_int, ctypes.POINTER(P)]
    L.magis_graph_load.restype = ctypes.c_int
    L.magis_graph_load_regions.argtypes = [ctypes.POINTER(GraphDesc), ctypes.POINTER(RegionDesc), ctypes.c_int,
                                           ctypes.POINTER(P)]
    L.magis_graph_load_regions.restype = ctypes.c_int
    L.magis_graph_free.argtypes = [P]
    L.magis_graph_free.restype = ctypes.c_int
    L.magis_graph_info_get.argtypes = [P, ctypes.POINTER(GraphInfo)]
    L.magis_graph_info_get.restype = ctypes.c_int
    L.magis_eval_schedules.argtypes = [P, i64, P, P, P, P, P, P]
    L.magis_eval_schedules.restype = ctypes.c_int
    L.magis_eval_schedules_argmax.argtypes = [P, i64, P, P, P, P, P, P, P]
    L.magis_eval_schedules_argmax.restype = ctypes.c_int
    L.magis_eval_schedules_host.argtypes = [P, i64, P, P, P, P, P, P]
    L.magis_eval_schedules_host.restype = ctypes.c_int
    L.magis_eval_schedules_host_u16.argtypes = [P, i64, P, P, P, P, P, P]
    L.magis_eval_schedules_host_u16.restype = ctypes.c_int
    L.magis_eval_schedules_host_delta8.argtypes = [P, i64, P, P, P, P, P, P, P, P]
    L.magis_eval_schedules_host_delta8.restype = ctypes.c_int
    L.magis_eval_schedules_host_delta4.argtypes = [P, i64, P, P, P, P, P, P, P, P]
    L.magis_eval_schedules_host_delta4.restype = ctypes.c_int
    L.magis_pareto_workspace_size.argtypes = [i64]
    L.magis_pareto_workspace_size.restype = i64
    L.magis_pareto_merge.argtypes = [i64, P, P, P, P, i64, i64, P, P, P, P, i64, d, P, P, i64, P]
    L.magis_pareto_merge.restype = ctypes.c_int
    L.magis_last_error.argtypes = []
    L.magis_last_error.restype = ctypes.c_char_p
    L.magis_abi_version.restype = ctypes.c_int
    L.magis_device_supported.argtypes = [ctypes.c_int]
    L.magis_device_supported.restype = ctypes.c_int
    L.magis_generate_candidates.argtypes = [P, ctypes.POINTER(GenSpec), ctypes.c_uint64, i64, P, P, P]
    L.magis_generate_candidates.restype = ctypes.c_int
    L.magis_base_create.argtypes = [P, P, P, ctypes.POINTER(P), P]
    L.magis_base_create.restype = ctypes.c_int
    L.magis_base_info.argtypes = [P, ctypes.POINTER(ctypes.c_int), ctypes.POINTER(i64), ctypes.POINTER(d)]
    L.magis_base_info.restype = ctypes.c_int
    L.magis_base_free.argtypes = [P]
    L.magis_base_free.restype = ctypes.c_int
    L.magis_eval_windows.argtypes = [P, i64, P, P, P, i32, P, P, P, P]
    L.magis_eval_windows.restype = ctypes.c_int
    L.magis_hotspots.argtypes = [P, i64, P, P, i32, P, P, P, P, P, P]
    L.magis_hotspots.restype = ctypes.c_int
    L.magis_graph_idom.argtypes = [P, P]
    L.magis_graph_idom.restype = ctypes.c_int
    L.magis_ghash_create.argtypes = [P, P, ctypes.POINTER(P)]
    L.magis_ghash_create.restype = ctypes.c_int
    L.magis_ghash_free.argtypes = [P]
    L.magis_ghash_free.restype = ctypes.c_int
    L.magis_graph_hash.argtypes = [P, i64, P, P, P, P]
    L.magis_graph_hash.restype = ctypes.c_int
    L.magis_ghash_info.argtypes = [P, ctypes.POINTER(i32), ctypes.POINTER(i32), ctypes.POINTER(i64),
                                   ctypes.POINTER(i32)]
    L.magis_ghash_info.restype = ctypes.c_int
    L.magis_hashset_create.argtypes = [ctypes.c_int, i64, ctypes.POINTER(P)]
    L.magis_hashset_create.restype = ctypes.c_int
    L.magis_hashset_free.argtypes = [P]
    L.magis_hashset_free.restype = ctypes.c_int
    L.magis_hashset_clear.argtypes = [P, P]
    L.magis_hashset_clear.restype = ctypes.c_int
    L.magis_hashset_filter.argtypes = [P, i64, P, P, P, P]
    L.magis_hashset_filter.restype = ctypes.c_int
    L.magis_hashset_stats.argtypes = [P, ctypes.POINTER(i64), ctypes.POINTER(i64)]
    L.magis_hashset_stats.restype = ctypes.c_int
    _lib = L
    return L


def _check(code: int):
    if code != MAGIS_SUCCESS:
        msg = lib().magis_last_error()
        raise MagisError(code, msg.decode() if msg else "")


def _np_ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None and a.size else None


def _tptr(t) -> Optional[int]:
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream_ptr(stream) -> Optional[ctypes.c_void_p]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def encode_delta8(perm: np.ndarray):
    """The delta8 wire format of magis_eval_schedules_host_delta8 (marshalling
    only): per step the int8 difference to the previous step's id (rows start
    from 0), -128 where it does not fit, with the absolute ids of those steps
    in a per-row exception list.  Ids outside [0, 65535] are clamped to 65535
    (still out of range for any graph the format supports, so the candidate
    stays MAGIS_ST_NOT_PERM).  -> (delta int8 [K, n], exc_ptr int32 [K+1],
    exc uint16 [E])."""
    p = np.asarray(perm, np.int64)
    if p.ndim == 1:
        p = p[None, :]
    p = np.where((p < 0) | (p > 65535), 65535, p)
    prev = np.concatenate([np.zeros((p.shape[0], 1), np.int64), p[:, :-1]], axis=1)
    d = p - prev
    esc = (d < -127) | (d > 127)
    delta = np.where(esc, -128, d).astype(np.int8)
    exc = np.ascontiguousarray(p[esc], np.uint16)
    exc_ptr = np.zeros(p.shape[0] + 1, np.int32)
    np.cumsum(esc.sum(axis=1), out=exc_ptr[1:])
    return np.ascontiguousarray(delta), exc_ptr, exc


def encode_delta4(perm: np.ndarray):
    """The delta4 wire format of magis_eval_schedules_host_delta4 (marshalling
    only): per step one nibble, c = d + 8 for a difference d in [-7, 7] to
    the previous step's id (rows start from 0), c = 0 where it does not fit,
    with the absolute ids of those steps in a per-row exception list; two
    steps per byte, the even step in the low nibble.  Ids outside [0, 65535]
    are clamped to 65535 (the candidate stays MAGIS_ST_NOT_PERM).
    -> (code uint8 [K, ceil(n / 2)], exc_ptr int32 [K+1], exc uint16 [E])."""
    p = np.asarray(perm, np.int64)
    if p.ndim == 1:
        p = p[None, :]
    p = np.where((p < 0) | (p > 65535), 65535, p)
    prev = np.concatenate([np.zeros((p.shape[0], 1), np.int64), p[:, :-1]], axis=1)
    d = p - prev
    esc = (d < -7) | (d > 7)
    c = np.where(esc, 0, d + 8).astype(np.uint8)
    if c.shape[1] % 2:
        c = np.concatenate([c, np.full((c.shape[0], 1), 8, np.uint8)], axis=1)
    code = (c[:, 0::2] | (c[:, 1::2] << 4)).astype(np.uint8)
    exc = np.ascontiguousarray(p[esc], np.uint16)
    exc_ptr = np.zeros(p.shape[0] + 1, np.int32)
    np.cumsum(esc.sum(axis=1), out=exc_ptr[1:])
    return np.ascontiguousarray(code), exc_ptr, exc


class Graph:
    """A loaded graph (magis_graph_load).  Arguments follow Table 1:
    out_bytes = size(v), cost = cost(v), is_output = outs(G), edges E, plus the
    eligible tensors t_r with late users U_r and the swap link model."""

    def __init__(self, out_bytes, cost, is_output, edge_src, edge_dst, eligible: Sequence[int] = (),
                 late_users: Sequence[Sequence[int]] = (), swap_bytes_per_s: float = 25e9,
                 swap_latency_s: float = 1e-5, device: int = 0, regions=None):
        L = lib()
        self._L = L
        self._h = None
        ob = np.ascontiguousarray(out_bytes, np.int64)
        co = np.ascontiguousarray(cost, np.float64)
        io = np.ascontiguousarray(is_output, np.uint8)
        es = np.ascontiguousarray(edge_src, np.int32)
        ed = np.ascontiguousarray(edge_dst, np.int32)
        el = np.ascontiguousarray(eligible, np.int32).reshape(-1)
        lu = [np.asarray(u, np.int32) for u in late_users]
        ptr = np.zeros(len(lu) + 1, np.int64)
        for i, u in enumerate(lu):
            ptr[i + 1] = ptr[i] + u.size
        idx = np.ascontiguousarray(np.concatenate(lu) if lu else np.zeros(0, np.int32), np.int32)
        self._keep = (ob, co, io, es, ed, el, ptr, idx)
        d = GraphDesc(int(ob.size), _np_ptr(ob), _np_ptr(co), _np_ptr(io), int(es.size), _np_ptr(es),
                      _np_ptr(ed), int(el.size), _np_ptr(el), ptr.ctypes.data_as(ctypes.c_void_p),
                      _np_ptr(idx), float(swap_bytes_per_s), float(swap_latency_s))
        h = ctypes.c_void_p()
        if regions is None:
            _check(L.magis_graph_load(ctypes.byref(d), int(device), ctypes.byref(h)))
        else:
            # F-Trans variant regions (NEXT-4): dict(n_variants, node_region, node_variant)
            nv = np.ascontiguousarray(regions["n_variants"], np.int32)
            nr = np.ascontiguousarray(regions["node_region"], np.int32)
            vn = np.ascontiguousarray(regions["node_variant"], np.uint8)
            self._keep_regions = (nv, nr, vn)
            rd = RegionDesc(int(nv.size), _np_ptr(nv), _np_ptr(nr), _np_ptr(vn))
            _check(L.magis_graph_load_regions(ctypes.byref(d), ctypes.byref(rd), int(device), ctypes.byref(h)))
        self._h = h
        self.device = device
        info = GraphInfo()
        _check(L.magis_graph_info_get(h, ctypes.byref(info)))
        self.info = {f: getattr(info, f) for f, _ in GraphInfo._fields_}
        self.n_total = info.n_total
        self.R = info.n_eligible
        self.n = info.n_nodes
        self.F = info.n_regions
        self.dec_len = self.R + self.F          # decision row: R eligible + F region variants

    @classmethod
    def from_workload(cls, wl, device: int = 0) -> "Graph":
        return cls(wl.size, wl.cost, wl.is_output, wl.src, wl.dst, wl.elig, wl.U, wl.swap_Bps,
                   wl.swap_lat, device, getattr(wl, "regions", None))

    def close(self):
        if self._h:
            self._L.magis_graph_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def eval_schedules(self, perm, dec=None, status=None, peak=None, latency=None, stream=None, argmax=None):
        """perm: cuda int32 [K, n_total]; dec: cuda uint8 [K, R + F] (or None if R + F == 0).
        Returns (status uint8 [K], peak int64 [K], latency float64 [K]) device tensors;
        with ``argmax`` (True, or an int32 [K] cuda tensor) also the first step
        reaching the peak (magis_eval_schedules_argmax) as a fourth tensor."""
        import torch
        K = int(perm.shape[0])
        assert perm.dtype == torch.int32 and perm.is_cuda and perm.is_contiguous()
        assert perm.shape[1] == self.n_total, (perm.shape, self.n_total)
        if self.dec_len:
            assert dec is not None and dec.dtype == torch.uint8 and dec.is_contiguous()
            assert dec.shape[0] == K and dec.shape[1] == self.dec_len
        dev = perm.device
        status = torch.empty(K, dtype=torch.uint8, device=dev) if status is None else status
        peak = torch.empty(K, dtype=torch.int64, device=dev) if peak is None else peak
        latency = torch.empty(K, dtype=torch.float64, device=dev) if latency is None else latency
        if argmax is not None and argmax is not False:
            am = torch.empty(K, dtype=torch.int32, device=dev) if argmax is True else argmax
            _check(self._L.magis_eval_schedules_argmax(self._h, K, _tptr(perm), _tptr(dec) if self.dec_len else None,
                                                       _tptr(status), _tptr(peak), _tptr(latency), _tptr(am),
                                                       _stream_ptr(stream)))
            return status, peak, latency, am
        _check(self._L.magis_eval_schedules(self._h, K, _tptr(perm), _tptr(dec) if self.dec_len else None,
                                            _tptr(status), _tptr(peak), _tptr(latency),
                                            _stream_ptr(stream)))
        return status, peak, latency

    def generate_candidates(self, id0: int, K: int, seed: int = 1, pct_random: int = 75, pct_local: int = 24,
                            p_remat: int = 500, p_swap: int = 500, wmax: int = 64, slack: int = 8,
                            perm=None, dec=None, stream=None):
        """Device candidate generator (magis_generate_candidates): returns
        (perm int32 [K, n_total], dec uint8 [K, max(R,1)]) cuda tensors."""
        import torch
        dev = torch.device("cuda", self.device)
        perm = torch.empty((K, self.n_total), dtype=torch.int32, device=dev) if perm is None else perm
        dec = torch.empty((K, max(self.R, 1)), dtype=torch.uint8, device=dev) if dec is None else dec
        spec = GenSpec(int(seed), pct_random, pct_local, p_remat, p_swap, wmax, slack)
        _check(self._L.magis_generate_candidates(self._h, ctypes.byref(spec), int(id0), int(K), _tptr(perm),
                                                 _tptr(dec), _stream_ptr(stream)))
        return perm, dec

    def hotspots(self, perm, dec=None, nsplit: int = 2, heat: bool = True, score: bool = True, stream=None):
        """Memory hot-spots and heat / score (magis_hotspots, NEXT-3) of the
        candidates in perm (cuda int32 [K, n_total]) / dec (cuda uint8 [K, R]).
        Returns (status [K], peak [K], hot uint8 [K, n], heat int64 [K, n] or
        None, score float64 [K, n] or None) device tensors."""
        import torch
        K = int(perm.shape[0])
        assert perm.dtype == torch.int32 and perm.is_cuda and perm.is_contiguous()
        assert perm.shape[1] == self.n_total
        if self.R:
            assert dec is not None and dec.dtype == torch.uint8 and dec.is_contiguous()
            assert dec.shape[0] == K and dec.shape[1] == self.R
        dev = perm.device
        st = torch.empty(K, dtype=torch.uint8, device=dev)
        pk = torch.empty(K, dtype=torch.int64, device=dev)
        hot = torch.empty((K, self.n), dtype=torch.uint8, device=dev)
        ht = torch.empty((K, self.n), dtype=torch.int64, device=dev) if heat else None
        sc = torch.empty((K, self.n), dtype=torch.float64, device=dev) if score else None
        _check(self._L.magis_hotspots(self._h, K, _tptr(perm), _tptr(dec) if self.R else None, int(nsplit),
                                      _tptr(st), _tptr(pk), _tptr(hot), _tptr(ht) if heat else None,
                                      _tptr(sc) if score else None, _stream_ptr(stream)))
        return st, pk, hot, ht, sc

    def idom(self) -> np.ndarray:
        """Immediate dominators of the original graph (-1: virtual root)."""
        out = np.empty(max(self.n, 1), np.int32)
        _check(self._L.magis_graph_idom(self._h, _np_ptr(out)))
        return out[:self.n]

    def eval_schedules_host(self, perm: np.ndarray, dec: Optional[np.ndarray] = None, out=None,
                            stream=None):
        """End-to-end call with host buffers (pinned numpy views or torch CPU
        tensors).  A (delta, exc_ptr, exc) tuple from encode_delta8 uses the
        delta8 wire format (magis_eval_schedules_host_delta8), a (code,
        exc_ptr, exc) tuple from encode_delta4 (uint8 codes) the delta4 one
        (magis_eval_schedules_host_delta4); uint16
        schedules the u16 format (magis_eval_schedules_host_u16); anything
        else is taken as int32."""
        import torch

        def as_np(x, dt):
            if isinstance(x, torch.Tensor):
                return x.numpy()
            return np.ascontiguousarray(x, dt)
        if isinstance(perm, tuple):           # delta8 / delta4 wire format (encode_delta8 / encode_delta4)
            delta, exc_ptr, exc = (as_np(x, None) for x in perm)
            K = delta.shape[0]
            d4 = delta.dtype == np.uint8
            assert exc_ptr.shape == (K + 1,)
            assert (d4 and delta.shape[1] == (self.n_total + 1) // 2) or (
                delta.dtype == np.int8 and delta.shape[1] == self.n_total)
            dd = as_np(dec, np.uint8) if (self.dec_len and dec is not None) else None
            if out is None:
                st, pk, lt = np.empty(K, np.uint8), np.empty(K, np.int64), np.empty(K, np.float64)
            else:
                st, pk, lt = (as_np(o, None) for o in out)
            fn = self._L.magis_eval_schedules_host_delta4 if d4 else self._L.magis_eval_schedules_host_delta8
            _check(fn(self._h, K, _np_ptr(delta), _np_ptr(exc_ptr), _np_ptr(exc), _np_ptr(dd), _np_ptr(st),
                      _np_ptr(pk), _np_ptr(lt), _stream_ptr(stream)))
            return st, pk, lt
        p = as_np(perm, None)
        u16 = p.dtype == np.uint16
        if not u16:
            p = np.ascontiguousarray(p, np.int32)
        K = p.shape[0]
        assert p.shape[1] == self.n_total
        dd = as_np(dec, np.uint8) if (self.dec_len and dec is not None) else None
        if out is None:
            st = np.empty(K, np.uint8)
            pk = np.empty(K, np.int64)
            lt = np.empty(K, np.float64)
        else:
            st, pk, lt = (as_np(o, None) for o in out)
        fn = self._L.magis_eval_schedules_host_u16 if u16 else self._L.magis_eval_schedules_host
        _check(fn(self._h, K, _np_ptr(p), _np_ptr(dd), _np_ptr(st), _np_ptr(pk), _np_ptr(lt), _stream_ptr(stream)))
        return st, pk, lt


class GraphHasher:
    """Batched GraphHash of candidate graphs (magis_ghash_create /
    magis_graph_hash; Alg. 3 lines 3-6).  labels: uint64 [n] op labels."""

    def __init__(self, graph: "Graph", labels):
        self._L = graph._L
        self.graph = graph
        lab = np.ascontiguousarray(labels, np.uint64)
        assert lab.shape == (graph.n,)
        h = ctypes.c_void_p()
        _check(self._L.magis_ghash_create(graph._h, _np_ptr(lab), ctypes.byref(h)))
        self._h = h
        ns, gs, gn, gr = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64(), ctypes.c_int32()
        _check(self._L.magis_ghash_info(h, ctypes.byref(ns), ctypes.byref(gs), ctypes.byref(gn), ctypes.byref(gr)))
        self.info = {"shared_slots": ns.value, "global_slots": gs.value, "global_nodes": gn.value,
                     "grid": gr.value}

    def hash(self, dec, status=None, out=None, stream=None):
        """dec: cuda uint8 [K, R] (R == 0: a [K, 1] tensor or an int K).
        Returns (status uint8 [K], hash int64 [K] holding the uint64 bits)."""
        import torch
        if isinstance(dec, int):
            K, dev, dp = dec, torch.device("cuda", self.graph.device), None
        else:
            K, dev = int(dec.shape[0]), dec.device
            assert dec.dtype == torch.uint8 and dec.is_contiguous()
            if self.graph.R:
                assert dec.shape[1] == self.graph.R
            dp = _tptr(dec) if self.graph.R else None
        status = torch.empty(K, dtype=torch.uint8, device=dev) if status is None else status
        out = torch.empty(K, dtype=torch.int64, device=dev) if out is None else out
        _check(self._L.magis_graph_hash(self._h, K, dp, _tptr(status), _tptr(out), _stream_ptr(stream)))
        return status, out

    def close(self):
        if getattr(self, "_h", None):
            self._L.magis_ghash_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class HashSet:
    """The seen-graph set X of Alg. 3 (lines 10-12) on the device."""

    def __init__(self, capacity: int, device: int = 0):
        self._L = lib()
        h = ctypes.c_void_p()
        _check(self._L.magis_hashset_create(int(device), int(capacity), ctypes.byref(h)))
        self._h = h
        self.device = device

    def filter(self, hashes, status=None, out=None, stream=None):
        """hashes: cuda int64 [K] (uint64 bits); status: cuda uint8 [K] or None.
        Returns is_new uint8 [K] (first valid occurrence not already in X)."""
        import torch
        K = int(hashes.shape[0])
        out = torch.empty(K, dtype=torch.uint8, device=hashes.device) if out is None else out
        _check(self._L.magis_hashset_filter(self._h, K, _tptr(hashes), _tptr(status), _tptr(out),
                                            _stream_ptr(stream)))
        return out

    def clear(self, stream=None):
        _check(self._L.magis_hashset_clear(self._h, _stream_ptr(stream)))

    def stats(self):
        n, o = ctypes.c_int64(), ctypes.c_int64()
        _check(self._L.magis_hashset_stats(self._h, ctypes.byref(n), ctypes.byref(o)))
        return n.value, o.value

    def close(self):
        if getattr(self, "_h", None):
            self._L.magis_hashset_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Base:
    """A base schedule evaluated once for windowed delta evaluation
    (magis_base_create / magis_eval_windows)."""

    def __init__(self, graph: "Graph", perm, dec=None, stream=None):
        import torch
        self._L = graph._L
        self.graph = graph
        self._keep = (perm, dec)
        h = ctypes.c_void_p()
        _check(self._L.magis_base_create(graph._h, _tptr(perm), _tptr(dec) if graph.R else None,
                                         ctypes.byref(h), _stream_ptr(stream)))
        self._h = h

    def info(self):
        st, pk, lt = ctypes.c_int(), ctypes.c_int64(), ctypes.c_double()
        _check(self._L.magis_base_info(self._h, ctypes.byref(st), ctypes.byref(pk), ctypes.byref(lt)))
        return st.value, pk.value, lt.value

    def eval_windows(self, wstart, wlen, wperm, status=None, peak=None, latency=None, stream=None):
        """wstart/wlen int32 [K], wperm int32 [K, wmax] cuda tensors."""
        import torch
        K = int(wstart.shape[0])
        dev = wstart.device
        status = torch.empty(K, dtype=torch.uint8, device=dev) if status is None else status
        peak = torch.empty(K, dtype=torch.int64, device=dev) if peak is None else peak
        latency = torch.empty(K, dtype=torch.float64, device=dev) if latency is None else latency
        _check(self._L.magis_eval_windows(self._h, K, _tptr(wstart), _tptr(wlen), _tptr(wperm),
                                          int(wperm.shape[1]), _tptr(status), _tptr(peak), _tptr(latency),
                                          _stream_ptr(stream)))
        return status, peak, latency

    def close(self):
        if getattr(self, "_h", None):
            self._L.magis_base_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def pareto_workspace_size(n: int) -> int:
    return int(lib().magis_pareto_workspace_size(int(n)))


def pareto_merge(peak, lat, status, ids=None, id_base: int = 0, cap: int = 4096,
                 mem_limit: int = -1, lat_limit: float = -1.0, workspace=None, out=None, stream=None):
    """Pareto front (ascending peak) + BetterThan-best ids, all on the device.
    Returns dict of device tensors: front_id, front_peak, front_lat [cap],
    front_n [1], best [2] (mem-limit mode, latency-limit mode)."""
    import torch
    n = int(peak.shape[0])
    dev = peak.device
    if out is None:
        out = {"front_id": torch.empty(cap, dtype=torch.int64, device=dev),
               "front_peak": torch.empty(cap, dtype=torch.int64, device=dev),
               "front_lat": torch.empty(cap, dtype=torch.float64, device=dev),
               "front_n": torch.empty(1, dtype=torch.int64, device=dev),
               "best": torch.empty(2, dtype=torch.int64, device=dev)}
    wsb = pareto_workspace_size(n)
    if workspace is None or workspace.numel() < wsb:
        workspace = torch.empty(max(wsb, 1), dtype=torch.uint8, device=dev)
    _check(lib().magis_pareto_merge(n, _tptr(peak), _tptr(lat), _tptr(status), _tptr(ids), int(id_base),
                                    int(cap), _tptr(out["front_id"]), _tptr(out["front_peak"]),
                                    _tptr(out["front_lat"]), _tptr(out["front_n"]), int(mem_limit),
                                    float(lat_limit), _tptr(out["best"]), _tptr(workspace),
                                    int(workspace.numel()), _stream_ptr(stream)))
    return out
