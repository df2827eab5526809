"""The C-ABI library loads and exports every symbol include/magis.h declares;
host-side argument checking works without a GPU (no compute calls here)."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_asplos_chend0zll024_b200 as pkg
from paper_conf_asplos_chend0zll024_b200 import magis

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "magis.h")


def declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(magis_[a-z_0-9]+)\s*\(", src)))


@pytest.fixture(scope="module")
def lib():
    from paper_conf_asplos_chend0zll024_b200 import build
    build.build()
    return magis.lib()


def test_header_declares_the_boundary():
    names = declared()
    for must in ("magis_graph_load", "magis_eval_schedules", "magis_pareto_merge"):
        assert must in names
    assert sorted(magis.EXPORTS) == names


def test_every_declared_symbol_is_exported(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", magis.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (magis_\w+)", out))
    for name in declared():
        assert name in exported, name
        assert getattr(lib, name) is not None
    # nothing else leaks (hidden visibility)
    assert exported == set(declared())


def test_abi_version_and_no_device_here(lib):
    assert lib.magis_abi_version() == 2
    import torch
    if not torch.cuda.is_available():
        assert lib.magis_device_supported(0) == 0


def test_pareto_workspace_size(lib):
    assert lib.magis_pareto_workspace_size(0) >= 0
    a = lib.magis_pareto_workspace_size(4096)
    b = lib.magis_pareto_workspace_size(4097)
    assert b > a > 0


def test_argument_errors_without_gpu(lib):
    # null desc / out
    h = ctypes.c_void_p()
    assert lib.magis_graph_load(None, 0, ctypes.byref(h)) == -1
    assert lib.magis_eval_schedules(None, 1, None, None, None, None, None, None) == -1
    assert b"NULL" in lib.magis_last_error()
    # negative n
    assert lib.magis_pareto_merge(-1, None, None, None, None, 0, 0, None, None, None, None, -1, -1.0,
                                  None, None, 0, None) == -1


def _desc(n, size, cost, iso, src, dst, elig=(), U=()):
    keep = []

    def arr(x, dt):
        a = np.ascontiguousarray(x, dt)
        keep.append(a)
        return a.ctypes.data_as(ctypes.c_void_p) if a.size else None
    ptr = np.zeros(len(U) + 1, np.int64)
    for i, u in enumerate(U):
        ptr[i + 1] = ptr[i] + len(u)
    keep.append(ptr)
    idx = np.concatenate([np.asarray(u, np.int32) for u in U]) if U else np.zeros(0, np.int32)
    d = magis.GraphDesc(n, arr(size, np.int64), arr(cost, np.float64), arr(iso, np.uint8), len(src),
                        arr(src, np.int32), arr(dst, np.int32), len(elig), arr(elig, np.int32),
                        ptr.ctypes.data_as(ctypes.c_void_p), arr(idx, np.int32), 25e9, 1e-5)
    return d, keep


@pytest.mark.parametrize("case,code", [
    (dict(size=[-1, 1, 1]), -1),                    # negative size
    (dict(cost=[0.0, float("nan"), 0.0]), -1),      # non-finite cost
    (dict(src=[0, 1], dst=[1, 1]), -1),             # self loop
    (dict(src=[0, 5], dst=[1, 2]), -1),             # id out of range
    (dict(src=[0, 1, 2], dst=[1, 2, 0]), -2),       # cycle
    (dict(elig=[2], U=[[1]]), -1),                  # output marked eligible / U not in cons
    (dict(elig=[0], U=[[2]]), -1),                  # U_r not a subset of cons(t_r)
    (dict(elig=[0], U=[[]]), -1),                   # empty U_r
])
def test_loader_validation_without_gpu(lib, case, code):
    """Graph validation runs on the host before any device work."""
    base = dict(size=[1, 1, 1], cost=[0.0, 0.0, 0.0], iso=[0, 0, 1], src=[0, 1], dst=[1, 2], elig=(), U=())
    base.update(case)
    d, keep = _desc(3, base["size"], base["cost"], base["iso"], base["src"], base["dst"], base["elig"],
                    base["U"])
    h = ctypes.c_void_p()
    rc = lib.magis_graph_load(ctypes.byref(d), 0, ctypes.byref(h))
    assert rc == code, lib.magis_last_error()
    assert not h.value


def test_valid_graph_needs_b200(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    d, keep = _desc(3, [1, 1, 1], [0.0] * 3, [0, 0, 1], [0, 1], [1, 2])
    h = ctypes.c_void_p()
    assert lib.magis_graph_load(ctypes.byref(d), 0, ctypes.byref(h)) == -5   # no CPU fallback
    with pytest.raises(magis.MagisError):
        magis.Graph([1, 1, 1], [0.0] * 3, [0, 0, 1], [0, 1], [1, 2])


@pytest.mark.parametrize("reg,elig,U,code", [
    (dict(nv=[5], nr=[-1, 0, -1, -1], vn=[0, 0, 0, 0]), (), (), -1),       # n_variants > 4
    (dict(nv=[2], nr=[-1, 0, -1, -1], vn=[0, 2, 0, 0]), (), (), -1),       # variant out of range
    (dict(nv=[2], nr=[-1, 3, -1, -1], vn=[0, 0, 0, 0]), (), (), -1),       # region out of range
    (dict(nv=[2], nr=[-1, 0, 0, -1], vn=[0, 0, 1, 0]), (), (), -1),        # edge between two variants
    (dict(nv=[2], nr=[-1, 0, -1, -1], vn=[0, 0, 0, 0]), [1], [[2]], -1),   # eligible inside a region
    (dict(nv=[2], nr=[-1, 0, -1, -1], vn=[0, 0, 0, 0]), [2], [[3]], -1),   # eligible reads a region
    (dict(nv=[2], nr=[-1, -1, 0, -1], vn=[0, 0, 0, 0]), [1], [[2]], -1),   # late user inside a region
    (dict(nv=[2], nr=[-1, 0, -1, -1], vn=[0, 0, 0, 0]), (), (), -5),       # valid: needs the B200
])
def test_region_validation_without_gpu(lib, reg, elig, U, code):
    """F-Trans variant regions (NEXT-4, reading F1) are validated on the host."""
    import torch
    if torch.cuda.is_available() and code == -5:
        pytest.skip("GPU present")
    # chain 0 -> 1 -> 2 -> 3 plus 1 -> 3
    d, keep = _desc(4, [4, 4, 4, 4], [0.0, 1.0, 1.0, 1.0], [0, 0, 0, 1], [0, 1, 2, 1], [1, 2, 3, 3], elig, U)
    nv = np.asarray(reg["nv"], np.int32)
    nr = np.asarray(reg["nr"], np.int32)
    vn = np.asarray(reg["vn"], np.uint8)
    rd = magis.RegionDesc(len(nv), nv.ctypes.data_as(ctypes.c_void_p), nr.ctypes.data_as(ctypes.c_void_p),
                          vn.ctypes.data_as(ctypes.c_void_p))
    h = ctypes.c_void_p()
    rc = lib.magis_graph_load_regions(ctypes.byref(d), ctypes.byref(rd), 0, ctypes.byref(h))
    assert rc == code, lib.magis_last_error()
