"""Build libmagis.so (sm_100a) in-tree with nvcc.

    python -m paper_conf_asplos_chend0zll024_b200.build [--force]
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libmagis.so")
SOURCES = ["magis_graph.cu", "magis_eval.cu", "magis_eval2.cu", "magis_eval2_m0t1.cu", "magis_eval2_m0t2.cu",
           "magis_eval2_m1.cu", "magis_eval2_m2.cu", "magis_eval2_m3.cu", "magis_eval2_am.cu", "magis_evalb.cu", "magis_plan.cu", "magis_pareto.cu",
           "magis_gen.cu", "magis_window.cu", "magis_hotspot.cu", "magis_ghash.cu", "magis_hashset.cu"]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-Xcompiler", "-fvisibility=hidden",
         "--expt-relaxed-constexpr", "-Xptxas", "-v"] + os.environ.get("MAGIS_NVCC_EXTRA", "").split()


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(INCLUDE, "magis.h"), __file__]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src: str) -> tuple[str, str]:
    obj = os.path.join(CSRC, src.replace(".cu", ".o"))
    cmd = [NVCC, *ARCH, *FLAGS, "-I", INCLUDE, "-I", CSRC, "-DMAGIS_BUILD", "-c",
           os.path.join(CSRC, src), "-o", obj]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src}:\n{r.stdout}\n{r.stderr}")
    return obj, r.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not _stale():
        return LIB
    # recompile the objects older than their source or any header, in parallel
    headers = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    headers += [os.path.join(INCLUDE, "magis.h"), __file__]
    th = max(os.path.getmtime(h) for h in headers)
    todo = []
    for src in SOURCES:
        obj = os.path.join(CSRC, src.replace(".cu", ".o"))
        if force or not os.path.exists(obj) or os.path.getmtime(obj) < max(th, os.path.getmtime(os.path.join(CSRC, src))):
            todo.append(src)
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=max(1, min(len(todo), os.cpu_count() or 1))) as ex:
        for obj, err in ex.map(_compile, todo):
            if verbose:
                sys.stderr.write(err)
    objs = [os.path.join(CSRC, src.replace(".cu", ".o")) for src in SOURCES]
    tmp = LIB + ".tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc link failed:\n{r.stdout}\n{r.stderr}")
    os.replace(tmp, LIB)
    return LIB


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
