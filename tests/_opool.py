"""Run the single-thread C oracle over chunks of a batch on several host
threads (ctypes releases the GIL during orc_eval_batch; the oracle graph is
read-only).  Test infrastructure only."""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np


def eval_parallel(o, perms, decs=None, nthreads: int | None = None):
    K = len(perms)
    nthreads = nthreads or max(1, min(os.cpu_count() or 1, 32))
    parts = [p for p in np.array_split(np.arange(K), nthreads * 4) if len(p)]
    with ThreadPoolExecutor(nthreads) as ex:
        res = list(ex.map(lambda p: o.eval_batch(perms[p[0]:p[-1] + 1],
                                                 None if decs is None else decs[p[0]:p[-1] + 1]), parts))
    return tuple(np.concatenate([r[i] for r in res]) if res else np.zeros(0) for i in range(3))
