"""B200-native batched schedule evaluation for MAGIS (ASPLOS '24).

The hot path -- inverse permutation, validity, last use, alloc/free events,
scan/max and the latency model -- runs in hand-written sm_100a kernels behind
the C ABI in include/magis.h (libmagis.so).  This package is the thin Python
binding (magis.py) plus the multi-GPU front merge over torch.distributed
(distributed.py).  PyTorch is used only for device memory, streams and
process groups.
"""
from .magis import (Base, Graph, GraphHasher, HashSet, MagisError, encode_delta4, encode_delta8, pareto_merge, pareto_workspace_size, lib, ST_NOT_PERM,
                    ST_EDGE, ST_BAD_DEC)

__all__ = ["Base", "Graph", "GraphHasher", "HashSet", "MagisError", "encode_delta4", "encode_delta8", "pareto_merge", "pareto_workspace_size", "lib", "ST_NOT_PERM",
           "ST_EDGE", "ST_BAD_DEC"]
