"""Cross-rank Pareto merge.

Candidates shard over ranks by contiguous global-id ranges; each rank scores
its shard and computes its local front with magis_pareto_merge; the padded
fronts (cap points of (id, peak, latency)) are all-gathered over the process
group (NCCL over NVLink on B200, gloo in the CPU tests) and every rank re-runs
the same deterministic merge, so all ranks hold the identical global front
and BetterThan-best ids (Alg. 3).  This is the path's only
exchange step.
"""
from __future__ import annotations

from typing import Callable, Dict, Optional

import torch
import torch.distributed as dist

from . import magis


def shard_range(K: int, rank: int, world: int):
    """Contiguous global-id range [lo, hi) of this rank."""
    return K * rank // world, K * (rank + 1) // world


class FrontCapacityError(RuntimeError):
    """Some rank's local front holds more points than the padded capacity, so
    the gathered fronts would silently miss points (magis_pareto_merge returned
    MAGIS_E_CAPACITY there and reported the size it needs)."""


def pack_front(front: Dict[str, torch.Tensor]) -> torch.Tensor:
    """One int64 record buffer [1 + 3 cap]: front_n, then cap ids, cap peaks
    and cap latencies (fp64 bit patterns), so a single all-gather moves it."""
    fid = front["front_id"].reshape(-1)
    cap = fid.numel()
    buf = torch.empty(1 + 3 * cap, dtype=torch.int64, device=fid.device)
    buf[0:1] = front["front_n"].reshape(-1)[:1].to(torch.int64)
    buf[1:1 + cap] = fid
    buf[1 + cap:1 + 2 * cap] = front["front_peak"].reshape(-1)
    buf[1 + 2 * cap:] = front["front_lat"].reshape(-1).contiguous().view(torch.int64)
    return buf


def gather_fronts(front: Dict[str, torch.Tensor], group=None) -> Dict[str, torch.Tensor]:
    """All-gather the padded local fronts (id, peak, lat; each [cap]) as one
    packed buffer (a single collective, 24 B per point + 8 B per rank), and
    check every rank's front size against the capacity: a front cut at cap
    would make the merged global front wrong, so it raises on every rank."""
    world = dist.get_world_size(group)
    t = pack_front(front)
    cap = (t.numel() - 1) // 3
    buf = torch.empty(world * t.numel(), dtype=torch.int64, device=t.device)
    dist.all_gather_into_tensor(buf, t, group=group)
    rec = buf.view(world, t.numel())
    sizes = rec[:, 0].cpu()
    if bool((sizes > cap).any()):
        raise FrontCapacityError(
            f"local front sizes {sizes.tolist()} exceed the capacity {cap}: re-run with cap >= {int(sizes.max())}")
    return {"front_id": rec[:, 1:1 + cap].reshape(-1),
            "front_peak": rec[:, 1 + cap:1 + 2 * cap].reshape(-1),
            "front_lat": rec[:, 1 + 2 * cap:].reshape(-1).view(torch.float64),
            "front_n": sizes}


def global_front(front: Dict[str, torch.Tensor], cap: int, mem_limit: int = -1,
                 lat_limit: float = -1.0, group=None,
                 merge: Optional[Callable] = None) -> Dict[str, torch.Tensor]:
    """Merge this rank's padded front with every other rank's.

    ``merge`` defaults to the device merge (magis_pareto_merge); the CPU gloo
    tests pass a host implementation with the same contract.  Raises
    FrontCapacityError (on every rank) if some local front exceeded its cap."""
    g = gather_fronts(front, group)
    merge = merge or (lambda peak, lat, ids, cap, M, L: magis.pareto_merge(
        peak, lat, None, ids=ids, cap=cap, mem_limit=M, lat_limit=L))
    return merge(g["front_peak"], g["front_lat"], g["front_id"], cap, mem_limit, lat_limit)


def global_filter(hashes: torch.Tensor, status: torch.Tensor, kmax: int, filt: Callable,
                  group=None) -> torch.Tensor:
    """Alg. 3 lines 10-12 across ranks (NEXT-2): each rank hashed its own
    contiguous shard of candidates; the (hash, status) pairs are all-gathered
    in rank order -- which is global candidate-id order -- padded to ``kmax``
    per rank with status 0xFF (ignored), and every rank runs the same filter
    over the gathered list, so every rank's seen-set X stays identical.
    ``filt(hashes, status) -> is_new`` is the caller's set (HashSet.filter on
    the device; a host stand-in in the CPU tests).  Returns this rank's slice
    of the new-flags."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    k = hashes.numel()
    h = torch.zeros(kmax, dtype=torch.int64, device=hashes.device)
    s = torch.full((kmax,), 0xFF, dtype=torch.uint8, device=status.device)
    h[:k] = hashes
    s[:k] = status
    hb = torch.empty(world * kmax, dtype=torch.int64, device=h.device)
    sb = torch.empty(world * kmax, dtype=torch.uint8, device=s.device)
    dist.all_gather_into_tensor(hb, h, group=group)
    dist.all_gather_into_tensor(sb, s, group=group)
    new = filt(hb, sb)
    return new[rank * kmax: rank * kmax + k]
