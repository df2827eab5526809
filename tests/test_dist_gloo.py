"""Multi-rank front merge over torch.distributed with the gloo
backend, world_size 2, on CPU.  The device merge (magis_pareto_merge) is
replaced by a host function with the same contract so the test runs without
a GPU; the plumbing under test -- shard ranges, padded fronts, the
all-gather, the identical result on every rank -- is the product code
(paper_conf_asplos_chend0zll024_b200.distributed)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_asplos_chend0zll024_b200 import distributed as pdist


def host_front(peak, lat, ids, cap, M=-1, L=-1.0):
    """Host stand-in for magis_pareto_merge (padding: id -1, peak -1, lat inf)."""
    peak = np.asarray(peak, np.int64)
    lat = np.asarray(lat, np.float64)
    ids = np.asarray(ids, np.int64)
    st = (ids < 0).astype(np.uint8)
    fr = oracle.pareto(peak, lat, st, ids)
    n = len(fr)
    out = {"front_id": torch.full((cap,), -1, dtype=torch.int64),
           "front_peak": torch.full((cap,), -1, dtype=torch.int64),
           "front_lat": torch.full((cap,), float("inf"), dtype=torch.float64),
           "front_n": torch.tensor([n], dtype=torch.int64),
           "best": torch.tensor([-1, -1], dtype=torch.int64)}
    k = min(n, cap)
    out["front_id"][:k] = torch.from_numpy(ids[fr[:k]])
    out["front_peak"][:k] = torch.from_numpy(peak[fr[:k]])
    out["front_lat"][:k] = torch.from_numpy(lat[fr[:k]])
    if n and M >= 0:
        out["best"][0] = int(ids[oracle.best_under_memory(peak, lat, st, M, ids)])
    if n and L >= 0:
        out["best"][1] = int(ids[oracle.best_under_latency(peak, lat, st, L, ids)])
    return out


def data(K, seed=0):
    rng = np.random.default_rng(seed)
    peak = rng.integers(0, 500, K).astype(np.int64)
    lat = rng.integers(0, 500, K).astype(np.float64)
    status = (rng.random(K) < 0.05).astype(np.uint8)
    return peak, lat, status


def _worker(rank, world, port, K, cap, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        peak, lat, status = data(K)
        lo, hi = pdist.shard_range(K, rank, world)
        ids = np.arange(lo, hi, dtype=np.int64)
        ids_valid = np.where(status[lo:hi] == 0, ids, -1)
        local = host_front(peak[lo:hi], lat[lo:hi], ids_valid, cap)
        g = pdist.global_front(local, cap, mem_limit=200, lat_limit=100.0,
                               merge=lambda p, l, i, c, M, L: host_front(p.numpy(), l.numpy(), i.numpy(), c, M, L))
        q.put((rank, int(g["front_n"][0]), g["front_id"].numpy().tolist(), g["best"].numpy().tolist()))
    finally:
        dist.destroy_process_group()


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("world", [2])
def test_gloo_merge_matches_single_rank(world):
    K, cap = 5000, 512
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, K, cap, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    peak, lat, status = data(K)
    single = host_front(peak, lat, np.where(status == 0, np.arange(K), -1), cap, 200, 100.0)
    exp_n = int(single["front_n"][0])
    exp_ids = single["front_id"].numpy().tolist()
    exp_best = single["best"].numpy().tolist()
    for rank, n, ids, best in res:
        assert n == exp_n
        assert ids == exp_ids            # identical on every rank, identical to 1 shard
        assert best == exp_best


def test_shard_ranges_cover_exactly():
    for K in (0, 1, 7, 65536):
        for world in (1, 2, 3, 8):
            r = [pdist.shard_range(K, i, world) for i in range(world)]
            assert r[0][0] == 0 and r[-1][1] == K
            assert all(r[i][1] == r[i + 1][0] for i in range(world - 1))


def _filter_worker(rank, world, port, K, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        rng = np.random.default_rng(9)
        X = set()

        def filt(hb, sb):
            nonlocal X
            new, X = oracle.hash_filter(hb.numpy().view(np.uint64), sb.numpy(), X)
            return torch.from_numpy(new)
        out = []
        for b in range(3):
            hv = rng.integers(0, 300, K).astype(np.uint64)
            st = ((rng.random(K) < 0.1) * 4).astype(np.uint8)
            lo, hi = pdist.shard_range(K, rank, world)
            kmax = max(pdist.shard_range(K, r, world)[1] - pdist.shard_range(K, r, world)[0] for r in range(world))
            new = pdist.global_filter(torch.from_numpy(hv[lo:hi].view(np.int64)), torch.from_numpy(st[lo:hi]),
                                      kmax, filt)
            out.append((lo, new.numpy().tolist()))
        q.put((rank, out, sorted(X)))
    finally:
        dist.destroy_process_group()


def test_gloo_hash_filter_matches_single_rank():
    """NEXT-2 across ranks: the gathered filter equals one filter over all
    candidates in id order, batch after batch, and every rank keeps the same X."""
    world, K = 2, 1001
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_filter_worker, args=(r, world, port, K, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    rng = np.random.default_rng(9)
    X = set()
    exp = []
    for b in range(3):
        hv = rng.integers(0, 300, K).astype(np.uint64)
        st = ((rng.random(K) < 0.1) * 4).astype(np.uint8)
        new, X = oracle.hash_filter(hv, st, X)
        exp.append(new)
    for rank, out, Xr in res:
        assert Xr == sorted(X)
        for b, (lo, new) in enumerate(out):
            assert new == exp[b][lo:lo + len(new)].tolist()


def _cap_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        cap = 8
        # rank 1's local front needed 11 points (magis_pareto_merge reports the
        # required size in front_n and returns MAGIS_E_CAPACITY)
        local = {"front_id": torch.arange(cap, dtype=torch.int64) + 100 * rank,
                 "front_peak": torch.arange(cap, dtype=torch.int64),
                 "front_lat": torch.arange(cap, 0, -1, dtype=torch.float64),
                 "front_n": torch.tensor([cap if rank == 0 else cap + 3], dtype=torch.int64)}
        try:
            pdist.global_front(local, cap, merge=lambda *a: None)
            q.put((rank, "no error"))
        except pdist.FrontCapacityError as e:
            q.put((rank, "raised" if "11" in str(e) else str(e)))
    finally:
        dist.destroy_process_group()


def test_gloo_front_over_capacity_raises_on_every_rank():
    """a local front cut at cap must not be merged silently; the
    packed all-gather carries every rank's front_n and all ranks raise."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=_cap_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(60)
        assert p.exitcode == 0
    assert res == {0: "raised", 1: "raised"}


def test_pack_front_roundtrip():
    cap = 5
    fr = {"front_id": torch.tensor([3, 1, 4, -1, -1]), "front_peak": torch.tensor([10, 20, 30, -1, -1]),
          "front_lat": torch.tensor([3.5, 2.25, 1e-300, float("inf"), float("inf")], dtype=torch.float64),
          "front_n": torch.tensor([3])}
    b = pdist.pack_front(fr)
    assert b.numel() == 1 + 3 * cap and int(b[0]) == 3
    assert torch.equal(b[1 + 2 * cap:].view(torch.float64), fr["front_lat"])
