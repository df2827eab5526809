#!/usr/bin/env python
"""Benchmark: batched MAGIS schedule evaluation on B200 (BASELINE.json metric).

One step = one pass of the whole hot path over one batch of synthetic
candidates resident in HBM: magis_eval_schedules (inverse permutation ->
validity -> last use -> alloc/free events -> scan/max -> latency) + the local
Pareto front (magis_pareto_merge) + at N > 1 the all-gather of the fronts and
the global merge.  Default workload: C3 (BASELINE configs[2], BERT-large +
F-Trans, 262,144 candidates), strong scaling at fixed K: rank r scores the
global ids [r K / N, (r + 1) K / N).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl magis|reference]
    python bench.py --config c1      # brute force over every order of the C1 diamonds
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "candidate schedules evaluated/sec (op-steps/s) at 1/2/4/8 B200; % HBM roofline"
UNIT = "candidates/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c3",
                    help="c3 (default, BASELINE configs[2]), c1 (brute force), c2, c4, c5, c3f")
    ap.add_argument("--K", type=int, default=0,
                    help="candidates of the whole job (default: the config's K); split over the ranks")
    ap.add_argument("--seed", type=int, default=1)
    ap.add_argument("--cap", type=int, default=4096)
    ap.add_argument("--impl", default="magis", choices=["magis", "reference"])
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target oracle CPU-baseline wall time")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-wire", default="int32", choices=["int32", "delta4", "delta8", "u16"],
                    help="host schedule format of the e2e call: int32 (the ABI's schedule format, default); "
                         "the compact wires include their host-side encoding in the timed region")
    ap.add_argument("--ghash", action="store_true",
                    help="batched GraphHash + duplicate filter of the K candidates' graphs (NEXT-2)")
    ap.add_argument("--windows", action="store_true",
                    help="local-move candidates scored by windowed delta evaluation (NEXT-1); default config c5, K=1M")
    return ap.parse_args()


# ----------------------------------------------------------------- oracle pool --
_WL = None


def _pool_init(arrays):
    global _WL
    _WL = arrays


def _oracle_chunk(args):
    perms, decs = args
    import oracle
    size, cost, iso, src, dst, elig, U, B, lam, regions = _WL
    g = oracle.OracleGraph(size, cost, iso, src, dst, elig, U, B, lam, regions)
    t = time.perf_counter()
    st, pk, lt = g.eval_batch(perms, decs)
    return st, pk, lt, time.perf_counter() - t


def oracle_pool_eval(pool, perms, decs, ncores):
    parts = np.array_split(np.arange(len(perms)), ncores * 4)
    jobs = [(perms[p], decs[p]) for p in parts if len(p)]
    t = time.perf_counter()
    res = pool.map(_oracle_chunk, jobs)
    wall = time.perf_counter() - t
    st = np.concatenate([r[0] for r in res])
    pk = np.concatenate([r[1] for r in res])
    lt = np.concatenate([r[2] for r in res])
    return st, pk, lt, wall


# ------------------------------------------------------------------- clocks --
REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
           0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
           0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}


class ClockSampler:
    """SM clocks and throttle reasons sampled through NVML every ~2 ms while
    the timed region runs (nvidia-smi's >= 100 ms period is longer than a
    short timed region)."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.stop = threading.Event()
        self.h = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            idx = int(vis.split(",")[self.index]) if vis and vis.split(",")[0].isdigit() else self.index
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.nv = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self._sample()
            self.thr = threading.Thread(target=self._run, daemon=True)
            self.thr.start()
        except Exception:
            self.h = None
        return self

    def _sample(self):
        nv = self.nv
        sm = nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM)
        try:
            rs = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
        except Exception:
            rs = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
        self.rows.append((float(sm), float(self.max_mhz), int(rs)))

    def _run(self):
        while not self.stop.is_set():
            try:
                self._sample()
            except Exception:
                return
            time.sleep(0.002)

    def __exit__(self, *a):
        self.stop.set()
        if self.h is not None:
            self.thr.join(1.0)
            try:
                self._sample()
            except Exception:
                pass

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = statistics.median(r[0] for r in self.rows)
        mx = max(r[1] for r in self.rows)
        mask = 0
        for r in self.rows:
            mask |= r[2]
        reasons = [name for bit, name in REASONS.items() if mask & bit and name != "gpu_idle"]
        return {"sm_mhz": sm, "sm_max_mhz": mx, "reasons": reasons, "samples": len(self.rows),
                "source": "NVML during the timed region"}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json copy bandwidth)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


EVAL_SOURCES = ("magis_eval2_kernel.cuh", "magis_eval2.cu", "magis_plan.cu", "magis_internal.h")


def eval_src_sha() -> str:
    """Hash of the sources that determine the eval kernel's memory traffic."""
    import hashlib
    h = hashlib.sha256()
    for f in EVAL_SOURCES:
        with open(os.path.join(ROOT, "paper_conf_asplos_chend0zll024_b200", "csrc", f), "rb") as fh:
            h.update(fh.read())
    return h.hexdigest()[:16]


def ncu_traffic(config: str, K: int):
    """dram read+write bytes of one eval launch of K candidates, from the
    ncu --set full capture recorded in profiles/ncu_traffic.json -- only if
    it was captured from the current kernel sources (else None: stale)."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_traffic.json")) as f:
            e = json.load(f).get(config)
        if e and e.get("src_sha") == eval_src_sha():
            return int(round(e["bytes_per_candidate"] * K)), e.get("capture")
    except Exception:
        pass
    return None, "no ncu capture of the current eval sources"


# -------------------------------------------------------------------- main --
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.gpus != world and world > 1:
        print(f"warning: --gpus {args.gpus} != WORLD_SIZE {world}", file=sys.stderr)

    from magis_inputs import CONFIGS, CandidateGenerator, CandidateSpec, build_workload
    cfg = args.config.lower()
    if args.windows and "--config" not in " ".join(sys.argv):
        cfg = "c5"
    if cfg == "c1":
        return run_c1(args, rank, world, local)
    K_total = args.K or CONFIGS[cfg]["K"]
    if cfg == "c5" and not args.K:
        K_total = 65536    # C5's 1M local moves are evaluated in 16 chunks of 64k; one chunk per step
    # strong scaling: this rank scores the contiguous global ids [id0, id0 + K)
    id0, id1 = K_total * rank // world, K_total * (rank + 1) // world
    K = id1 - id0

    ncores = os.cpu_count() or 1
    pool = None
    need_pool = (args.impl == "reference" and rank == 0) or (
        args.impl == "magis" and rank == 0 and world == 1 and not args.no_cpu_baseline)
    wl = build_workload(cfg)
    if need_pool:
        import multiprocessing as mp
        arrays = (wl.size, wl.cost, wl.is_output, wl.src, wl.dst, wl.elig, wl.U, wl.swap_Bps, wl.swap_lat,
                  wl.regions)
        pool = mp.get_context("fork").Pool(ncores, initializer=_pool_init, initargs=(arrays,))

    workload = {"workload": f"{cfg}: {CONFIGS[cfg]['desc']}", "graph": wl.name, "n_nodes": wl.n,
                "n_edges": wl.n_edges, "R": wl.R, "n_total": wl.n_total, "K": K_total, "K_per_rank": K,
                "candidates": "75% random topo orders, 24% local moves (w<=64), 1% transposition; "
                              "P(remat)=P(swap)=5%", "seed": args.seed}
    if wl.F:
        workload["regions"] = wl.F
        workload["candidates"] = ("99% random topo orders of the chosen variants, 1% transposition; "
                                  "variant uniform per region; P(remat)=P(swap)=5%")

    if args.impl == "reference":
        return run_reference(args, wl, K, workload, pool, ncores, rank, world)
    if args.windows:
        if pool is not None:
            pool.close()
        return run_windows(args, wl, cfg, rank, world, local)
    if args.ghash:
        return run_ghash(args, wl, cfg, K, workload, pool, ncores, rank, world, local)

    import torch
    import torch.distributed as dist
    from paper_conf_asplos_chend0zll024_b200 import Graph, pareto_merge
    from paper_conf_asplos_chend0zll024_b200.distributed import global_front

    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)

    # --- inputs: generated (seeded, shard-independent) and made resident in HBM
    t0 = time.perf_counter()
    gen = CandidateGenerator(wl, CandidateSpec(seed=args.seed))
    Ph, Dh = gen.generate(id0, K)
    gen_s = time.perf_counter() - t0
    Ph_t = torch.from_numpy(Ph).pin_memory()
    Dh_t = torch.from_numpy(Dh).pin_memory()
    P = Ph_t.to(dev)
    D = Dh_t.to(dev)
    t0 = time.perf_counter()
    g = Graph.from_workload(wl, device=local)
    load_s = time.perf_counter() - t0
    R, NT = g.R, g.n_total
    # device candidate generator (§8(a) a1), timed separately from evaluation
    # (the F-Trans variant graphs of NEXT-4 are generated on the host only)
    gen_dev_ms, gen_match = None, None
    if wl.F == 0:
        Pg, Dg = g.generate_candidates(id0, K, seed=args.seed)               # warm-up / scratch allocation
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.generate_candidates(id0, K, seed=args.seed, perm=Pg, dec=Dg)
        e1.record()
        torch.cuda.synchronize()
        gen_dev_ms = e0.elapsed_time(e1)
        gen_match = bool(torch.equal(Pg, P) and (R == 0 or torch.equal(Dg[:, :R], D[:, :R])))
        del Pg, Dg
    stream = torch.cuda.current_stream()
    st = torch.empty(K, dtype=torch.uint8, device=dev)
    pk = torch.empty(K, dtype=torch.int64, device=dev)
    lt = torch.empty(K, dtype=torch.float64, device=dev)
    ws = torch.empty(max(1, __import__("paper_conf_asplos_chend0zll024_b200").pareto_workspace_size(max(K, world * args.cap, 1))),
                     dtype=torch.uint8, device=dev)
    mem_limit = int(wl.size.sum() // 8)

    def step(ev_pair=None):
        if ev_pair:
            ev_pair[0].record(stream)
        g.eval_schedules(P, D if g.dec_len else None, st, pk, lt, stream=stream)
        if ev_pair:
            ev_pair[1].record(stream)
        fr = pareto_merge(pk, lt, st, id_base=id0, cap=args.cap, mem_limit=mem_limit,
                          lat_limit=float(wl.cost.sum() * 1.05), workspace=ws, stream=stream)
        if world > 1:
            fr = global_front(fr, args.cap, mem_limit, float(wl.cost.sum() * 1.05))
        return fr

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(local)
    with clk:
        start.record(stream)
        for i in range(args.steps):
            fr = step(evs[i])
        end.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ms = start.elapsed_time(end)
    kern_ms = [a.elapsed_time(b) for a, b in evs]
    front_n = int(fr["front_n"].item())
    t = torch.tensor([ms, max(kern_ms), statistics.mean(kern_ms)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max, _, kern_avg = t.tolist()
    ms_per_step = ms_max / args.steps
    value = K_total / (ms_per_step / 1e3)

    # --- roofline of the dominant kernel (eval): algorithmic bytes per launch
    bytes_per_cand = 4 * NT + g.dec_len + 17
    alg_bytes = K * bytes_per_cand
    achieved = alg_bytes / (kern_avg / 1e3) / 1e9
    peak_gbs, peak_src = peaks()
    tr, tr_src = ncu_traffic(cfg, K)
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak_gbs, "unit": "GB/s",
            "frac": round(achieved / peak_gbs, 4), "traffic": tr, "traffic_source": tr_src, "peak_source": peak_src,
            "kernel": {0: "magis::eval_kernel<smem>", 1: "magis::eval_kernel<global>", 2: "magis::eval2_kernel",
                       3: "magis::evalb_kernel (2-CTA cluster per candidate)"}[g.info["variant"]],
            "alg_bytes_per_launch": alg_bytes,
            "bytes_per_candidate": bytes_per_cand, "kernel_ms_avg": round(kern_avg, 4),
            "kernel_share_of_step": round(kern_avg / ms_per_step, 4)}

    # --- end to end: the C-ABI host-buffer call (H2D perms+dec, eval, D2H results)
    e2e = None
    if not args.no_e2e:
        out_pinned = (torch.empty(K, dtype=torch.uint8).pin_memory(), torch.empty(K, dtype=torch.int64).pin_memory(),
                      torch.empty(K, dtype=torch.float64).pin_memory())
        # int32 schedules (the ABI's schedule format, magis_eval_schedules_host) by
        # default; a compact wire (delta4 / delta8 / u16, n_total <= 65535) is
        # encoded from the int32 schedules INSIDE the timed region
        wire = args.e2e_wire if NT <= 65535 else "int32"
        from paper_conf_asplos_chend0zll024_b200 import encode_delta4, encode_delta8

        def encode():
            if wire in ("delta4", "delta8"):
                enc = encode_delta4 if wire == "delta4" else encode_delta8
                return tuple(torch.from_numpy(a) for a in enc(Ph))
            if wire == "u16":
                return torch.from_numpy(Ph.astype(np.uint16))
            return Ph_t

        def e2e_step():
            w = encode()
            g.eval_schedules_host(w, Dh_t, out=out_pinned)
            return w

        Ph_w = e2e_step()                                  # warm (allocates staging once)
        wire_bytes = (sum(int(a.numel()) * a.element_size() for a in Ph_w) if isinstance(Ph_w, tuple)
                      else int(Ph_w.numel()) * Ph_w.element_size())
        if world > 1:
            dist.barrier()
        n_e2e = max(1, min(args.steps, 5))
        t0 = time.perf_counter()
        for _ in range(n_e2e):
            e2e_step()
        e2e_s = (time.perf_counter() - t0) / n_e2e
        te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        api = {"delta4": "magis_eval_schedules_host_delta4 (int32 schedules encoded to delta4 on the host "
                         "inside the timed region",
               "delta8": "magis_eval_schedules_host_delta8 (int32 schedules encoded to delta8 on the host "
                         "inside the timed region",
               "u16": "magis_eval_schedules_host_u16 (uint16 schedules, narrowed inside the timed region",
               "int32": "magis_eval_schedules_host (int32 schedules"}[wire]
        e2e = {"value": round(K_total / te.item(), 1), "unit": UNIT,
               "h2d_bytes_per_step": int(wire_bytes + K * g.dec_len), "d2h_bytes_per_step": int(K * 17),
               "api": api + ", pinned host buffers, chunked double-buffered copies)",
               "s_per_step": round(te.item(), 5)}
        ok_same = bool((out_pinned[1].numpy() == pk.cpu().numpy()).all())
        e2e["matches_device_path"] = ok_same

    # --- CPU baseline: the oracle, as it stands, on the host cores (rank 0, N=1)
    cpu = None
    if pool is not None:
        st_h, pk_h, lt_h = st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy()
        probe = 256
        _, _, _, w = oracle_pool_eval(pool, Ph[:probe], Dh[:probe], ncores)
        rate = probe / max(w, 1e-6)
        S = int(min(K, max(probe, rate * args.cpu_seconds)))
        rs, rp, rl, wall = oracle_pool_eval(pool, Ph[:S], Dh[:S], ncores)
        okm = rs == 0
        parity = bool((rs == st_h[:S]).all() and (rp == pk_h[:S]).all() and
                      np.all(np.abs(rl[okm] - lt_h[:S][okm]) <= 1e-9 * np.abs(rl[okm])))
        cpu = {"value": round(S / wall, 1), "unit": UNIT, "cores": ncores, "kind": "oracle",
               "sample": f"first {S} of the {K} candidates (single-thread C oracle per process, "
                         f"{ncores} processes), {wall:.1f} s",
               "op_steps_per_s": round(S / wall * NT, 1), "parity_on_sample": parity}
        pool.close()

    if rank == 0:
        gpu_launches = args.steps * (1 + 6 + (6 if world > 1 else 0))
        line = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
                "op_steps_per_s": round(value * NT, 1),
                "config": {**workload, "parallelism": f"candidate-dp{world}",
                           "l2": f"inputs larger than L2 ({K * NT * 4 / 1e9:.2f} GB of perms per rank)",
                           "front_cap": args.cap, "front_n": front_n},
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": clk.summary(),
                "gpu_launches": gpu_launches,
                "setup": {"candidate_gen_s": round(gen_s, 3), "graph_load_s": round(load_s, 3),
                          "device_gen_ms": round(gen_dev_ms, 3) if gen_dev_ms else None,
                          "device_gen_cand_per_s": round(K / (gen_dev_ms / 1e3), 1) if gen_dev_ms else None,
                          "device_gen_matches_host": gen_match,
                          "eval_variant": g.info["variant"], "grid": g.info["grid"], "block": g.info["block"],
                          "smem_bytes": g.info["smem_bytes"]}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


C1_SHAPES = ([4, 4], [3, 3, 2], [2, 2, 2, 2], [2, 2, 2, 1, 1])


def run_c1(args, rank, world, local):
    """BASELINE configs[0]: 10-op diamonds (source -> parallel chains -> sink,
    sizes 512 B x U[1, 2^20)), 256 random topological orders each, against the
    brute force over ALL topological orders (a schedule is any
    topological order).  CPU leg: the oracle enumerates and scores every
    order (single thread), its seconds are the baseline.  GPU leg (the timed
    step): magis_eval_schedules over every order of the four diamonds plus
    the 256 random orders, and magis_pareto_merge per set (its first front
    point is the minimum peak).  Parity on every order; the brute-force
    minimum must match.  Replicas only at N > 1 (the sets are tiny)."""
    import torch
    import oracle
    from magis_inputs import CandidateGenerator, CandidateSpec, models
    from magis_inputs.enumerate import topo_orders
    from paper_conf_asplos_chend0zll024_b200 import Graph, pareto_merge
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    wls = [models.diamond(br, seed=args.seed) for br in C1_SHAPES]
    # --- CPU brute force: enumerate every order, score it with the oracle
    cpu_rows, ref = [], []
    t_all = time.perf_counter()
    for br, wl in zip(C1_SHAPES, wls):
        t0 = time.perf_counter()
        orders = topo_orders(wl.n, wl.src, wl.dst)
        t1 = time.perf_counter()
        o = oracle.OracleGraph.from_workload(wl)
        rs, rp, rl = o.eval_batch(orders)
        t2 = time.perf_counter()
        ref.append((orders, rs, rp, rl))
        cpu_rows.append({"shape": br, "orders": int(len(orders)), "enumerate_s": round(t1 - t0, 5),
                         "oracle_s": round(t2 - t1, 5), "min_peak": int(rp.min()), "max_peak": int(rp.max())})
    cpu_s = time.perf_counter() - t_all
    # --- 256 random orders per diamond (random-priority Kahn, the C1 recipe)
    rnd = [CandidateGenerator(wl, CandidateSpec(seed=args.seed, pct_random=100, pct_local=0)).generate(0, 256)[0]
           for wl in wls]
    gs = [Graph.from_workload(wl, device=local) for wl in wls]
    sets = [torch.from_numpy(np.concatenate([r[0], q])).to(dev) for r, q in zip(ref, rnd)]
    outs = [(torch.empty(len(x), dtype=torch.uint8, device=dev), torch.empty(len(x), dtype=torch.int64, device=dev),
             torch.empty(len(x), dtype=torch.float64, device=dev)) for x in sets]
    stream = torch.cuda.current_stream()
    wss = [torch.empty(max(1, __import__("paper_conf_asplos_chend0zll024_b200").pareto_workspace_size(len(x))),
                       dtype=torch.uint8, device=dev) for x in sets]

    def step():
        frs = []
        for g, x, (st, pk, lt), ws in zip(gs, sets, outs, wss):
            g.eval_schedules(x, None, st, pk, lt, stream=stream)
            frs.append(pareto_merge(pk, lt, st, cap=64, workspace=ws, stream=stream))
        return frs

    for _ in range(max(args.warmup, 3)):
        step()
    torch.cuda.synchronize()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(local)
    with clk:
        start.record(stream)
        for _ in range(args.steps):
            frs = step()
        end.record(stream)
        torch.cuda.synchronize()
    ms = start.elapsed_time(end) / args.steps
    n_all = sum(len(x) for x in sets)
    # parity on every order + the brute-force minimum
    parity, rows = True, []
    for (orders, rs, rp, rl), q, (st, pk, lt), fr, wl, crow in zip(ref, rnd, outs, frs, wls, cpu_rows):
        n = len(orders)
        st_h, pk_h, lt_h = st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy()
        ok = rs == 0
        parity &= bool((st_h[:n] == rs).all() and (pk_h[:n] == rp).all() and
                       np.all(np.abs(lt_h[:n][ok] - rl[ok]) <= 1e-9 * np.abs(rl[ok])))
        qs, qp, _ = oracle.OracleGraph.from_workload(wl).eval_batch(q)
        parity &= bool((st_h[n:] == qs).all() and (pk_h[n:] == qp).all())
        gmin = int(fr["front_peak"][0].item())
        parity &= gmin == crow["min_peak"] == int(pk_h.min())
        rows.append({**crow, "gpu_min_peak": gmin, "random256_best_peak": int(qp.min()),
                     "random256_gap": round(float(qp.min()) / crow["min_peak"] - 1.0, 4)})
    # e2e: host orders through the host-buffer call, results back
    hsets = [x.cpu() for x in sets]
    t0 = time.perf_counter()
    for _ in range(max(1, min(args.steps, 5))):
        for g, x in zip(gs, hsets):
            g.eval_schedules_host(x)
    e2e_s = (time.perf_counter() - t0) / max(1, min(args.steps, 5))
    peak_gbs, peak_src = peaks()
    bpc = 4 * 10 + 17
    if rank == 0:
        line = {"metric": METRIC, "value": round(n_all / (ms / 1e3), 1), "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4), "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
                "config": {"workload": "c1: 10-op diamonds, every topological order + 256 random orders each "
                                       "(brute force vs GPU)", "shapes": [list(b) for b in C1_SHAPES],
                           "candidates_per_step": n_all, "seed": args.seed, "parallelism": f"replicas{world}",
                           "l2": "inputs in L2 (tiny)"},
                "brute_force": {"cpu_s": round(cpu_s, 4), "gpu_s": round(ms / 1e3, 6),
                                "cpu_over_gpu": round(cpu_s / (ms / 1e3), 1), "shapes": rows,
                                "parity_on_every_order": parity},
                "roofline": {"bound": "hbm", "achieved": round(n_all * bpc / (ms / 1e3) / 1e9, 3), "peak": peak_gbs,
                             "unit": "GB/s", "frac": round(n_all * bpc / (ms / 1e3) / 1e9 / peak_gbs, 6),
                             "traffic": None, "peak_source": peak_src,
                             "note": "launch-latency bound: 8 launches over 8.8k tiny schedules"},
                "cpu_baseline": {"value": round(sum(r["orders"] for r in rows) / cpu_s, 1), "unit": UNIT, "cores": 1,
                                 "kind": "oracle", "sample": "every topological order of the four diamonds, "
                                 "enumerated and scored by the single-thread oracle", "parity_on_sample": parity},
                "e2e": {"value": round(n_all / e2e_s, 1), "unit": UNIT, "h2d_bytes_per_step": int(n_all * 40),
                        "d2h_bytes_per_step": int(n_all * 17), "api": "magis_eval_schedules_host (int32 schedules)",
                        "s_per_step": round(e2e_s, 6)},
                "clocks": clk.summary(), "gpu_launches": args.steps * len(sets) * 7}
        print(json.dumps(line), flush=True)


def run_windows(args, wl, cfg, rank, world, local):
    """Local-move sweep (SURVEY config 5, NEXT-1): a base schedule with swaps,
    K window candidates (w <= 64) scored by magis_eval_windows; local fronts
    merged across ranks like the full path."""
    import torch
    import torch.distributed as dist
    from magis_inputs import CandidateGenerator, CandidateSpec, WindowGenerator
    from paper_conf_asplos_chend0zll024_b200 import Base, Graph, pareto_merge
    from paper_conf_asplos_chend0zll024_b200.distributed import global_front
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    K = args.K or 1 << 20
    g = Graph.from_workload(wl, device=local)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=args.seed)).generate(0, 64)
    Pd, Dd = torch.from_numpy(P).to(dev), torch.from_numpy(D).to(dev)
    st, pk, lt = g.eval_schedules(Pd, Dd if wl.R else None)
    st = st.cpu().numpy()
    ok = np.nonzero((st == 0) & (D[:, :max(wl.R, 1)] == 2).any(axis=1))[0]
    bi = int(ok[0]) if len(ok) else int(np.argmax(st == 0))
    base = Base(g, Pd[bi].contiguous(), Dd[bi].contiguous() if wl.R else None)
    t0 = time.perf_counter()
    wg = WindowGenerator(wl, P[bi], D[bi], seed=args.seed + 1)
    ws, wln, wp = wg.generate(rank * K, K)
    gen_s = time.perf_counter() - t0
    wsd, wld, wpd = (torch.from_numpy(a).to(dev) for a in (ws, wln, wp))
    st = torch.empty(K, dtype=torch.uint8, device=dev)
    pk = torch.empty(K, dtype=torch.int64, device=dev)
    lt = torch.empty(K, dtype=torch.float64, device=dev)
    stream = torch.cuda.current_stream()

    def step(evp=None):
        if evp:
            evp[0].record(stream)
        base.eval_windows(wsd, wld, wpd, st, pk, lt, stream=stream)
        if evp:
            evp[1].record(stream)
        fr = pareto_merge(pk, lt, st, id_base=rank * K, cap=args.cap, stream=stream)
        if world > 1:
            fr = global_front(fr, args.cap)
        return fr

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(local)
    with clk:
        start.record(stream)
        for i in range(args.steps):
            fr = step(evs[i])
        end.record(stream)
        torch.cuda.synchronize()
    t = torch.tensor([start.elapsed_time(end), statistics.mean(a.elapsed_time(b) for a, b in evs)],
                     dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms, kern = t.tolist()
    ms_per_step = ms / args.steps
    value = world * K / (ms_per_step / 1e3)
    bytes_per_cand = 4 + 4 + 4 * wg.wmax + 17
    achieved = K * bytes_per_cand / (kern / 1e3) / 1e9
    peak_gbs, peak_src = peaks()
    if rank == 0:
        line = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
                "op_steps_per_s": round(value * wl.n_total, 1),
                "window_steps_per_s": round(world * float(wln.sum()) / (ms_per_step / 1e3), 1),
                "config": {"workload": f"{cfg} local-move sweep: {K} windows (w <= {wg.wmax}) over one base schedule, "
                                       "windowed delta evaluation (NEXT-1)", "graph": wl.name, "n_total": wl.n_total,
                           "K_per_rank": K, "mean_window": round(float(wln.mean()), 2),
                           "base_peak_latency": list(base.info()[1:]), "parallelism": f"candidate-dp{world}",
                           "front_n": int(fr["front_n"].item())},
                "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak_gbs, "unit": "GB/s",
                             "frac": round(achieved / peak_gbs, 4), "traffic": None, "peak_source": peak_src,
                             "kernel": "magis::window_kernel", "bytes_per_candidate": bytes_per_cand,
                             "kernel_ms_avg": round(kern, 4)},
                "cpu_baseline": None, "e2e": None, "clocks": clk.summary(), "gpu_launches": args.steps * 7,
                "setup": {"window_gen_s": round(gen_s, 3)}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def _oracle_hash_chunk(args):
    decs, labels = args
    import oracle
    size, cost, iso, src, dst, elig, U, B, lam, regions = _WL
    g = oracle.OracleGraph(size, cost, iso, src, dst, elig, U, B, lam, regions)
    t = time.perf_counter()
    st, hs = g.graph_hash_batch(labels, decs)
    return st, hs, time.perf_counter() - t


def ghash_words(wl, D):
    """Words absorbed by hash() per candidate (algorithmic work of Alg. 3
    line 5-6): per active node 1 + |pre(v)|, plus 1 for line 6."""
    indeg = np.bincount(np.unique(wl.src.astype(np.int64) * wl.n + wl.dst) % wl.n, minlength=wl.n)
    w0 = int((1 + indeg).sum()) + 1
    if wl.R == 0:
        return float(w0)
    extra_remat = 1 + indeg[wl.elig]                  # clone: 1 + |pre(t_r)|
    Dv = D[:, :wl.R]
    per = w0 + (Dv == 1).astype(np.int64) @ extra_remat + 4 * (Dv == 2).sum(axis=1)   # Store 2 + Load 2
    return float(per.mean())


def run_ghash(args, wl, cfg, K, workload, pool, ncores, rank, world, local):
    """NEXT-2: one step = magis_graph_hash over the K candidates' decision
    vectors (the transformed graphs) + the hash-set filter (Alg. 3 lines
    10-12) into a set cleared at the start of the step."""
    import torch
    import torch.distributed as dist
    from magis_inputs import CandidateGenerator, CandidateSpec
    from magis_inputs.labels import node_labels
    from paper_conf_asplos_chend0zll024_b200 import Graph, GraphHasher, HashSet
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    labels = node_labels(wl)
    _, Dh = CandidateGenerator(wl, CandidateSpec(seed=args.seed)).generate(rank * K, K)
    Dh = np.ascontiguousarray(Dh[:, :max(wl.R, 1)])
    Dh_t = torch.from_numpy(Dh).pin_memory()
    D = Dh_t.to(dev)
    g = Graph.from_workload(wl, device=local)
    hz = GraphHasher(g, labels)
    hs = HashSet(max(2 * K * world, 1024), device=local)
    from paper_conf_asplos_chend0zll024_b200.distributed import global_filter
    st = torch.empty(K, dtype=torch.uint8, device=dev)
    hv = torch.empty(K, dtype=torch.int64, device=dev)
    new = torch.empty(K, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def step(evp=None):
        hs.clear(stream=stream)
        if evp:
            evp[0].record(stream)
        hz.hash(D if wl.R else K, status=st, out=hv, stream=stream)
        if evp:
            evp[1].record(stream)
        if world > 1:      # the seen-set X is global: all-gather (hash, status), filter in id order
            new.copy_(global_filter(hv, st, K, lambda hb, sb: hs.filter(hb, sb, stream=stream)))
        else:
            hs.filter(hv, st, out=new, stream=stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clk = ClockSampler(local)
    with clk:
        start.record(stream)
        for i in range(args.steps):
            step(evs[i])
        end.record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t = torch.tensor([start.elapsed_time(end), statistics.mean(a.elapsed_time(b) for a, b in evs)],
                     dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms, kern = t.tolist()
    ms_per_step = ms / args.steps
    value = world * K / (ms_per_step / 1e3)
    n_new = int(new.sum().item())
    # roofline: ALU-pipe bound (DESIGN.md §6 GraphHash): one absorbed word =
    # h ^ w + mix64 = 12.5 ALU-pipe (LOP3/SHF) + 8 FMA-pipe (IMAD) SASS ops (cuobjdump); ALU pipe 16 lanes/clk/SMSP
    words = ghash_words(wl, Dh)
    sms = torch.cuda.get_device_properties(dev).multi_processor_count
    clk_mhz = (clk.summary() or {}).get("sm_mhz") or 1965.0
    peak_words = sms * 4 * 16 * clk_mhz * 1e6 / 12.5
    achieved = K * words / (kern / 1e3)
    # e2e: decisions H2D from pinned memory, hash + filter, results D2H
    hst = torch.empty(K, dtype=torch.uint8).pin_memory()
    hnew = torch.empty(K, dtype=torch.uint8).pin_memory()
    hhash = torch.empty(K, dtype=torch.int64).pin_memory()
    Dd = torch.empty_like(D)

    def e2e_step():
        Dd.copy_(Dh_t, non_blocking=True)
        hs.clear(stream=stream)
        hz.hash(Dd if wl.R else K, status=st, out=hv, stream=stream)
        hs.filter(hv, st, out=new, stream=stream)
        hst.copy_(st, non_blocking=True)
        hhash.copy_(hv, non_blocking=True)
        hnew.copy_(new, non_blocking=True)
        torch.cuda.synchronize()
    e2e_step()
    n_e2e = max(1, min(args.steps, 5))
    t0 = time.perf_counter()
    for _ in range(n_e2e):
        e2e_step()
    e2e_s = (time.perf_counter() - t0) / n_e2e
    te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e = {"value": round(world * K / te.item(), 1), "unit": UNIT, "h2d_bytes_per_step": int(Dh.nbytes),
           "d2h_bytes_per_step": int(K * 10), "api": "GraphHasher.hash + HashSet.filter (magis_graph_hash, "
           "magis_hashset_filter) with pinned host decisions / results", "s_per_step": round(te.item(), 5)}
    cpu = None
    if pool is not None:
        hh = hv.cpu().numpy().view(np.uint64)
        sth = st.cpu().numpy()
        probe = 64
        S = probe
        parts = np.array_split(np.arange(probe), ncores)
        t0 = time.perf_counter()
        pool.map(_oracle_hash_chunk, [(Dh[p], labels) for p in parts if len(p)])
        rate = probe / max(time.perf_counter() - t0, 1e-6)
        S = int(min(K, max(probe, rate * args.cpu_seconds)))
        parts = np.array_split(np.arange(S), ncores * 4)
        t0 = time.perf_counter()
        res = pool.map(_oracle_hash_chunk, [(Dh[p], labels) for p in parts if len(p)])
        wall = time.perf_counter() - t0
        rs = np.concatenate([r[0] for r in res])
        rh = np.concatenate([r[1] for r in res])
        cpu = {"value": round(S / wall, 1), "unit": UNIT, "cores": ncores, "kind": "oracle",
               "sample": f"first {S} of the {K} candidates' graphs hashed (single-thread C oracle per process, "
                         f"{ncores} processes), {wall:.1f} s",
               "parity_on_sample": bool((rs == sth[:S]).all() and (rh == hh[:S]).all())}
        pool.close()
    if rank == 0:
        line = {"metric": "candidate graphs hashed + filtered/sec (GraphHash, Alg. 3 lines 3-6, 10-12)",
                "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4), "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
                "config": {**workload, "workload": f"{cfg}: GraphHash of {K} candidate graphs (decisions of the "
                           "bench candidates) + duplicate filter (NEXT-2)", "parallelism": f"candidate-dp{world}",
                           "new_graphs": n_new, "words_per_candidate": round(words, 1), "ghash": hz.info,
                           "l2": "decisions stream once (K x R bytes); value slots L2-resident"},
                "roofline": {"bound": "alu", "achieved": round(achieved / 1e9, 2), "peak": round(peak_words / 1e9, 1),
                             "unit": "Gword/s", "frac": round(achieved / peak_words, 4), "traffic": None,
                             "peak_source": "derived: SMs x 4 SMSP x 16 ALU lanes/clk (B300_MICROARCH rt_SMSP=2) x "
                                            "SM clock / 12.5 ALU-pipe ops per absorbed word (SASS count)",
                             "kernel": "magis::ghash_kernel", "kernel_ms_avg": round(kern, 4),
                             "kernel_share_of_step": round(kern / ms_per_step, 4)},
                "cpu_baseline": cpu, "e2e": e2e, "clocks": clk.summary(), "gpu_launches": args.steps * 3}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def run_reference(args, wl, K, workload, pool, ncores, rank, world):
    """--impl reference: the oracle (plain single-thread C per process) timed
    as it stands on the host cores, rank 0 only, on bounded samples."""
    if rank != 0:
        return
    from magis_inputs import CandidateGenerator, CandidateSpec
    import oracle
    gen = CandidateGenerator(wl, CandidateSpec(seed=args.seed))
    S = 2048
    Ph, Dh = gen.generate(0, S)
    for _ in range(args.warmup):
        oracle_pool_eval(pool, Ph[:256], Dh[:256], ncores)
    walls = []
    for _ in range(args.steps):
        st, pk, lt, w = oracle_pool_eval(pool, Ph, Dh, ncores)
        t0 = time.perf_counter()
        oracle.pareto(pk, lt, st)
        walls.append(w + time.perf_counter() - t0)
    pool.close()
    s = statistics.mean(walls)
    value = S / s
    line = {"metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(s * 1e3, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int64", "data": "synthetic", "impl": "reference",
            "op_steps_per_s": round(value * wl.n_total, 1),
            "config": {**workload, "parallelism": "cpu"},
            "cpu_baseline": {"value": round(value, 1), "unit": UNIT, "cores": ncores, "kind": "oracle",
                             "sample": f"{S} candidates per step (first {S} of the workload), {ncores} processes"},
            "e2e": {"value": round(value, 1), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
