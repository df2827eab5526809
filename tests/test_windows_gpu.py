"""Windowed delta evaluation (NEXT-1, Alg. 2 P:1591-1613 applied to scoring)
against the oracle on the expanded schedules, and against the full GPU
evaluation of the same schedules."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from magis_inputs import CandidateGenerator, CandidateSpec, WindowGenerator, build_workload  # noqa: E402
from magis_inputs.graph import Workload  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Base, Graph  # noqa: E402
from tests.test_oracle_pins import random_case, random_valid_perm  # noqa: E402
from tests.test_parity_gpu import DEV, assert_parity, gpu_eval  # noqa: E402


def run_windows(g, base_perm, base_dec, ws, wln, wp):
    t = lambda a, dt=np.int32: torch.from_numpy(np.ascontiguousarray(a, dt)).to(DEV)
    b = Base(g, t(base_perm), t(base_dec, np.uint8) if g.R else None)
    st, pk, lt = b.eval_windows(t(ws), t(wln), t(wp))
    torch.cuda.synchronize()
    return b, (st.cpu().numpy(), pk.cpu().numpy(), lt.cpu().numpy())


@pytest.mark.parametrize("cfg", ["c2", "c5"])
def test_windows_match_oracle(cfg):
    wl = build_workload(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=4)).generate(0, 32)
    o = OracleGraph.from_workload(wl)
    st, pk, lt = o.eval_batch(P, D)
    i = int(np.argmax((st == 0) & (D == 2).any(axis=1)))      # a valid base with swaps
    wg = WindowGenerator(wl, P[i], D[i], seed=9, pct_bad=2)
    ws, wln, wp = wg.generate(0, 3000)
    g = Graph.from_workload(wl)
    b, res = run_windows(g, P[i], D[i], ws, wln, wp)
    assert b.info()[:2] == (0, int(pk[i]))
    assert abs(b.info()[2] - lt[i]) <= 1e-9 * lt[i]
    E = wg.expand(ws, wln, wp)
    Dk = np.repeat(D[i][None], len(ws), axis=0)
    ref = o.eval_batch(E, Dk)
    assert_parity(*res, *ref)
    assert (ref[0] == 0).mean() > 0.9 and (ref[0] == 2).any()
    # and equal to the full GPU evaluation of the expanded schedules
    full = gpu_eval(g, E, Dk)
    np.testing.assert_array_equal(res[0], full[0])
    np.testing.assert_array_equal(res[1], full[1])


def test_windows_small_graphs_with_swaps_and_bad_windows():
    rng = np.random.default_rng(31)
    for trial in range(40):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng)
        R = len(elig)
        iso = np.zeros(n, np.uint8)
        iso[list(outs)] = 1
        wl = Workload("rand", np.asarray(size, np.int64), np.asarray(cost), iso,
                      np.asarray([u for u, _ in edges], np.int32), np.asarray([v for _, v in edges], np.int32),
                      [""] * n, ["op"] * n, np.asarray(elig, np.int32), [list(u) for u in U], 1e3, 0.25)
        d = rng.integers(0, 3, R).astype(np.uint8)
        for r in range(R):
            if d[r] == 1 and not any(v == elig[r] for _, v in edges):
                d[r] = 2
        base, _, _ = random_valid_perm(rng, n, edges, elig, U, d)
        NT = n + 3 * R
        wg = WindowGenerator(wl, base, d if R else None, seed=trial, wmax=min(64, NT), pct_bad=25)
        ws, wln, wp = wg.generate(0, 200)
        # a few windows that are not permutations of the base window
        for k in range(0, 200, 23):
            if wln[k] >= 2:
                wp[k, 1] = wp[k, 0]
        g = Graph.from_workload(wl)
        o = OracleGraph.from_workload(wl)
        _, res = run_windows(g, base, d if R else np.zeros(1, np.uint8), ws, wln, wp)
        E = wg.expand(ws, wln, wp)
        ref = o.eval_batch(E, np.repeat(d[None], len(ws), 0) if R else None)
        assert_parity(*res, *ref)


@pytest.mark.parametrize("cfg", ["c2", "c5"])
def test_windows_dense_swap_events(cfg):
    """A base with P(swap) = 40%: most windows hold swap events, so the walk
    starts at the window from the base's state (end times written before the
    window read through from the base), and rejoins the base after it when
    its state is unchanged -- every window against the oracle."""
    wl = build_workload(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=6, p_swap=4000, p_remat=500)).generate(0, 16)
    o = OracleGraph.from_workload(wl)
    st, pk, lt = o.eval_batch(P, D)
    i = int(np.argmax(st == 0))
    assert st[i] == 0 and (D[i][:wl.R] == 2).sum() > wl.R // 4
    wg = WindowGenerator(wl, P[i], D[i], seed=13, pct_bad=1)
    ws, wln, wp = wg.generate(0, 2000)
    g = Graph.from_workload(wl)
    b, res = run_windows(g, P[i], D[i], ws, wln, wp)
    E = wg.expand(ws, wln, wp)
    Dk = np.repeat(D[i][None], len(ws), axis=0)
    ref = o.eval_batch(E, Dk)
    assert (ref[0] == 0).mean() > 0.9
    assert_parity(*res, *ref)
