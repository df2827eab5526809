"""NEXT-3 on the GPU: magis_hotspots (hot-spots, Eq. 3 heat, Eq. 4 score)
and magis_graph_idom against the oracle, element by element and bit-exact
(heat is an int64 byte sum; score is computed with the same two roundings)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from magis_inputs import CandidateGenerator, CandidateSpec, build_workload  # noqa: E402
from magis_inputs.graph import Workload  # noqa: E402
from oracle import OracleGraph  # noqa: E402
from paper_conf_asplos_chend0zll024_b200 import Graph  # noqa: E402
from tests.test_oracle_pins import fig2a_graph, random_case, random_valid_perm  # noqa: E402
from tests.test_parity_gpu import DEV, gpu_eval  # noqa: E402


def wl_of(n, edges, size, cost, outs, elig, U):
    iso = np.zeros(n, np.uint8)
    iso[list(outs)] = 1
    return Workload("t", np.asarray(size, np.int64), np.asarray(cost, np.float64), iso,
                    np.asarray([u for u, _ in edges], np.int32), np.asarray([v for _, v in edges], np.int32),
                    [""] * n, ["op"] * n, np.asarray(elig, np.int32), [list(u) for u in U], 1e3, 0.25)


def gpu_hot(g, perms, decs, nsplit):
    P = torch.from_numpy(np.ascontiguousarray(perms, np.int32)).to(DEV)
    D = torch.from_numpy(np.ascontiguousarray(decs, np.uint8).reshape(len(perms), g.R)).to(DEV) if g.R else None
    out = g.hotspots(P, D, nsplit)
    torch.cuda.synchronize()
    return [x.cpu().numpy() for x in out]


def check(g, o, perms, decs, nsplit):
    st, pk, hot, heat, score = gpu_hot(g, perms, decs, nsplit)
    for k in range(len(perms)):
        s2, p2, h2, he2, sc2 = o.hotspots(perms[k], decs[k] if o.R else None, nsplit)
        assert st[k] == s2 and pk[k] == p2, k
        np.testing.assert_array_equal(hot[k], h2)
        np.testing.assert_array_equal(heat[k], he2)
        np.testing.assert_array_equal(score[k], sc2)
    return st, pk


def test_fig2a_on_gpu():
    n, edges, size, outputs, f, b = fig2a_graph()
    wl = wl_of(n, edges, size, [0.0] * n, outputs, [], [])
    g, o = Graph.from_workload(wl), OracleGraph.from_workload(wl)
    assert g.idom().tolist() == o.idom().tolist()
    order = np.asarray([f(i) for i in range(1, 33)] + [b(i) for i in range(1, 33)], np.int32)
    bad = order.copy()
    bad[0], bad[1] = bad[1], bad[0]
    st, pk = check(g, o, np.stack([order, bad]), np.zeros((2, 1), np.uint8), 2)
    assert pk[0] == 1056 and st[1] == 2


def test_random_graphs_with_decisions():
    rng = np.random.default_rng(41)
    for trial in range(60):
        n, edges, size, cost, outs, elig, U, dec = random_case(rng, nmax=12)
        for r in range(len(elig)):
            if dec[r] == 1 and not any(v == elig[r] for _, v in edges):
                dec[r] = 2
        wl = wl_of(n, edges, size, cost, outs, elig, U)
        g, o = Graph.from_workload(wl), OracleGraph.from_workload(wl)
        assert g.idom().tolist() == o.idom().tolist(), trial
        R = len(elig)
        perms, decs = [], []
        for _ in range(6):
            d = dec.copy()
            if R and rng.random() < 0.5:
                d = rng.integers(0, 3, R).astype(np.uint8)
                for r in range(R):
                    if d[r] == 1 and not any(v == elig[r] for _, v in edges):
                        d[r] = 0
            p, _, _ = random_valid_perm(rng, n, edges, elig, U, d)
            perms.append(p)
            decs.append(d if R else np.zeros(1, np.uint8))
        perms = np.asarray(perms, np.int32)
        # one invalid (swapped neighbours) and one non-permutation candidate
        perms[1, [0, 1]] = perms[1, [1, 0]]
        perms[2, 0] = perms[2, 1]
        decs = np.asarray(decs, np.uint8)
        check(g, o, perms, decs if R else np.zeros((6, 1), np.uint8), int(rng.integers(1, 5)))


@pytest.mark.parametrize("cfg,K", [("c2", 12), ("c5", 12), ("c3", 3)])
def test_workloads(cfg, K):
    wl = build_workload(cfg)
    P, D = CandidateGenerator(wl, CandidateSpec(seed=21)).generate(0, K)
    g, o = Graph.from_workload(wl), OracleGraph.from_workload(wl)
    assert g.idom().tolist() == o.idom().tolist()
    st, pk = check(g, o, P, D, 2)
    # the same status / peak as the batch evaluator
    st2, pk2, _ = gpu_eval(g, P, D)
    np.testing.assert_array_equal(st, st2)
    np.testing.assert_array_equal(pk, pk2)
    assert (st == 0).sum() >= K - 1
