"""delta8 wire format of the end-to-end call (host marshalling): a plain
numpy decoder must give back the schedules (ids clamped to 65535 when out of
[0, 65535]); the GPU test checks the device decoder through the C ABI."""
import numpy as np

from paper_conf_asplos_chend0zll024_b200.magis import encode_delta8


def decode(delta, exc_ptr, exc):
    K, n = delta.shape
    out = np.zeros((K, n), np.int64)
    for k in range(K):
        prev, e = 0, int(exc_ptr[k])
        for i in range(n):
            if delta[k, i] == -128:
                prev = int(exc[e])
                e += 1
            else:
                prev += int(delta[k, i])
            out[k, i] = prev
        assert e == exc_ptr[k + 1]
    return out


def test_round_trip():
    rng = np.random.default_rng(0)
    for n in (1, 5, 31, 32, 33, 300):
        P = np.stack([rng.permutation(n) for _ in range(20)]).astype(np.int64)
        P[3, 0] = 200                    # exception at a row start
        P[4] = np.arange(n)              # all small steps
        P[5, -1] = -7                    # out of range -> 65535
        P[6, 0] = 70000                  # out of range -> 65535
        d, xp, x = encode_delta8(P)
        assert d.dtype == np.int8 and xp.dtype == np.int32 and x.dtype == np.uint16
        want = np.where((P < 0) | (P > 65535), 65535, P)
        assert (decode(d, xp, x) == want).all()


def test_compact_for_topological_orders():
    from magis_inputs import CandidateGenerator, CandidateSpec, build_workload
    wl = build_workload("c2")
    P, _ = CandidateGenerator(wl, CandidateSpec(seed=1)).generate(0, 256)
    d, xp, x = encode_delta8(P)
    bytes_per_step = (d.nbytes + xp.nbytes + x.nbytes) / P.size
    assert bytes_per_step < 1.3          # vs 2 (u16) and 4 (int32)
    assert (decode(d[:8], xp[:9], x) == P[:8]).all()


def decode4(code, exc_ptr, exc, n):
    """Plain decoder of the delta4 format (magis.h magis_eval_schedules_host_delta4)."""
    K = code.shape[0]
    out = np.zeros((K, n), np.int64)
    for k in range(K):
        prev, e = 0, int(exc_ptr[k])
        for i in range(n):
            c = (int(code[k, i // 2]) >> (4 * (i % 2))) & 15
            if c == 0:
                prev = int(exc[e])
                e += 1
            else:
                prev += c - 8
            out[k, i] = prev
        assert e == exc_ptr[k + 1]
    return out


def test_delta4_round_trip():
    from paper_conf_asplos_chend0zll024_b200.magis import encode_delta4
    rng = np.random.default_rng(1)
    for n in (1, 2, 5, 31, 32, 33, 300):
        P = np.stack([rng.permutation(n) for _ in range(20)]).astype(np.int64)
        P[3, 0] = 200
        P[4] = np.arange(n)
        P[5, -1] = -7
        P[6, 0] = 70000
        P[7, :] = np.arange(n)[::-1] * 7 % max(n, 1)     # deltas of exactly +-7 and larger
        c, xp, x = encode_delta4(P)
        assert c.dtype == np.uint8 and c.shape == (20, (n + 1) // 2) and xp.dtype == np.int32
        want = np.where((P < 0) | (P > 65535), 65535, P)
        assert (decode4(c, xp, x, n) == want).all()


def test_delta4_smaller_than_delta8_for_topological_orders():
    from magis_inputs import CandidateGenerator, CandidateSpec, build_workload
    from paper_conf_asplos_chend0zll024_b200.magis import encode_delta4
    wl = build_workload("c2")
    P, _ = CandidateGenerator(wl, CandidateSpec(seed=1)).generate(0, 256)
    c, xp, x = encode_delta4(P)
    d, xp8, x8 = encode_delta8(P)
    b4 = (c.nbytes + xp.nbytes + x.nbytes) / P.size
    b8 = (d.nbytes + xp8.nbytes + x8.nbytes) / P.size
    assert b4 < 0.85 * b8
    assert (decode4(c[:8], xp[:9], x, P.shape[1]) == P[:8]).all()
