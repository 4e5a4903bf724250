"""Pins of the NEXT-3 collective oracles (O8 reduce-scatter, O9 allgather,
O10 broadcast) against things other than themselves: brute-force integer sums,
exactness of integer-valued fp32, the independently pinned DIRECT allreduce
oracle O6 (whose rank-order fold is the same association, R25), and the
special cases P = 1 / P = 2."""
import numpy as np
import pytest

import oracle
import synth

SEED = synth.BASE_SEED


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("Np,count", [(1, 1), (3, 5), (7, 16)])
def test_rs_int32_brute_force(P, Np, count):
    """int32 sum (wrapping) / max / min against a Python-int loop per element."""
    rng = np.random.default_rng(P * 100 + Np)
    x = rng.integers(-2**31, 2**31, size=(P, Np * P * count), dtype=np.int64).astype(np.int32)
    for op in (oracle.SUM, oracle.MAX, oracle.MIN):
        y = oracle.reduce_scatter_def(x, Np, op)
        for d in range(P):
            for u in range(Np):
                for i in range(count):
                    vals = [int(x[k, (u * P + d) * count + i]) for k in range(P)]
                    if op == oracle.SUM:
                        want = sum(vals) % 2**32
                        want = want - 2**32 if want >= 2**31 else want
                    else:
                        want = max(vals) if op == oracle.MAX else min(vals)
                    assert int(y[d, u * count + i]) == want


@pytest.mark.parametrize("P", [2, 4, 8])
def test_rs_fp32_integer_valued_is_exact(P):
    """|x| < 2^24 / P: every summation order is exact, so the fp32 fold equals
    the integer sum."""
    Np, count = 4, 33
    rng = np.random.default_rng(7)
    xi = rng.integers(-(2**24) // P + 1, 2**24 // P, size=(P, Np * P * count))
    y = oracle.reduce_scatter_def(xi.astype(np.float32), Np)
    want = xi.reshape(P, Np, P, count).sum(axis=0).transpose(1, 0, 2).reshape(P, Np * count)
    np.testing.assert_array_equal(y, want.astype(np.float32))


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_rs_equals_direct_allreduce_chunks(P, dt):
    """With count a multiple of the chunk quantum, partition u of the DIRECT
    allreduce (O6, pinned in test_oracle_allreduce / _dtypes) has chunk d = block
    d, so rank d's reduce-scatter block equals the allreduce result's chunk d."""
    Np = 3
    q = 4 if dt == np.float32 else 2  # R4 / R27 chunk quantum (16-B multiples)
    count = 5 * q
    L = P * count
    x = np.stack([synth.normal_f32(SEED, r, 0, Np * L) for r in range(P)]).astype(dt)
    ar, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT)
    rs = oracle.reduce_scatter_def(x, Np)
    for d in range(P):
        chunks = ar[d].reshape(Np, P, count)[:, d, :].reshape(-1)
        np.testing.assert_array_equal(rs[d].view(np.uint8), chunks.view(np.uint8))


def test_rs_bf16_matches_pairwise_oracle_op():
    P, Np, count = 3, 2, 8
    x = np.stack([oracle.bf16_round(synth.normal_f32(SEED, r, 1, Np * P * count).astype(np.float64))
                  for r in range(P)])
    y = oracle.reduce_scatter_def(x, Np)
    b = x.reshape(P, Np, P, count)
    for d in range(P):
        want = oracle.bf16_op(oracle.bf16_op(b[0, :, d].reshape(-1), b[1, :, d].reshape(-1)), b[2, :, d].reshape(-1))
        np.testing.assert_array_equal(y[d], want)


def test_rs_special_cases():
    x = synth.normal_f32(SEED, 0, 2, 3 * 7)[None]
    np.testing.assert_array_equal(oracle.reduce_scatter_def(x, 3), x)  # P = 1: a copy
    x2 = np.stack([synth.normal_f32(SEED, r, 3, 2 * 2 * 6) for r in range(2)])
    y = oracle.reduce_scatter_def(x2, 2)
    b = x2.reshape(2, 2, 2, 6)
    for d in range(2):  # P = 2: x0 + x1 under every association
        np.testing.assert_array_equal(y[d], (b[0, :, d] + b[1, :, d]).reshape(-1))


def test_allgather_and_bcast_definitions():
    P, n = 4, 10
    x = np.arange(P * n, dtype=np.int32).reshape(P, n)
    ag = oracle.allgather_def(x)
    for r in range(P):
        for k in range(P):
            np.testing.assert_array_equal(ag[r, k * n:(k + 1) * n], x[k])
    bc = oracle.bcast_def(x, 2)
    assert (bc == x[2]).all()
