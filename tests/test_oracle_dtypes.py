"""Pins for the fp64 and bf16 allreduce oracle (O3/O4/O6 with reading R27) — CPU only.

What pins it: the bf16 rounding and bf16 (+) against torch's own CPU bf16
conversion/arithmetic (an independent library routine; torch adds bf16 in
fp32 and rounds once, which equals the correctly rounded result because
24 >= 2*8+2), hand-worked tie cases, and the literal Alg 2 simulations
against folds in the schedule's order computed with numpy float64 / torch
bf16 (a different derivation of the same result), integer-valued inputs
(exact in every order), the chunking of R4 at 16/esize elements per vector.
"""
import numpy as np
import pytest
import torch

import oracle
import synth


def _t(b):
    return torch.from_numpy(np.asarray(b, dtype=np.uint16).view(np.int16).copy()).view(torch.bfloat16)


def _b(t):
    return t.contiguous().view(torch.int16).numpy().view(np.uint16)


# ------------------------------------------------------------- bf16 arithmetic
def test_bf16_round_hand_cases():
    x = np.array([1.0, 1 + 2**-8, 1 + 3 * 2**-8, 1 + 2**-9, -2.5, 0.0, -0.0, np.inf, -np.inf,
                  2.0**-134, 1.5 * 2.0**-133, 2.0**-133, (2 - 2**-7) * 2.0**127,
                  (2 - 2**-7) * 2.0**127 * (1 + 2**-10), (2 - 2**-8) * 2.0**127])
    want = [0x3F80, 0x3F80, 0x3F82, 0x3F80, 0xC020, 0x0000, 0x8000, 0x7F80, 0xFF80,
            0x0000, 0x0002, 0x0001, 0x7F7F, 0x7F7F, 0x7F80]  # max finite; overflow on the tie
    assert [int(v) for v in oracle.bf16_round(x)] == want
    assert oracle.bf16_round(np.array([np.nan]))[0] & 0x7FFF > 0x7F80


def test_bf16_round_matches_torch():
    rng = np.random.default_rng(5)
    x = np.concatenate([rng.standard_normal(50000),
                        rng.standard_normal(20000) * 2.0 ** rng.integers(-140, 128, 20000),
                        # exact ties: 9 significant bits with the last one set
                        (rng.integers(256, 512, 20000) * 2 + 1) * 2.0 ** rng.integers(-60, 60, 20000)])
    # torch's float64 -> bf16 goes through fp32 (double rounding), so pin on
    # fp32-representable inputs, where torch's conversion is a single rounding.
    x32 = x.astype(np.float32)
    got = oracle.bf16_round(x32.astype(np.float64))
    ref = _b(torch.from_numpy(x32).to(torch.bfloat16))
    np.testing.assert_array_equal(got, ref)
    # just above a tie: the correctly rounded result rounds up (a double-rounding
    # implementation through fp32 would land on the tie and round to even)
    assert oracle.bf16_round(np.array([2.6015625 + 2.0**-40]))[0] == 0x4027
    assert oracle.bf16_round(np.array([2.6015625]))[0] == 0x4026


@pytest.mark.parametrize("op", [oracle.SUM, oracle.MAX, oracle.MIN])
def test_bf16_op_matches_torch(op):
    a = synth.bf16_bits_raw(61, 0, 0, 200000)
    b = synth.bf16_bits_raw(61, 1, 0, 200000)
    got = oracle.bf16_op(a, b, op)
    ta, tb = _t(a), _t(b)
    if op == oracle.SUM:
        np.testing.assert_array_equal(got, _b(ta + tb))
    else:
        ref = torch.maximum(ta, tb) if op == oracle.MAX else torch.minimum(ta, tb)
        # value comparison: -0 and +0 are interchangeable under max/min
        np.testing.assert_array_equal(oracle.bf16_to_f64(got), oracle.bf16_to_f64(_b(ref)))


def test_bf16_add_tie_to_even_by_hand():
    one = oracle.bf16_round(np.array([1.0]))
    half_ulp = oracle.bf16_round(np.array([2.0**-8]))
    three_half = oracle.bf16_round(np.array([3 * 2.0**-8]))
    assert oracle.bf16_op(one, half_ulp)[0] == 0x3F80          # 1 + ulp/2 -> 1 (even)
    assert oracle.bf16_op(one, three_half)[0] == 0x3F82        # 1 + 3ulp/2 -> 1 + 2ulp (even)


# ---------------------------------------------------------- schedule folds
def _fold_ring(x, start, add):
    P, n = x.shape
    idx = np.arange(n)
    acc = x[start, idx]
    for j in range(1, P):
        acc = add(x[(start + j) % P, idx], acc)
    return acc


def _fold_tree(x, add):
    v = [x[r] for r in range(x.shape[0])]
    m = 1
    while m < len(v):
        v = [add(v[r], v[r ^ m]) for r in range(len(v))]
        m <<= 1
    return v[0]


def _fold_rank_order(x, add):
    acc = x[0]
    for r in range(1, x.shape[0]):
        acc = add(acc, x[r])
    return acc


def _add_f64(a, b):
    return a + b


def _add_bf16(a, b):
    return _b(_t(a) + _t(b))


@pytest.mark.parametrize("algo,Ps", [(oracle.RING, [2, 3, 5, 8]), (oracle.RD, [2, 4, 8]),
                                     (oracle.DIRECT, [2, 3, 6, 8])])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (2, 100), (4, 9)])
def test_f64_schedule_folds(algo, Ps, Np, L):
    for P in Ps:
        x = np.stack([synth.normal_f64(71, r, 0, Np * L) for r in range(P)])
        y, red, arr = oracle.pallreduce(x, Np, algo)
        if algo == oracle.RING:
            ref = _fold_ring(x, oracle.chunk_ids(L, P, Np, esize=8), _add_f64)
        elif algo == oracle.RD:
            ref = _fold_tree(x, _add_f64)
        else:
            ref = _fold_rank_order(x, _add_f64)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint64), ref.view(np.uint64))
        assert (arr <= max(P - 1, 1)).all()


@pytest.mark.parametrize("algo,Ps", [(oracle.RING, [2, 3, 5, 8]), (oracle.RD, [2, 4, 8]),
                                     (oracle.DIRECT, [2, 3, 6, 8])])
@pytest.mark.parametrize("Np,L", [(1, 1), (3, 17), (2, 100), (4, 9)])
def test_bf16_schedule_folds(algo, Ps, Np, L):
    for P in Ps:
        x = np.stack([synth.bf16_bits(73, r, 0, Np * L) for r in range(P)])
        y, _, _ = oracle.pallreduce(x, Np, algo)
        if algo == oracle.RING:
            ref = _fold_ring(x, oracle.chunk_ids(L, P, Np, esize=2), _add_bf16)
        elif algo == oracle.RD:
            ref = _fold_tree(x, _add_bf16)
        else:
            ref = _fold_rank_order(x, _add_bf16)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("algo", [oracle.RING, oracle.RD, oracle.DIRECT])
def test_integer_valued_exact(algo):
    """|partial sums| <= 256 are exact in bf16 and any int sum is exact in fp64,
    so every order gives the plain definition."""
    P, Np, L = 4, 3, 21
    ints = np.stack([synth.int32_range(75, r, 0, Np * L, -32, 33) for r in range(P)])
    y64, _, _ = oracle.pallreduce(ints.astype(np.float64), Np, algo)
    np.testing.assert_array_equal(y64[1], ints.sum(0).astype(np.float64))
    xb = oracle.bf16_round(ints.astype(np.float64))
    yb, _, _ = oracle.pallreduce(xb, Np, algo)
    np.testing.assert_array_equal(oracle.bf16_to_f64(yb[2]), ints.sum(0).astype(np.float64))


def test_chunking_scales_with_element_size():
    """R4: a chunk is a whole number of 16-byte vectors for every dtype."""
    for esize, v in [(2, 8), (4, 4), (8, 2)]:
        c = oracle.chunk_ids(100, 3, 1, esize=esize)
        q = -(-100 // (v * 3)) * v
        assert q % v == 0
        np.testing.assert_array_equal(c, np.minimum(np.arange(100) // q, 2))


def test_bf16_ring_differs_from_rd_somewhere():
    """Schedules are distinguishable in bf16 too (so GPU parity checks the order)."""
    P, n = 8, 4096
    x = np.stack([synth.bf16_bits(77, r, 0, n) for r in range(P)])
    ring, _, _ = oracle.pallreduce(x, 1, oracle.RING)
    rd, _, _ = oracle.pallreduce(x, 1, oracle.RD)
    assert (ring[0] != rd[0]).any()
