"""Pins for the allreduce oracle (O2, O3, O4) — CPU only.

What pins it: brute-force sums by numpy (an independent
library routine) on tiny inputs, exact int semantics, integer-valued fp32
(every order exact), the Alg 1 worked table (tests/golden), schedule
invariants, special cases (P=1 copy, P=2, constant inputs), exactly-once
reduce/arrival counts, all-ranks-identical, NaN propagation, and the
R16 error bound against a float64 sum computed by numpy.
"""
import os

import numpy as np
import pytest

import oracle
import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def wrap_sum(x):
    s = x.astype(np.int64).sum(axis=0)
    return ((s + 2**31) % 2**32 - 2**31).astype(np.int32)


# ---------------------------------------------------------------- Alg 1 table
def test_alg1_golden_P4():
    rows = np.loadtxt(os.path.join(GOLD, "alg1_ring_P4_r0.txt"), dtype=np.int32, comments="#")
    t = oracle.alg1_table(4, 0)
    assert t.shape == (6, 5)
    np.testing.assert_array_equal(t, rows[:, 1:])


@pytest.mark.parametrize("P", [2, 3, 4, 5, 6, 7, 8])
def test_alg1_invariants(P):
    """R_i == A_{i-1}; RS arrivals are every chunk but r; AG arrivals every chunk
    but r+1; the right neighbour receives at step i what r sends at step i;
    op on exactly the first P-1 steps."""
    tabs = [oracle.alg1_table(P, r) for r in range(P)]
    for r, t in enumerate(tabs):
        assert len(t) == 2 * (P - 1)
        I, R, op, O, A = t.T
        assert (I == (r - 1) % P).all() and (O == (r + 1) % P).all()
        assert (R[1:] == A[:-1]).all()
        assert list(op) == [1] * (P - 1) + [0] * (P - 1)
        assert sorted(A[: P - 1]) == sorted(set(range(P)) - {r})
        assert sorted(A[P - 1:]) == sorted(set(range(P)) - {(r + 1) % P})
        assert R[0] == r
        nxt = tabs[(r + 1) % P]
        assert (nxt[:, 4] == R).all()


# ----------------------------------------------------- brute force, int32
MATRIX_P = [1, 2, 3, 4, 5, 8]
MATRIX_NP = [1, 2, 3, 7, 8]
MATRIX_L = [0, 1, 3, 4, 5, 16, 17, 64]


@pytest.mark.parametrize("P", MATRIX_P)
@pytest.mark.parametrize("Np", MATRIX_NP)
def test_ring_int32_sum_bruteforce(P, Np):
    for L in MATRIX_L:
        x = np.stack([synth.int32_full(11, r, 0, Np * L) for r in range(P)])
        orders = np.stack([synth.permutation(5, r, L, Np) for r in range(P)])[None]
        y, red, arr = oracle.pallreduce(x, Np, oracle.RING, orders=orders, jitter_seed=L + 1)
        ref = wrap_sum(x)
        for r in range(P):
            np.testing.assert_array_equal(y[r], ref)
        if P > 1:
            assert (arr == 1).all(), "every (u, step) must arrive exactly once"
            exp = np.array([1] * (P - 1) + [0] * (P - 1), dtype=np.uint32)
            assert (red == exp[None, None, :]).all(), "reduce exactly once per MPI_Op step (P:L213)"


@pytest.mark.parametrize("op,fn", [(oracle.MAX, np.max), (oracle.MIN, np.min)])
@pytest.mark.parametrize("algo,Ps", [(oracle.RING, [1, 2, 3, 5, 8]), (oracle.RD, [1, 2, 4, 8])])
def test_int32_maxmin(op, fn, algo, Ps):
    for P in Ps:
        for Np, L in [(1, 1), (3, 17), (8, 5), (2, 64)]:
            x = np.stack([synth.int32_full(3, r, 0, Np * L) for r in range(P)])
            y, _, _ = oracle.pallreduce(x, Np, algo, op=op)
            for r in range(P):
                np.testing.assert_array_equal(y[r], fn(x, axis=0))
            np.testing.assert_array_equal(oracle.allreduce_def_i32(x, op), fn(x, axis=0))


@pytest.mark.parametrize("P", [1, 2, 4, 8])
def test_rd_int32_sum_bruteforce(P):
    for Np in MATRIX_NP:
        for L in MATRIX_L:
            x = np.stack([synth.int32_full(12, r, 0, Np * L) for r in range(P)])
            y, red, arr = oracle.pallreduce(x, Np, oracle.RD)
            for r in range(P):
                np.testing.assert_array_equal(y[r], wrap_sum(x))
            if P > 1:
                assert (arr == 1).all() and (red == 1).all()


def test_rd_rejects_non_power_of_two():
    x = np.zeros((3, 8), dtype=np.int32)
    with pytest.raises(oracle.OracleError):
        oracle.pallreduce(x, 1, oracle.RD)


def test_def_i32_matches_numpy():
    x = np.stack([synth.int32_full(4, r, 0, 1000) for r in range(8)])
    np.testing.assert_array_equal(oracle.allreduce_def_i32(x), wrap_sum(x))


# ----------------------------------------------------------- fp32
@pytest.mark.parametrize("algo,P", [(oracle.RING, 3), (oracle.RING, 8), (oracle.RD, 8), (oracle.RD, 4)])
def test_fp32_integer_valued_exact(algo, P):
    """|x| < 2^24/P: every summation order is exact, so the fp32 result equals
    the integer sum bit for bit."""
    Np, L = 7, 64
    bound = (1 << 24) // P
    x = np.stack([synth.int_valued_f32(21, r, 0, Np * L, bound) for r in range(P)])
    y, _, _ = oracle.pallreduce(x, Np, algo)
    ref = x.astype(np.int64).sum(axis=0).astype(np.float32)
    for r in range(P):
        np.testing.assert_array_equal(y[r], ref)


@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("Np,L", [(1, 1), (2, 3), (3, 17), (7, 64), (1, 4), (8, 100)])
def test_ring_fp32_closed_form_and_bound(P, Np, L):
    """O3 literal simulation == the closed-form ring fold (a different derivation
    of the same result) bit for bit; all ranks identical; within R16 of fp64."""
    x = np.stack([synth.normal_f32(31, r, 0, Np * L) for r in range(P)])
    y, _, _ = oracle.pallreduce(x, Np, oracle.RING)
    cf = oracle.ring_fold_f32(x, oracle.chunk_ids(L, P, Np))
    for r in range(P):
        np.testing.assert_array_equal(y[r].view(np.uint32), cf.view(np.uint32))
    ref = x.astype(np.float64).sum(axis=0)
    bound = 1e-5 * np.abs(x.astype(np.float64)).sum(axis=0)
    assert (np.abs(y[0].astype(np.float64) - ref) <= bound).all()


def test_ring_fold_differs_from_tree_somewhere():
    """The schedule fixes the bits: ring and RD orders are different roundings
    (so a bit-exact parity test can tell the schedules apart)."""
    P, n = 8, 4096
    x = np.stack([synth.normal_f32(32, r, 0, n) for r in range(P)])
    ring = oracle.ring_fold_f32(x, np.zeros(n, np.int32))
    tree = oracle.rd_tree_f32(x)
    assert (ring != tree).any()
    ref = x.astype(np.float64).sum(0)
    b = 1e-5 * np.abs(x.astype(np.float64)).sum(0)
    assert (np.abs(ring - ref) <= b).all() and (np.abs(tree - ref) <= b).all()


def test_ring_fold_small_by_hand():
    """Fold start = chunk id (c.1 O3): for P=3 and chunk 1, ((x1+x2)+x0)."""
    x = np.array([[1e8], [1.0], [-1e8]], dtype=np.float32)
    # start at 1: (1 + -1e8) + 1e8 = (-1e8 after rounding) + 1e8 = 0
    assert oracle.ring_fold_f32(x, np.array([1], np.int32))[0] == 0.0
    # start at 0: (1e8 + 1) + -1e8 = 1e8 + -1e8 = 0 ; start at 2: (-1e8 + 1e8) + 1 = 1
    assert oracle.ring_fold_f32(x, np.array([2], np.int32))[0] == 1.0


@pytest.mark.parametrize("P", [2, 4, 8])
def test_rd_fp32_tree(P):
    Np, L = 3, 33
    x = np.stack([synth.normal_f32(41, r, 0, Np * L) for r in range(P)])
    y, _, _ = oracle.pallreduce(x, Np, oracle.RD)
    t = oracle.rd_tree_f32(x)
    for r in range(P):
        np.testing.assert_array_equal(y[r].view(np.uint32), t.view(np.uint32))
    if P == 4:
        # by hand: ((x0+x1)+(x2+x3))
        h = ((x[0] + x[1]) + (x[2] + x[3])).astype(np.float32)
        np.testing.assert_array_equal(t, h)


def test_special_cases():
    # P = 1: a copy
    x = synth.normal_f32(1, 0, 0, 40)[None]
    for algo in (oracle.RING, oracle.RD):
        y, _, _ = oracle.pallreduce(x, 4, algo)
        np.testing.assert_array_equal(y, x)
    # P = 2: x0 + x1 under every schedule
    x = np.stack([synth.normal_f32(2, r, 0, 64) for r in range(2)])
    for algo in (oracle.RING, oracle.RD):
        y, _, _ = oracle.pallreduce(x, 2, algo)
        np.testing.assert_array_equal(y[0], x[0] + x[1])
        np.testing.assert_array_equal(y[1], x[0] + x[1])
    # all x_r = v (dyadic, P*v exact) -> P*v
    for P in (3, 8):
        x = np.full((P, 48), 0.375, dtype=np.float32)
        y, _, _ = oracle.pallreduce(x, 3, oracle.RING)
        assert (y == np.float32(0.375 * P)).all()


def test_nan_propagates():
    P, n = 4, 32
    x = np.stack([synth.normal_f32(3, r, 0, n) for r in range(P)])
    x[2, 5] = np.nan
    for algo in (oracle.RING, oracle.RD):
        y, _, _ = oracle.pallreduce(x, 2, algo)
        assert np.isnan(y[:, 5]).all() and not np.isnan(np.delete(y, 5, axis=1)).any()


@pytest.mark.parametrize("algo,P", [(oracle.RING, 5), (oracle.RD, 8)])
def test_inplace_and_epochs(algo, P):
    """R22: sendbuf == recvbuf gives the same bits; 3 back-to-back epochs with
    epoch-tagged inputs each give their own epoch's result."""
    Np, L, E = 3, 20, 3
    x = np.stack([np.stack([synth.normal_f32(50, r, e, Np * L) for r in range(P)]) for e in range(E)])
    orders = np.stack([np.stack([synth.permutation(9, r, e, Np) for r in range(P)]) for e in range(E)])
    y0, _, _ = oracle.pallreduce(x, Np, algo, orders=orders)
    y1, _, _ = oracle.pallreduce(x, Np, algo, orders=orders, inplace=True, jitter_seed=77)
    np.testing.assert_array_equal(y0.view(np.uint32), y1.view(np.uint32))
    for e in range(E):
        ref = (oracle.ring_fold_f32(x[e], oracle.chunk_ids(L, P, Np)) if algo == oracle.RING
               else oracle.rd_tree_f32(x[e]))
        np.testing.assert_array_equal(y0[e, 0].view(np.uint32), ref.view(np.uint32))


def test_random_orders_exactly_once():
    """16 seeded Pready permutations: termination, exactly-once, same bits."""
    P, Np, L = 4, 8, 16
    x = np.stack([synth.normal_f32(60, r, 0, Np * L) for r in range(P)])
    first = None
    for s in range(16):
        orders = np.stack([synth.permutation(100 + s, r, 0, Np) for r in range(P)])[None]
        y, red, arr = oracle.pallreduce(x, Np, oracle.RING, orders=orders, jitter_seed=s)
        assert (arr == 1).all()
        if first is None:
            first = y
        np.testing.assert_array_equal(y.view(np.uint32), first.view(np.uint32))


def test_def_f64_is_exactish():
    x = np.stack([synth.normal_f32(7, r, 0, 1000) for r in range(8)])
    y, a = oracle.allreduce_def_f64(x)
    np.testing.assert_allclose(y, x.astype(np.float64).sum(0), rtol=0, atol=1e-12)
    np.testing.assert_allclose(a, np.abs(x.astype(np.float64)).sum(0), rtol=1e-15)


# ------------------------------------------------------------- DIRECT (O6)
@pytest.mark.parametrize("P", [1, 2, 3, 4, 5, 8])
def test_direct_int32_bruteforce_and_counts(P):
    for Np in (1, 3, 8):
        for L in (0, 1, 5, 17, 64):
            x = np.stack([synth.int32_full(13, r, 0, Np * L) for r in range(P)])
            orders = np.stack([synth.permutation(17, r, L, Np) for r in range(P)])[None]
            y, red, arr = oracle.pallreduce(x, Np, oracle.DIRECT, orders=orders, jitter_seed=L)
            for r in range(P):
                np.testing.assert_array_equal(y[r], wrap_sum(x))
            if P > 1:
                # S_0: P-1 arrivals, P-1 reduces (one per incoming neighbour); S_1: P-1 arrivals
                assert (red[:, :, 0] == P - 1).all() and (red[:, :, 1] == 0).all()
                assert (arr == P - 1).all()


@pytest.mark.parametrize("P", [2, 3, 5, 8])
def test_direct_fp32_rank_order_fold(P):
    """R25: the arrivals are folded in rank order, so every element is the left
    fold over ranks 0..P-1 (the ring fold started at rank 0), on every rank,
    whatever the arrival order."""
    Np, L = 3, 101
    x = np.stack([synth.normal_f32(71, r, 0, Np * L) for r in range(P)])
    ref = oracle.ring_fold_f32(x, np.zeros(Np * L, np.int32))
    for s in range(4):
        orders = np.stack([synth.permutation(300 + s, r, 0, Np) for r in range(P)])[None]
        y, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT, orders=orders, jitter_seed=s)
        for r in range(P):
            np.testing.assert_array_equal(y[r].view(np.uint32), ref.view(np.uint32))
    # by hand for P = 3: ((x0 + x1) + x2)
    if P == 3:
        np.testing.assert_array_equal(ref, ((x[0] + x[1]) + x[2]).astype(np.float32))
    assert (np.abs(ref - x.astype(np.float64).sum(0)) <= 1e-5 * np.abs(x.astype(np.float64)).sum(0)).all()


def test_direct_inplace_epochs_maxmin():
    P, Np, L, E = 4, 2, 33, 3
    x = np.stack([np.stack([synth.int32_full(5, r, e, Np * L) for r in range(P)]) for e in range(E)])
    y, _, _ = oracle.pallreduce(x, Np, oracle.DIRECT, inplace=True)
    for e in range(E):
        for r in range(P):
            np.testing.assert_array_equal(y[e, r], wrap_sum(x[e]))
    y, _, _ = oracle.pallreduce(x[0], Np, oracle.DIRECT, op=oracle.MAX)
    np.testing.assert_array_equal(y[0], x[0].max(0))
