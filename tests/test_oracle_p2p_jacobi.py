"""Pins for the p2p oracle (O1) and the Jacobi oracle (O5) — CPU only.

O1 is pinned by its definition (recv == send byte for byte, i.e. memcpy),
exactly-once publication of every transport partition under seeded random
Pready orders and concurrent workers, and the restart hazard of P:L60 that
Pbuf_prepare exists to prevent.

O5 is pinned by closed forms: constant and integer-linear fields are exact
fixed points, the one-step response of a unit boundary, the eigenmode decay
u_k = cos(pi/(n+1))^k u_0, and decomposition invariance.
"""
import numpy as np
import pytest

import oracle
import synth


def tagged(E, nbytes, rank=0, seed=9):
    return np.stack([synth.bytes_tagged(seed, rank, e, nbytes) for e in range(E)])


@pytest.mark.parametrize("partitions,part_bytes,agg", [(8, 128, 1), (8, 128, 3), (8, 128, 8), (1, 64, 1),
                                                       (13, 8, 4), (32, 256, 32), (7, 0, 2)])
@pytest.mark.parametrize("workers", [1, 4])
def test_p2p_bytes_and_exactly_once(partitions, part_bytes, agg, workers):
    E = 3
    send = tagged(E, partitions * part_bytes)
    orders = np.stack([synth.permutation(3, 0, e, partitions) for e in range(E)])
    consumed, arrivals = oracle.p2p(send, partitions, agg, orders, workers=workers)
    np.testing.assert_array_equal(consumed, send)
    assert arrivals.shape == (E, -(-partitions // agg))
    assert (arrivals == 1).all()


def test_p2p_many_permutations():
    """>=100 seeded permutations x 4 concurrent workers: exactly-once every time."""
    partitions, agg = 16, 4
    for s in range(100):
        send = tagged(2, partitions * 8, seed=s)
        orders = np.stack([synth.permutation(1000 + s, 0, e, partitions) for e in range(2)])
        consumed, arrivals = oracle.p2p(send, partitions, agg, orders, workers=4, jitter_seed=s)
        assert (arrivals == 1).all()
        np.testing.assert_array_equal(consumed, send)


def test_restart_hazard_needs_rtr():
    """without the ready-to-receive handshake a restarted sender
    overwrites a receiver that has not consumed the previous epoch; with it
    (Pbuf_prepare) every epoch is consumed intact."""
    E, partitions = 3, 4
    send = tagged(E, partitions * 64)
    orders = np.tile(np.arange(partitions, dtype=np.int32), (E, 1))
    bad, _ = oracle.p2p(send, partitions, 1, orders, use_rtr=False, recv_delay_us=30000)
    assert not (bad[0] == send[0]).all(), "epoch 1 should have been overwritten"
    good, arr = oracle.p2p(send, partitions, 1, orders, use_rtr=True, recv_delay_us=30000)
    np.testing.assert_array_equal(good, send)
    assert (arr == 1).all()


# ------------------------------------------------------------------ Jacobi
def test_jacobi_constant_fixed_point():
    a = np.full((20, 24), 0.7, dtype=np.float32)
    np.testing.assert_array_equal(oracle.jacobi_seq(a, 7), a)


def test_jacobi_integer_linear_fixed_point():
    """u = a*i + b*j + d with small integers: each update is exact and the
    discrete Laplacian of a linear field is 0, so u is a bit-exact fixed point."""
    i, j = np.mgrid[0:18, 0:22]
    u = (3 * i - 5 * j + 7).astype(np.float32)
    np.testing.assert_array_equal(oracle.jacobi_seq(u, 5), u)
    np.testing.assert_array_equal(oracle.jacobi_decomp(u, 5, 2, 2), u)


def test_jacobi_one_step_unit_boundary():
    n = 8
    a = np.zeros((n, n), dtype=np.float32)
    a[0, :] = a[-1, :] = a[:, 0] = a[:, -1] = 1.0
    b = oracle.jacobi_seq(a, 1)
    exp = np.zeros_like(a)
    exp[0, :] = exp[-1, :] = exp[:, 0] = exp[:, -1] = 1.0
    exp[1, 1:-1] = exp[-2, 1:-1] = exp[1:-1, 1] = exp[1:-1, -2] = 0.25
    for (r, c) in [(1, 1), (1, n - 2), (n - 2, 1), (n - 2, n - 2)]:
        exp[r, c] = 0.5
    np.testing.assert_array_equal(b, exp)


@pytest.mark.parametrize("n", [30, 62])
def test_jacobi_eigenmode_decay(n):
    """Zero boundary, u0 = sin(pi i/(n+1)) sin(pi j/(n+1)) on the n x n interior:
    Jacobi multiplies it by cos(pi/(n+1)) per sweep."""
    N = n + 2
    i, j = np.mgrid[0:N, 0:N]
    u0 = (np.sin(np.pi * i / (n + 1)) * np.sin(np.pi * j / (n + 1)))
    u0[0, :] = u0[-1, :] = u0[:, 0] = u0[:, -1] = 0.0
    k = 100
    out = oracle.jacobi_seq(u0.astype(np.float32), k)
    exact = np.cos(np.pi / (n + 1)) ** k * u0
    assert np.abs(out - exact).max() <= 1e-6 * np.abs(exact).max()


@pytest.mark.parametrize("Py,Px", [(1, 1), (2, 1), (1, 2), (2, 2), (4, 2), (8, 1), (3, 2)])
def test_jacobi_decomposition_invariance(Py, Px):
    a0 = synth.jacobi_init(48, 36, "random")
    if 48 % Py or 36 % Px:
        pytest.skip("not divisible")
    np.testing.assert_array_equal(oracle.jacobi_decomp(a0, 25, Py, Px), oracle.jacobi_seq(a0, 25))


def test_jacobi_perf_init_decomp():
    a0 = synth.jacobi_init(64, 64, "perf")
    s = oracle.jacobi_seq(a0, 40)
    np.testing.assert_array_equal(oracle.jacobi_decomp(a0, 40, 4, 2), s)
    assert s[1, 1:-1].min() > 0 and (s[-1] == 0).all()
