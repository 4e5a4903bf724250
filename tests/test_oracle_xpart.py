"""Pins of O11 (MPI-4 partitioned send/recv with different partition counts on
the two sides, reading R30) against things other than itself: the hand-worked
example in tests/golden/xpart_2x3.txt, the equal-partitioning special case
(receive partition p complete iff its transport partition p // g is — the O1
semantics), monotonicity, and the whole-buffer / single-byte extremes."""
import itertools
import os

import numpy as np
import pytest

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "xpart_2x3.txt")


def test_golden_2x3():
    rows = [ln.split("->") for ln in open(GOLDEN) if ln.strip() and not ln.startswith("#")]
    assert len(rows) == 4
    for lhs, rhs in rows:
        readied = [bool(int(v)) for v in lhs.split()]
        want = [bool(int(v)) for v in rhs.split()]
        assert oracle.xpart_arrived(2, 6, 1, 3, 4, np.array(readied)).tolist() == want


@pytest.mark.parametrize("N,g", [(1, 1), (5, 1), (5, 2), (8, 3), (8, 8)])
def test_equal_partitioning_is_transport_flag(N, g):
    """Same partitioning on both sides: p is complete iff every user partition
    of its transport partition p // g is readied (the O1 / flag[p // g] rule)."""
    rng = np.random.default_rng(N * 10 + g)
    for _ in range(20):
        readied = rng.random(N) < 0.6
        got = oracle.xpart_arrived(N, 12, g, N, 12, readied)
        for p in range(N):
            t = p // g
            assert got[p] == all(readied[t * g:min((t + 1) * g, N)])


@pytest.mark.parametrize("Ns,Nr,g", [(2, 3, 1), (3, 2, 1), (4, 6, 2), (6, 4, 1), (1, 5, 1), (5, 1, 1), (6, 4, 4)])
def test_monotone_and_extremes(Ns, Nr, g):
    total = 60  # divisible by every Ns, Nr above
    none = oracle.xpart_arrived(Ns, total // Ns, g, Nr, total // Nr, np.zeros(Ns, bool))
    full = oracle.xpart_arrived(Ns, total // Ns, g, Nr, total // Nr, np.ones(Ns, bool))
    assert not none.any() and full.all()
    # readying more never un-arrives anything
    for bits in itertools.product([0, 1], repeat=Ns):
        r = np.array(bits, bool)
        a = oracle.xpart_arrived(Ns, total // Ns, g, Nr, total // Nr, r)
        for u in np.nonzero(~r)[0]:
            r2 = r.copy()
            r2[u] = True
            b = oracle.xpart_arrived(Ns, total // Ns, g, Nr, total // Nr, r2)
            assert (b | ~a).all()
    # a single receive partition covering the whole buffer needs every send partition
    one = [oracle.xpart_arrived(Ns, total // Ns, g, 1, total, np.eye(Ns, dtype=bool)[u] | True)[0] for u in range(Ns)]
    assert all(one)
    miss = oracle.xpart_arrived(Ns, total // Ns, g, 1, total, ~np.eye(Ns, dtype=bool)[0])
    assert not miss[0]
