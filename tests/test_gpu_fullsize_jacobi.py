"""GPU parity at the bench's C4 configuration (SURVEY §8(d) C4
§VI-D1): Jacobi on the full 16384^2 fp32 grid with 64-row CTA tiles (the
"rows" kernel the bench times), 4 x 2 and 8 x 1 virtual-rank decompositions
(every halo pushed by pc_pready_warp inside the kernel), 100 iterations —
bit-exact against the sequential oracle O5 (fixed fp32 expression, R17), and
within the north_star 1e-5 relative bound of its fp64 image."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_temucinslsga24_b200 as pc
import synth
from paper_conf_sc_temucinslsga24_b200 import apps

from gpu_util import comms

pytestmark = pytest.mark.gpu

N, ITERS = 16384, 100


@pytest.fixture(scope="module")
def grids():
    a0 = synth.jacobi_init(N, N, "random")
    return a0, oracle.jacobi_seq(a0, ITERS)  # ~40 s of CPU


@pytest.mark.parametrize("Py,Px", [(4, 2), (8, 1)])
def test_jacobi_16384_bitexact(grids, Py, Px):
    a0, ref = grids
    P = Py * Px
    with comms(P, timeout_ms=60000) as cs:
        st = torch.cuda.Stream()
        js = apps.JacobiSolver(cs, list(range(P)), N, Py, Px, ITERS, H=64, kernel="rows")
        js.set_initial(a0)
        torch.cuda.synchronize()
        js.solve(st, first_prepare=lambda lists: pc.run_ranks(
            [(lambda l=l: [q.pbuf_prepare(st) for q in l]) for l in lists]))
        torch.cuda.synchronize()
        assert js.errors() == []
        got = js.result()
        js.free()
    np.testing.assert_array_equal(got, ref)
    ref64 = ref.astype(np.float64)
    assert np.abs(got - ref64).max() <= 1e-5 * np.abs(ref64).max()
