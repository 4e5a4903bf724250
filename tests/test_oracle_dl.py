"""Pins for O7, the DL proxy producer (reading R28: gradient of the mean binary
cross-entropy w.r.t. the predictions, §VI-D2) — CPU only.

What pins it: closed forms at p = 1/2 and the y = 0 / y = 1 limits, and
torch autograd of ``F.binary_cross_entropy(reduction="mean")`` in float64 (an
independent library derivative) within the fp32 error of five correctly
rounded operations."""
import numpy as np
import torch

import oracle
import synth


def test_closed_forms():
    p = np.array([0.5, 0.5, 0.25, 0.75], np.float32)
    y = np.array([1.0, 0.0, 0.0, 1.0], np.float32)
    g = oracle.bce_grad(p, y, 1.0)
    # (0.5-1)/(0.25) = -2 ; 0.5/0.25 = 2 ; 0.25/(0.1875) = 4/3 ; -0.25/0.1875 = -4/3
    np.testing.assert_array_equal(g[:2], [-2.0, 2.0])
    assert g[2] == np.float32(np.float32(0.25) / np.float32(0.1875))
    assert g[3] == -g[2]
    # scaling by n is one more rounding of the denominator: exact for powers of two
    np.testing.assert_array_equal(oracle.bce_grad(p, y, 1024.0), g / 1024)


def test_matches_torch_autograd_fp64():
    n = 200_000
    p, y = synth.bce_inputs(81, 0, 0, n)
    g = oracle.bce_grad(p, y, float(n))
    pt = torch.from_numpy(p.astype(np.float64)).requires_grad_(True)
    loss = torch.nn.functional.binary_cross_entropy(pt, torch.from_numpy(y.astype(np.float64)), reduction="mean")
    loss.backward()
    ref = pt.grad.numpy()
    rel = np.abs(g.astype(np.float64) - ref) / np.abs(ref)
    assert rel.max() <= 8 * 2.0**-24, rel.max()
    # the sign follows the target: y = 1 pulls p up (negative gradient)
    assert ((g < 0) == (y == 1)).all()


def test_inputs_recipe():
    p, y = synth.bce_inputs(82, 3, 1, 10_000)
    assert p.dtype == np.float32 and (p >= 0.02).all() and (p < 0.98).all()
    assert set(np.unique(y)) == {0.0, 1.0}
    assert 0.45 < y.mean() < 0.55
