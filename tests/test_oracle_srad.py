"""Pins for oracle O5 -- SRAD (Table 2, Fig. 10; update rule per
reading R-SRAD = Rodinia srad_v2, ref [6] P:L1147, since the paper gives no formula).

Pinned against invariants, not its own loop:
  * the update is in divergence form with zero-flux borders: sum(J) is conserved;
  * maximum principle (c in [0,1], lambda <= 1): min/max never leave the initial range;
  * lambda = 0 is the identity; ROI statistics equal numpy's mean / variance;
  * transpose equivariance: the flux between two cells uses the south / east cell's
    coefficient, so transposing the image (and the ROI) transposes the result; a mirror
    does not (the discretisation is one-sided), which the test also checks.
"""
import numpy as np
import pytest

import oracle
import synth


def _img(W, H, seed=1):
    # SRAD works on positive intensities (ultrasound-like speckle): exp of a noisy field
    t0, _ = synth.thermal_inputs(W, H, seed=seed)
    return np.exp((t0.astype(np.float64) - 323.15) / 20.0)


def test_conservation_and_maximum_principle():
    j0 = _img(50, 40)
    j, q0 = oracle.srad(j0, 30, 0.5, (0, 19, 0, 19))
    assert j.sum() == pytest.approx(j0.sum(), rel=1e-12)
    assert j.min() >= j0.min() - 1e-12 and j.max() <= j0.max() + 1e-12
    assert j.std() < j0.std()          # it diffuses
    assert (q0 > 0).all()


def test_lambda_zero_is_identity():
    j0 = _img(33, 21)
    j, _ = oracle.srad(j0, 5, 0.0, (0, 9, 0, 9))
    np.testing.assert_array_equal(j, j0)


def test_roi_statistics_match_numpy():
    j0 = _img(40, 30, seed=3)
    _, q0 = oracle.srad(j0, 1, 0.5, (2, 17, 5, 30))
    roi = j0[2:18, 5:31]
    assert q0[0] == pytest.approx(roi.var() / roi.mean() ** 2, rel=1e-10)


def test_transpose_equivariance_and_one_sided_flux():
    j0 = _img(30, 24, seed=5)
    a, _ = oracle.srad(j0, 10, 0.5, (2, 15, 4, 20))
    c, _ = oracle.srad(np.ascontiguousarray(j0.T), 10, 0.5, (4, 20, 2, 15))
    np.testing.assert_allclose(c.T, a, rtol=1e-12)
    b, _ = oracle.srad(np.ascontiguousarray(j0[:, ::-1]), 10, 0.5, (2, 15, 9, 25))
    assert not np.allclose(b[:, ::-1], a, rtol=1e-9)
