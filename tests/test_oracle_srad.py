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


def _impulse_closed_form(a, delta, n_roi, lam):
    """SRAD (reading R-SRAD: Yu & Acton's instantaneous coefficient of variation, Rodinia
    srad_v2) worked by hand for a constant image J = a with ONE interior cell raised to
    a + delta, the ROI holding that cell and n_roi - 1 cells of value a.

    ROI: mean = a + delta/n, var = delta^2 (n - 1) / n^2, q0^2 = var / mean^2.
    Centre (all four differences -delta, J = a + delta):
        |grad J|^2 / J^2 = 4 delta^2 / J^2,  lap J / J = -4 delta / J
        q^2 = (2 delta^2 - delta^2) / J^2 / (1 - delta / J)^2 = delta^2 / a^2
    A 4-neighbour (one difference +delta, J = a):
        q^2 = (delta^2 / (2 a^2) - delta^2 / (16 a^2)) / (1 + delta / (4 a))^2 = 7 delta^2 / (4 a + delta)^2
    Everything else has q^2 = 0 -> c = (1 + q0^2) / q0^2 > 1 -> clamped to 1 (no flux anyway).
    c(q) = 1 / (1 + (q^2 - q0^2) / (q0^2 (1 + q0^2))).
    Update J' = J + lam/4 (c dN + c_S dS + c dW + c_E dE): the north / west fluxes use the
    cell's own c, the south / east ones the neighbour's.  So
        centre: a + delta - lam/4 delta (2 c_ctr + 2 c_nb)     (its S and E neighbours are 4-neighbours)
        north / west neighbour: a + lam/4 c_ctr delta           (their S / E neighbour is the centre)
        south / east neighbour: a + lam/4 c_nb delta            (their own c, difference +delta)
    """
    n = float(n_roi)
    mean = a + delta / n
    var = delta * delta * (n - 1.0) / (n * n)
    q0 = var / (mean * mean)

    def c(q2):
        return 1.0 / (1.0 + (q2 - q0) / (q0 * (1.0 + q0)))
    c_ctr = c(delta * delta / (a * a))
    c_nb = c(7.0 * delta * delta / (4.0 * a + delta) ** 2)
    return dict(q0=q0, c_ctr=c_ctr, c_nb=c_nb,
                centre=a + delta - lam / 4.0 * delta * (2.0 * c_ctr + 2.0 * c_nb),
                nw=a + lam / 4.0 * c_ctr * delta, se=a + lam / 4.0 * c_nb * delta)


@pytest.mark.parametrize("a,delta,roi,lam", [(1.0, 0.25, (4, 5, 6, 7), 0.5),      # 2x2 ROI
                                              (2.5, -0.4, (3, 5, 5, 7), 0.5),      # 3x3 ROI, a dip
                                              (0.7, 0.1, (4, 4, 6, 9), 1.0)])      # 1x4 ROI
def test_single_cell_perturbation_closed_form(a, delta, roi, lam):
    # Pins the diffusion coefficient itself (G2, L, q^2 and c), which the invariants above do not
    # constrain: a wrong 1/16, a wrong 1 + L/4, a swapped (q^2 - q0^2) or a mirrored one-sided
    # flux each change at least one of the five cells checked here.
    H, W, y0, x0 = 12, 14, 4, 6
    j0 = np.full((H, W), a, np.float64)
    j0[y0, x0] = a + delta
    r1, r2, c1, c2 = roi
    assert r1 <= y0 <= r2 and c1 <= x0 <= c2
    want = _impulse_closed_form(a, delta, (r2 - r1 + 1) * (c2 - c1 + 1), lam)
    assert 0.0 < want["c_ctr"] < 1.0 and 0.0 < want["c_nb"] < 1.0   # not clamped: c is really tested
    j, q0 = oracle.srad(j0, 1, lam, roi)
    assert q0[0] == pytest.approx(want["q0"], rel=1e-12)
    assert j[y0, x0] == pytest.approx(want["centre"], rel=1e-13)
    assert j[y0 - 1, x0] == pytest.approx(want["nw"], rel=1e-13)
    assert j[y0, x0 - 1] == pytest.approx(want["nw"], rel=1e-13)
    assert j[y0 + 1, x0] == pytest.approx(want["se"], rel=1e-13)
    assert j[y0, x0 + 1] == pytest.approx(want["se"], rel=1e-13)
    rest = np.ones((H, W), bool)
    rest[y0, x0] = rest[y0 - 1, x0] = rest[y0 + 1, x0] = rest[y0, x0 - 1] = rest[y0, x0 + 1] = False
    np.testing.assert_array_equal(j[rest], a)


def test_coefficient_is_one_where_q_equals_q0():
    # c(q) = 1 exactly where q^2 = q0^2 (no smoothing at the ROI's own speckle level).  With a
    # 16-cell ROI the neighbour's q^2 = 7 d^2 / (4a + d)^2 meets q0^2 = 15 d^2 / (16a + d)^2 at
    # d = a (16 sqrt7 - 4 sqrt15) / (sqrt15 - sqrt7); there c_nb = 1 and each south / east
    # neighbour gains exactly lam/4 * d.
    a, lam = 1.0, 0.5
    d = a * (16.0 * 7 ** 0.5 - 4.0 * 15 ** 0.5) / (15 ** 0.5 - 7 ** 0.5)
    w = _impulse_closed_form(a, d, 16, lam)
    assert w["c_nb"] == pytest.approx(1.0, rel=1e-12)
    H, W, y0, x0 = 10, 10, 4, 4
    j0 = np.full((H, W), a)
    j0[y0, x0] = a + d
    j, _ = oracle.srad(j0, 1, lam, (2, 5, 3, 6))      # 4 x 4 = 16 ROI cells incl. the centre
    assert j[y0 + 1, x0] == pytest.approx(a + lam / 4.0 * d, rel=1e-11)
    assert j[y0, x0 + 1] == pytest.approx(a + lam / 4.0 * d, rel=1e-11)
