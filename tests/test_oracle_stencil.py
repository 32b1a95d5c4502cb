"""Pins for oracle O3 -- the thermal stencil (hotspot, Table 2; Rodinia [6]
P:L1147; update rule per reading R-O3, constants per reading R-A15).

Pinned against closed forms / invariants, not against its own loop:
  * T = amb, P = 0 is an exact fixed point;
  * uniform T, constant P: T_n - amb follows the scalar recursion
    e_{n+1} = (1 - sdc*rz) e_n + sdc*P (geometric closed form);
  * Neumann cosine modes cos(pi k (x+1/2)/W) cos(pi l (y+1/2)/H) are eigenvectors of
    the clamp-to-edge stencil with eigenvalue 1 + sdc(rx(2cos(pi k/W)-2) + ry(2cos(pi l/H)-2) - rz);
  * heat conservation when rz = 0 and P = 0; the maximum principle;
  * the fp32 form stays within the fp32 error bound of the f64 definition.
"""
import math

import numpy as np
import pytest

import oracle
import synth


def test_constants_fixed_cell_size():
    c = oracle.hotspot_constants()
    assert c["rx"] == pytest.approx(0.1) and c["ry"] == pytest.approx(0.1)
    assert c["sdc"] == pytest.approx(0.341333, rel=1e-5)
    assert c["rz"] == pytest.approx(1.953125e-4)
    assert c["sdc"] * c["rx"] < 0.25          # explicit-scheme stability (reading R-A15)


@pytest.mark.parametrize("precision", ["f64", "f32"])
def test_ambient_fixed_point(precision):
    t0 = np.full((9, 13), 80.0)
    out = oracle.hotspot(t0, np.zeros_like(t0), 100, precision=precision)
    assert (out == 80.0).all()


def test_uniform_power_closed_form():
    c = oracle.hotspot_constants()
    P, n = 0.03, 57
    out = oracle.hotspot(np.full((6, 7), 100.0), np.full((6, 7), P), n)
    a = 1.0 - c["sdc"] * c["rz"]
    e = (100.0 - c["amb"]) * a ** n + c["sdc"] * P * (1 - a ** n) / (1 - a)
    np.testing.assert_allclose(out, c["amb"] + e, rtol=1e-13)


@pytest.mark.parametrize("k,l", [(1, 0), (0, 2), (3, 5), (7, 1)])
def test_neumann_cosine_mode_eigenvalue(k, l):
    c = oracle.hotspot_constants()
    W, H, n, A = 24, 20, 40, 5.0
    x = np.arange(W)[None, :]
    y = np.arange(H)[:, None]
    mode = np.cos(math.pi * k * (x + 0.5) / W) * np.cos(math.pi * l * (y + 0.5) / H)
    lam = 1 + c["sdc"] * (c["rx"] * (2 * math.cos(math.pi * k / W) - 2)
                          + c["ry"] * (2 * math.cos(math.pi * l / H) - 2) - c["rz"])
    out = oracle.hotspot(c["amb"] + A * mode, np.zeros((H, W)), n)
    np.testing.assert_allclose(out - c["amb"], A * lam ** n * mode, atol=1e-11)


def test_conservation_without_sink():
    c = dict(oracle.hotspot_constants(), rz=0.0)
    t0, _ = synth.thermal_inputs(31, 17, seed=4)
    out = oracle.hotspot(t0, np.zeros_like(t0), 100, consts=c)
    assert out.sum() == pytest.approx(t0.astype(np.float64).sum(), rel=1e-12)


def test_maximum_principle():
    c = oracle.hotspot_constants()
    t0, _ = synth.thermal_inputs(33, 29, seed=9)
    out = oracle.hotspot(t0, np.zeros_like(t0), 100)
    assert out.min() >= min(t0.min(), c["amb"]) - 1e-9
    assert out.max() <= max(t0.max(), c["amb"]) + 1e-9


def test_f32_form_within_fp32_bound():
    t0, p = synth.thermal_inputs(40, 36, seed=1)
    d = oracle.hotspot(t0, p, 100, precision="f64")
    f = oracle.hotspot(t0, p, 100, precision="f32")
    assert np.max(np.abs(f - d) / np.abs(d)) < 2e-6
