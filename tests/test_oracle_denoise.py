"""Pins for oracle O2 -- imageDenoising KNN / NLM (Table 2 P:L733;
math per reading R-O2, the CUDA-SDK sample [20] P:L1175, since the paper gives none).

Pinned against things other than the oracle's own loop:
  * constant image -> identity; Noise -> inf -> identity (closed forms);
  * a gray impulse on black: closed-form value at the impulse pixel for KNN
    (each neighbour at squared distance 3v^2) and NLM (two patch terms of 3v^2);
  * flip / transpose equivariance (clamp-to-edge and the window are symmetric);
  * an independent array formulation (edge-padded shifted copies, numpy) on
    tiny images, which fails on a wrong offset sign, a transposed patch or a
    dropped geometric term.
"""
import math

import numpy as np
import pytest

import oracle
import synth


def _img(W, H, seed=3, sigma=0.2):
    return synth.noisy_rgba(W, H, seed=seed, sigma=sigma)


def numpy_reference(kind, img):
    """Independent vectorised formulation: shifted edge-padded planes."""
    P = oracle.KNN if kind == "knn" else oracle.NLM
    R, B = P["R"], P["B"]
    A = (2 * R + 1) ** 2
    H, W = img.shape[:2]
    rgb = img[..., :3].astype(np.float64)
    pad = R + B
    big = np.pad(rgb, ((pad, pad), (pad, pad), (0, 0)), mode="edge")

    def shifted(dy, dx):  # plane q(y, x) = p(x + dx, y + dy)
        return big[pad + dy: pad + dy + H, pad + dx: pad + dx + W]

    c00 = shifted(0, 0)
    acc = np.zeros_like(rgb)
    sw = np.zeros((H, W))
    cnt = np.zeros((H, W), np.int64)
    for i in range(-R, R + 1):
        for j in range(-R, R + 1):
            if kind == "knn":
                d = ((shifted(i, j) - c00) ** 2).sum(-1)
            else:
                d = np.zeros((H, W))
                for n in range(-B, B + 1):
                    for m in range(-B, B + 1):
                        d += ((shifted(i + n, j + m) - shifted(n, m)) ** 2).sum(-1)
            w = np.exp(-(d * P["noise"] + (i * i + j * j) / A))
            acc += w[..., None] * shifted(i, j)
            sw += w
            cnt += w > P["wthr"]
    clr = acc / sw[..., None]
    q = np.where(cnt / A > P["lthr"], P["lerpc"], 1 - P["lerpc"])[..., None]
    return clr + (c00 - clr) * q


@pytest.mark.parametrize("kind", ["knn", "nlm"])
def test_independent_array_formulation(kind):
    img = _img(13, 11, seed=5, sigma=0.13 if kind == "nlm" else 0.2)
    out, alt, amb = oracle.denoise(kind, img)
    ref = numpy_reference(kind, img)
    ok = np.isclose(out, ref, atol=1e-12).all(-1) | (amb & np.isclose(alt, ref, atol=1e-12).all(-1))
    assert ok.all()


@pytest.mark.parametrize("kind", ["knn", "nlm"])
def test_constant_image_is_identity(kind):
    img = np.zeros((9, 12, 4), np.float32)
    img[..., :3] = (0.3, 0.55, 0.8)
    img[..., 3] = 1
    out, _, amb = oracle.denoise(kind, img)
    assert not amb.any()
    np.testing.assert_allclose(out, np.broadcast_to(img[..., :3], out.shape), atol=1e-14)


@pytest.mark.parametrize("kind", ["knn", "nlm"])
def test_infinite_noise_is_identity(kind):
    img = _img(10, 9, seed=7)
    out, _, _ = oracle.denoise(kind, img, params={"noise": 1e30})
    np.testing.assert_allclose(out, img[..., :3], atol=1e-14)


@pytest.mark.parametrize("kind", ["knn", "nlm"])
def test_flip_and_transpose_equivariance(kind):
    img = _img(12, 12, seed=11, sigma=0.13)
    out, _, amb = oracle.denoise(kind, img)
    for f in (lambda a: a[:, ::-1], lambda a: a[::-1], lambda a: a.swapaxes(0, 1)):
        o2, _, amb2 = oracle.denoise(kind, np.ascontiguousarray(f(img)))
        sel = ~(amb | f(amb2))
        np.testing.assert_allclose(o2[f(sel)], f(out)[f(sel)], atol=1e-12)


@pytest.mark.parametrize("kind,v", [("knn", 0.05), ("knn", 0.12), ("knn", 0.5), ("nlm", 0.3), ("nlm", 0.6),
                                    ("nlm", 1.0)])
def test_impulse_closed_form(kind, v):
    P = oracle.KNN if kind == "knn" else oracle.NLM
    img = np.zeros((17, 17, 4), np.float32)
    img[8, 8, :3] = v
    v = float(np.float32(v))
    # every neighbour differs from the centre by (v,v,v): KNN d = 3v^2; NLM: the impulse
    # appears once in each of the two patches -> d = 2 * 3v^2.
    d = 3 * v * v * (1 if kind == "knn" else 2)
    ws = [math.exp(-(d * P["noise"] + (i * i + j * j) / 49.0))
          for i in range(-3, 4) for j in range(-3, 4) if (i, j) != (0, 0)]
    clr = v / (1.0 + sum(ws))
    cnt = 1 + sum(w > P["wthr"] for w in ws)
    q = P["lerpc"] if cnt / 49.0 > P["lthr"] else 1 - P["lerpc"]
    want = clr + (v - clr) * q
    out, _, amb = oracle.denoise_points(kind, img, [8], [8])
    assert not amb[0]
    np.testing.assert_allclose(out[0], [want] * 3, rtol=0, atol=1e-14)


def test_points_match_rows_and_slabs():
    W, H = 40, 30
    img = _img(W, H, seed=2, sigma=0.13)
    full, _, _ = oracle.denoise("nlm", img)
    xs = np.array([0, 39, 5, 20, 0, 39])
    ys = np.array([0, 29, 14, 7, 29, 0])
    pts, _, _ = oracle.denoise_points("nlm", img, xs, ys)
    np.testing.assert_array_equal(pts, full[ys, xs])
    # a slab holding only the rows the window reaches (row-sharding, reading R-A16)
    slab = img[4:26]
    part, _, _ = oracle.denoise("nlm", slab, height=H, row0=4, y_begin=10, y_end=20)
    np.testing.assert_array_equal(part, full[10:20])


def test_ambiguous_pixels_are_rare_and_branches_differ():
    img = _img(64, 64, seed=1, sigma=0.2)
    out, alt, amb = oracle.denoise("knn", img)
    assert amb.mean() < 0.01
    if amb.any():
        assert not np.allclose(out[amb], alt[amb])
    assert np.array_equal(out[~amb], alt[~amb])
