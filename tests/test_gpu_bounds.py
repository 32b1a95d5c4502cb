"""Bounds checks of our own (the GPU pool has closed compute-sanitizer): every kernel family at
its first and last occupancy level, on ragged shapes, with every buffer it touches placed inside
a larger allocation whose guard zones are poisoned --

* INPUT guards hold NaN: a read outside the input that reaches a result turns it into NaN, so
  the launch no longer equals the same launch on unguarded buffers (bit for bit);
* OUTPUT guards hold a sentinel bit pattern: a store outside the output changes it;
* the result is compared bit for bit with the unguarded launch (which the parity tests compare
  with the oracle) and must be finite.

Covers the staged tiles' clamp-to-edge reads, row bands read from exactly-sized slabs (the C5 /
kernel-splitting launch shape), the fan-out epilogue's stores into another image, the stencils'
cp.async rings, SRAD's statistics slots behind the grid, and chained iterations."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

G = 8192                       # guard floats on each side (32 KiB)
SENT = -7.25e30                # output guard sentinel (finite, never a result)


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


class Guarded:
    """n floats inside [G guard | n | G guard] of one allocation."""

    def __init__(self, n, guard_value, data=None):
        self.buf = torch.full((G + n + G,), guard_value, device="cuda", dtype=torch.float32)
        self.n = n
        self.inner = self.buf[G:G + n]
        if data is not None:
            self.inner.copy_(data.reshape(-1))
        self.guard_value = guard_value

    def ptr(self):
        return self.inner.data_ptr()

    def guards_intact(self):
        lo, hi = self.buf[:G], self.buf[G + self.n:]
        if np.isnan(self.guard_value):
            return bool(torch.isnan(lo).all() and torch.isnan(hi).all())
        return bool((lo == self.guard_value).all() and (hi == self.guard_value).all())


def _sp():
    return torch.cuda.current_stream().cuda_stream


DENOISERS = [("knn_f4", 3), ("knn_f4_p1", 3), ("knn_f4_t16", 3), ("nlm_f4", 6), ("nlm_f4_w", 6),
             ("nlm_f4_direct", 6), ("nlm_f4_regheavy", 6)]
FANOUT = ("knn_f4", "knn_f4_p1", "knn_f4_t16", "nlm_f4", "nlm_f4_w")


@pytest.mark.parametrize("kernel,halo", DENOISERS)
@pytest.mark.parametrize("W,H", [(70, 45), (129, 24), (1, 1), (3, 130)])
def test_denoiser_stays_in_bounds(dev, kernel, halo, W, H):
    sp = _sp()
    v, _ = O.build_all_levels(0, kernel)
    img = torch.from_numpy(synth.noisy_rgba(W, H, seed=5, sigma=0.13)).cuda()
    for lvl in sorted({0, len(v) - 1}):
        ref = torch.empty_like(img)
        v.launch(lvl, O.denoise_args(kernel, img.data_ptr(), ref.data_ptr(), W, H), sp)
        src = Guarded(img.numel(), float("nan"), img)
        dst = Guarded(img.numel(), SENT)
        fan = Guarded(img.numel(), SENT) if kernel in FANOUT else None
        a = O.denoise_args(kernel, src.ptr(), dst.ptr(), W, H)
        if fan is not None:
            a = O.with_fanout(a, [fan.ptr()])
        v.launch(lvl, a, sp)
        torch.cuda.synchronize()
        out = dst.inner.view(H, W, 4)
        assert dst.guards_intact() and src.guards_intact(), (kernel, lvl, "store outside the output")
        assert torch.isfinite(out).all(), (kernel, lvl, "a read outside the input reached a result")
        assert torch.equal(out, ref), (kernel, lvl)
        if fan is not None:
            assert fan.guards_intact(), (kernel, lvl, "fan-out store outside the image")
            assert torch.equal(fan.inner.view(H, W, 4), ref), (kernel, lvl)


@pytest.mark.parametrize("kernel,halo", DENOISERS)
def test_denoiser_band_from_exact_slab_in_bounds(dev, kernel, halo):
    """A row band [r0, r1) read from a slab of exactly rows [r0 - halo, r1 + halo) (clamped to the
    image), written to an exactly-sized band buffer: the kernel-splitting / C5 launch shape."""
    sp = _sp()
    W, H = 131, 77
    v, _ = O.build_all_levels(0, kernel)
    img = torch.from_numpy(synth.noisy_rgba(W, H, seed=6, sigma=0.13)).cuda()
    ref = torch.empty_like(img)
    v.launch(len(v) - 1, O.denoise_args(kernel, img.data_ptr(), ref.data_ptr(), W, H), sp)
    for r0, r1 in ((0, 9), (9, 40), (40, 77), (76, 77), (5, 6)):
        s0, s1 = max(0, r0 - halo), min(H, r1 + halo)
        for lvl in sorted({0, len(v) - 1}):
            slab = Guarded((s1 - s0) * W * 4, float("nan"), img[s0:s1])
            band = Guarded((r1 - r0) * W * 4, SENT)
            v.launch(lvl, O.denoise_args(kernel, slab.ptr(), band.ptr(), W, H, r0, r1, s0, s1, r0), sp)
            torch.cuda.synchronize()
            got = band.inner.view(r1 - r0, W, 4)
            assert band.guards_intact() and slab.guards_intact(), (kernel, r0, r1, lvl)
            assert torch.equal(got, ref[r0:r1]), (kernel, r0, r1, lvl)


def _thermal(W, H, seed=1):
    t0, p = synth.thermal_inputs(W, H, seed=seed)
    return torch.from_numpy(np.ascontiguousarray(t0)).cuda(), torch.from_numpy(np.ascontiguousarray(p)).cuda()


@pytest.mark.parametrize("kernel", ["hotspot_f32", "hotspot2h_f32", "hotspot4h_f32"])
@pytest.mark.parametrize("W,H", [(132, 37), (8, 3), (516, 130), (4, 1)])
def test_hotspot_stays_in_bounds(dev, kernel, W, H):
    sp = _sp()
    v, _ = O.build_all_levels(0, kernel)
    t0, p = _thermal(W, H)
    for lvl in sorted({0, len(v) - 1}):
        ref = torch.empty_like(t0)
        v.launch(lvl, O.hotspot_args(t0.data_ptr(), ref.data_ptr(), p.data_ptr(), W, H), sp)
        gt, gp, go = Guarded(W * H, float("nan"), t0), Guarded(W * H, float("nan"), p), Guarded(W * H, SENT)
        v.launch(lvl, O.hotspot_args(gt.ptr(), go.ptr(), gp.ptr(), W, H), sp)
        torch.cuda.synchronize()
        assert go.guards_intact() and gt.guards_intact() and gp.guards_intact(), (kernel, lvl)
        out = go.inner.view(H, W)
        assert torch.isfinite(out).all(), (kernel, lvl)
        assert torch.equal(out, ref), (kernel, lvl)


def test_hotspot4h_band_from_exact_slab_in_bounds(dev):
    """A C3 row band read from exactly its rows plus 4 halo rows per side (P:L691 kernel splitting,
    the row-sharded C3 shape)."""
    sp = _sp()
    W, H, S = 264, 90, 4
    v, _ = O.build_all_levels(0, "hotspot4h_f32")
    t0, p = _thermal(W, H, seed=2)
    ref = torch.empty_like(t0)
    v.launch(0, O.hotspot_args(t0.data_ptr(), ref.data_ptr(), p.data_ptr(), W, H), sp)
    for r0, r1 in ((0, 13), (13, 70), (70, 90), (45, 46)):
        s0, s1 = max(0, r0 - S), min(H, r1 + S)
        for lvl in sorted({0, len(v) - 1}):
            gt = Guarded((s1 - s0) * W, float("nan"), t0[s0:s1])
            gp = Guarded((s1 - s0) * W, float("nan"), p[s0:s1])
            go = Guarded((r1 - r0) * W, SENT)
            a = O.hotspot_args(gt.ptr(), go.ptr(), gp.ptr(), W, H, r0, r1, src_row_begin=s0, src_row_end=s1,
                               dst_row_begin=r0)
            v.launch(lvl, a, sp)
            torch.cuda.synchronize()
            assert go.guards_intact() and gt.guards_intact() and gp.guards_intact(), (r0, r1, lvl)
            assert torch.equal(go.inner.view(r1 - r0, W), ref[r0:r1]), (r0, r1, lvl)


@pytest.mark.parametrize("kernel", ["srad_f32", "srad_f32h", "srad_f32_tile"])
@pytest.mark.parametrize("W,H", [(132, 37), (129, 5), (8, 2)])
def test_srad_stays_in_bounds(dev, kernel, W, H):
    if kernel == "srad_f32h" and W % 4:
        pytest.skip("srad_f32h takes widths % 4 == 0")
    sp = _sp()
    v, _ = O.build_all_levels(0, kernel)
    j, _ = _thermal(W, H, seed=3)
    q0 = torch.empty(1, device="cuda")
    O.srad_roi_stats(0, j.data_ptr(), W, H, (0, min(H, 20) - 1, 0, min(W, 20) - 1), q0.data_ptr(), sp)
    for lvl in sorted({0, len(v) - 1}):
        ref = torch.empty_like(j)
        v.launch(lvl, O.srad_args(j.data_ptr(), ref.data_ptr(), q0.data_ptr(), W, H), sp)
        gj, go = Guarded(W * H, float("nan"), j), Guarded(W * H, SENT)
        gq = Guarded(1, float("nan"), q0)
        v.launch(lvl, O.srad_args(gj.ptr(), go.ptr(), gq.ptr(), W, H), sp)
        torch.cuda.synchronize()
        assert go.guards_intact() and gj.guards_intact() and gq.guards_intact(), (kernel, lvl)
        out = go.inner.view(H, W)
        assert torch.isfinite(out).all(), (kernel, lvl)
        assert torch.equal(out, ref), (kernel, lvl)


@pytest.mark.parametrize("W,H,roi", [(132, 37, (2, 30, 100, 131)), (252, 100, (0, 99, 0, 251)),
                                     (8, 3, (0, 2, 0, 7))])
def test_srad_fused_statistics_in_bounds(dev, W, H, roi):
    """srad_f32hs reads the statistics slots behind its input grid and writes those behind its output
    grid: the slot area is part of each guarded buffer, the guards start after it."""
    sp = _sp()
    v, _ = O.build_all_levels(0, "srad_f32hs")
    j, _ = _thermal(W, H, seed=4)
    n = W * H + O.SRAD_STATS_FLOATS
    for lvl in sorted({0, len(v) - 1}):
        a_ref = torch.zeros(n, device="cuda")
        a_ref[:W * H] = j.reshape(-1)
        b_ref = torch.zeros(n, device="cuda")
        O.srad_stats_init(0, a_ref.data_ptr(), W, H, roi, sp)
        v.launch(lvl, O.srad_args(a_ref.data_ptr(), b_ref.data_ptr(), 0, W, H, roi=roi), sp)
        ga = Guarded(n, float("nan"))
        ga.inner.zero_()
        ga.inner[:W * H] = j.reshape(-1)
        gb = Guarded(n, SENT)
        O.srad_stats_init(0, ga.ptr(), W, H, roi, sp)
        v.launch(lvl, O.srad_args(ga.ptr(), gb.ptr(), 0, W, H, roi=roi), sp)
        torch.cuda.synchronize()
        assert gb.guards_intact() and ga.guards_intact(), lvl
        assert torch.isfinite(gb.inner[:W * H]).all(), lvl
        assert torch.equal(gb.inner[:W * H], b_ref[:W * H]), lvl


@pytest.mark.parametrize("kernel", ["hotspot4h_f32", "srad_f32hs"])
def test_chained_iterations_in_bounds(dev, kernel):
    """orion_chain: 12 chained launches over several tiles in both directions ping-ponging between
    two guarded grids == the same launches on plain buffers, unchained."""
    sp = _sp()
    W, H = 252, 1100
    v, _ = O.build_all_levels(0, kernel)
    t0, p = _thermal(W, H, seed=7)
    extra = O.SRAD_STATS_FLOATS if kernel == "srad_f32hs" else 0
    roi = (300, 700, 100, 200)
    n = W * H + extra

    def run(bufs, pw, chain):
        a, b = bufs
        if extra:
            O.srad_stats_init(0, a, W, H, roi, sp)
        for it in range(12):
            lvl = it % len(v)
            if kernel == "srad_f32hs":
                args = O.srad_args(a, b, 0, W, H, roi=roi, chain=chain)
            else:
                args = O.hotspot_args(a, b, pw, W, H, chain=chain)
            v.launch(lvl, args, sp)
            a, b = b, a
        return a

    pa, pb = torch.zeros(n, device="cuda"), torch.zeros(n, device="cuda")
    pa[:W * H] = t0.reshape(-1)
    ref_ptr = run((pa.data_ptr(), pb.data_ptr()), p.data_ptr(), None)
    ref = (pa if ref_ptr == pa.data_ptr() else pb)[:W * H].clone()
    ga, gb = Guarded(n, float("nan")), Guarded(n, float("nan"))
    ga.inner.zero_()
    gb.inner.zero_()
    ga.inner[:W * H] = t0.reshape(-1)
    gp = Guarded(W * H, float("nan"), p)
    ch = O.Chain(v, W, H)
    got_ptr = run((ga.ptr(), gb.ptr()), gp.ptr(), ch)
    torch.cuda.synchronize()
    ch.close()
    got = (ga if got_ptr == ga.ptr() else gb).inner[:W * H]
    assert ga.guards_intact() and gb.guards_intact() and gp.guards_intact()
    assert torch.isfinite(got).all()
    assert torch.equal(got, ref)
