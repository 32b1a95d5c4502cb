"""SRAD on the GPU (NEXT-4; Table 2, Fig. 10): every occupancy level
realised and bit-exact to every other, the ROI statistics against numpy, and the iterated
update against the double oracle O5 (reading R-SRAD)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

ROI = (0, 127, 0, 127)


class Built(tuple):
    """(variants, resources) plus the kernel id."""


@pytest.fixture(scope="module", params=["srad_f32", "srad_f32h"])
def srad(request):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    b = Built(O.build_all_levels(0, request.param, mode=O.REALISE_MIN_CARVEOUT))
    b.kernel = request.param
    return b


def aligned(srad, W):
    """srad_f32h needs width % 4 == 0 (float4 lanes only)."""
    return W + (-W % 4) if srad.kernel == "srad_f32h" else W


def run(v, level, j0, iters, lam=0.5, roi=ROI):
    sp = torch.cuda.current_stream().cuda_stream
    H, W = j0.shape
    a = torch.from_numpy(np.ascontiguousarray(j0, dtype=np.float32)).cuda()
    b = torch.empty_like(a)
    q0 = torch.empty(1, device="cuda")
    qs = []
    for _ in range(iters):
        O.srad_roi_stats(0, a.data_ptr(), W, H, roi, q0.data_ptr(), sp)
        qs.append(q0.clone())
        v.launch(level, O.srad_args(a.data_ptr(), b.data_ptr(), q0.data_ptr(), W, H, lam), sp)
        a, b = b, a
    torch.cuda.synchronize()
    return a.cpu().numpy(), [float(q) for q in qs]


def test_levels_verified_and_ladder_per_fig8(srad):
    from oracle import occupancy as OC
    from oracle import tuner as OT
    v, res = srad
    t = O.Tuner(v)
    d, ladder = t.ladder()
    ol = OC.levels(OC.B200, res.block_threads, res.regs_per_thread, res.static_smem_bytes, res.dyn_smem_bytes,
                   mode=OC.REALISE_MIN_CARVEOUT)
    od, oladder, _ = OT.candidates(ol, res.regs_per_thread, OT.TunerCfg())
    assert d == od and [v.level(i).ctas_per_sm for i in ladder] == [ol[i].ctas_per_sm for i in oladder]
    for i in range(len(v)):
        assert v.info(i).verified_ctas == v.level(i).ctas_per_sm


def test_bit_exact_across_levels_and_vs_oracle(srad):
    v, _ = srad
    t0, _ = synth.thermal_inputs(300, 203, seed=2)
    outs = [run(v, i, t0, 12)[0] for i in range(len(v))]
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    ref, _ = oracle.srad(t0.astype(np.float64), 12, 0.5, ROI)
    rel = np.abs(outs[0] - ref) / np.abs(ref)
    assert rel.max() < 1e-5, rel.max()
    # divergence form with zero-flux borders: total intensity conserved to fp32 rounding
    assert abs(outs[0].astype(np.float64).sum() - t0.astype(np.float64).sum()) < 1e-6 * t0.sum()


def test_tile_and_sliding_kernels_identical(srad):
    vt, _ = O.build_all_levels(0, "srad_f32_tile", mode=O.REALISE_MIN_CARVEOUT)
    t0, _ = synth.thermal_inputs(aligned(srad, 257), 190, seed=8)
    a, _ = run(srad[0], len(srad[0]) - 1, t0, 6)
    b, _ = run(vt, 0, t0, 6)
    assert np.array_equal(a, b)


def test_roi_statistics(srad):
    t0, _ = synth.thermal_inputs(200, 150, seed=7)
    _, qs = run(srad[0], 0, t0, 1, roi=(3, 120, 10, 170))
    roi = t0[3:121, 10:171].astype(np.float64)
    assert qs[0] == pytest.approx(roi.var() / roi.mean() ** 2, rel=1e-6)


@pytest.mark.parametrize("shape", [(33, 17), (129, 130), (1, 64)])
def test_ragged_shapes(srad, shape):
    W, H = aligned(srad, shape[0]), shape[1]
    t0, _ = synth.thermal_inputs(W, H, seed=3)
    roi = (0, H - 1, 0, W - 1)
    g, _ = run(srad[0], len(srad[0]) - 1, t0, 3, roi=roi)
    ref, _ = oracle.srad(t0.astype(np.float64), 3, 0.5, roi)
    assert np.max(np.abs(g - ref) / np.abs(ref)) < 1e-5


# ---- srad_f32hs: the ROI statistics fused into the update (slots behind the grids) -------------
def run_fused(v, level, j0, iters, lam=0.5, roi=ROI):
    sp = torch.cuda.current_stream().cuda_stream
    H, W = j0.shape
    n = H * W + O.SRAD_STATS_FLOATS
    a = torch.zeros(n, device="cuda")
    b = torch.zeros(n, device="cuda")
    a[:H * W] = torch.from_numpy(np.ascontiguousarray(j0, dtype=np.float32).ravel()).cuda()
    O.srad_stats_init(0, a.data_ptr(), W, H, roi, sp)
    q0s = []
    for _ in range(iters):
        q0s.append(_q0_of_slots(a, H, W, roi))
        v.launch(level, O.srad_args(a.data_ptr(), b.data_ptr(), 0, W, H, lam, roi=roi), sp)
        a, b = b, a
    torch.cuda.synchronize()
    return a[:H * W].reshape(H, W).cpu().numpy(), q0s, a


def _q0_of_slots(buf, H, W, roi):
    """q0sqr from the statistics slots behind a grid (the kernel reduces them the same way)."""
    torch.cuda.synchronize()
    tail = buf[H * W:].cpu().numpy().view(np.float64).reshape(-1, 2)
    r1, r2, c1, c2 = roi
    nslots = (r2 // 42 - r1 // 42 + 1) * (c2 // 120 - c1 // 120 + 1)
    s, s2 = tail[:nslots, 0].sum(), tail[:nslots, 1].sum()
    n = (r2 - r1 + 1) * (c2 - c1 + 1)
    mean = s / n
    return (s2 / n - mean * mean) / (mean * mean)


@pytest.fixture(scope="module")
def fused():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return O.build_all_levels(0, "srad_f32hs", mode=O.REALISE_MIN_CARVEOUT)


@pytest.mark.parametrize("roi", [ROI, (5, 150, 100, 290), (0, 202, 0, 299), (60, 60, 7, 7)])
def test_fused_stats_vs_oracle_all_levels(fused, roi):
    v, _ = fused
    t0, _ = synth.thermal_inputs(300, 203, seed=2)
    outs = []
    for i in range(len(v)):
        o, q0s, _ = run_fused(v, i, t0, 12, roi=roi)
        outs.append(o)
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])                       # bit-exact across levels
    ref, q0_ref = oracle.srad(t0.astype(np.float64), 12, 0.5, roi)
    assert np.max(np.abs(outs[0] - ref) / np.abs(ref)) < 1e-5
    # the slots reproduce the ROI statistics of every iteration's input (double partial sums)
    _, q0s, _ = run_fused(v, len(v) - 1, t0, 12, roi=roi)
    np.testing.assert_allclose(q0s, q0_ref, rtol=1e-5)


def test_fused_stats_slots_equal_a_fused_launch(fused):
    # orion_srad_stats_init writes exactly the slots a fused launch stores for the same grid: run
    # one iteration, then re-initialise the slots of its output and compare them bit for bit
    v, _ = fused
    t0, _ = synth.thermal_inputs(256, 130, seed=5)
    roi = (3, 100, 10, 250)
    _, _, out = run_fused(v, 0, t0, 1, roi=roi)
    H, W = 130, 256
    launched = out[H * W:].clone()
    O.srad_stats_init(0, out.data_ptr(), W, H, roi, torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    assert torch.equal(out[H * W:], launched)


def test_fused_matches_unfused_kernel(fused, srad):
    # the fused and the separate-statistics forms compute q0sqr in double in different orders;
    # rounded to float they agree, so the grids stay within 1e-6 of each other
    v, _ = fused
    t0, _ = synth.thermal_inputs(aligned(srad, 300), 203, seed=3)
    a, _, _ = run_fused(v, len(v) - 1, t0, 8)
    b, _ = run(srad[0], len(srad[0]) - 1, t0, 8)
    assert np.max(np.abs(a - b) / np.abs(b)) < 1e-6


def test_fused_whole_grid_8192(fused):
    v, _ = fused
    W = H = 8192
    sp = torch.cuda.current_stream().cuda_stream
    a = torch.zeros(H * W + O.SRAD_STATS_FLOATS, device="cuda")
    b = torch.zeros_like(a)
    pw = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, a.data_ptr(), pw.data_ptr(), W, H, seed=1, stream=sp)
    O.srad_stats_init(0, a.data_ptr(), W, H, ROI, sp)
    lvl = max((i for i, l in enumerate(v.planned) if l.reg_cap == 0), key=lambda i: v.planned[i].ctas_per_sm)
    for _ in range(2):
        v.launch(lvl, O.srad_args(a.data_ptr(), b.data_ptr(), 0, W, H, roi=ROI), sp)
        a, b = b, a
    torch.cuda.synchronize()
    t0, _ = synth.thermal_inputs(W, H, seed=1)
    ref, _ = oracle.srad(t0.astype(np.float64), 2, 0.5, ROI)
    assert np.max(np.abs(a[:H * W].reshape(H, W).cpu().numpy() - ref) / ref) < 1e-5


def test_fused_rejects_bad_roi(fused):
    v, _ = fused
    a = torch.zeros(64 * 64 + O.SRAD_STATS_FLOATS, device="cuda")
    sp = torch.cuda.current_stream().cuda_stream
    with pytest.raises(O.OrionError):
        v.launch(0, O.srad_args(a.data_ptr(), a.data_ptr(), 0, 64, 64, roi=(0, 64, 0, 10)), sp)   # r2 >= H
    with pytest.raises(O.OrionError):
        O.srad_stats_init(0, a.data_ptr(), 64, 64, (0, 10, 5, 4), sp)                            # c2 < c1
