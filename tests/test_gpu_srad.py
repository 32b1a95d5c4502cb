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
