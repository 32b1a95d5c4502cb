"""orion_tune_run_host: a whole stencil run from HOST grids (copy in, tuned iterations, copy
out; the Rodinia driver shape, PAPER.md P:L731 / P:L739) -- bit-identical to the oracle's fp32
hotspot form and within the SRAD tolerance of the double oracle, with the tuner exploring
levels inside the run (the iterations Fig. 9 tunes across, P:L651-P:L653)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


def _pinned(x):
    return torch.from_numpy(np.ascontiguousarray(x, dtype=np.float32)).pin_memory()


def _run(kernel, t0, pw, iterations, roi=None):
    H, W = t0.shape
    v, _ = O.build_all_levels(0, kernel, mode=O.REALISE_MIN_CARVEOUT)
    tuner = O.Tuner(v)
    hs, hout = _pinned(t0), torch.empty((H, W), dtype=torch.float32).pin_memory()
    extra = O.SRAD_STATS_FLOATS if kernel == "srad_f32hs" else 0    # statistics slots behind the grids
    da, db = torch.empty(H * W + extra, device="cuda"), torch.empty(H * W + extra, device="cuda")
    if kernel.startswith("srad"):
        aux = torch.empty(1, device="cuda")
        args = O.srad_args(hs.data_ptr(), hout.data_ptr(), 0, W, H)
    else:
        hp = _pinned(pw)
        aux = torch.empty((H, W), device="cuda")
        args = O.hotspot_args(hs.data_ptr(), hout.data_ptr(), hp.data_ptr(), W, H)
    sp = torch.cuda.current_stream().cuda_stream
    h2d, d2h = tuner.run_host(args, iterations, da.data_ptr(), db.data_ptr(), aux.data_ptr(), roi, sp)
    return hout.numpy().copy(), h2d, d2h, tuner


@pytest.mark.parametrize("kernel,shape,launches,steps", [("hotspot_f32", (300, 203), 9, 9),
                                                          ("hotspot_f32", (97, 1), 4, 4),
                                                          ("hotspot2h_f32", (244, 131), 6, 12),
                                                          ("hotspot4h_f32", (244, 131), 5, 20)])
def test_hotspot_run_host_bit_exact(dev, kernel, shape, launches, steps):
    W, H = shape
    t0, pw = synth.thermal_inputs(W, H, seed=4)
    out, h2d, d2h, _ = _run(kernel, t0, pw, launches)
    assert np.array_equal(out, oracle.hotspot(t0, pw, steps, precision="f32"))
    assert h2d == 2 * W * H * 4 and d2h == W * H * 4


@pytest.mark.parametrize("kernel", ["srad_f32", "srad_f32hs"])
def test_srad_run_host_vs_oracle(dev, kernel):
    W, H = 260, 190
    t0, _ = synth.thermal_inputs(W, H, seed=6)
    roi = (0, 127, 0, 127)
    out, h2d, d2h, _ = _run(kernel, t0, None, 10, roi)
    ref, _ = oracle.srad(t0.astype(np.float64), 10, 0.5, roi)
    assert np.max(np.abs(out - ref) / np.abs(ref)) < 1e-5
    assert h2d == W * H * 4 and d2h == W * H * 4


def test_run_host_rejects_bad_calls(dev):
    t0, pw = synth.thermal_inputs(64, 32, seed=1)
    with pytest.raises(O.OrionError) as e:       # srad needs the ROI
        _run("srad_f32", t0, None, 2, None)
    assert e.value.status == -1
    v, _ = O.build_all_levels(0, "knn_f4")
    img = torch.zeros((8, 8, 4)).pin_memory()
    d = torch.empty((8, 8, 4), device="cuda")
    with pytest.raises(O.OrionError) as e:       # not a stencil kernel
        O.Tuner(v).run_host(O.denoise_args("knn_f4", img.data_ptr(), img.data_ptr(), 8, 8), 1, d.data_ptr(),
                            d.data_ptr(), d.data_ptr())
    assert e.value.status == -1
    v2, _ = O.build_all_levels(0, "hotspot_f32")
    hs = _pinned(t0)
    a = O.hotspot_args(hs.data_ptr(), hs.data_ptr(), hs.data_ptr(), 64, 32, row_begin=8)
    dd = torch.empty((32, 64), device="cuda")
    with pytest.raises(O.OrionError) as e:       # partial row range
        O.Tuner(v2).run_host(a, 1, dd.data_ptr(), dd.data_ptr(), dd.data_ptr())
    assert e.value.status == -1
