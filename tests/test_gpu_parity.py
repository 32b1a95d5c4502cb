"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars (BASELINE.json north_star):
  * outputs bit-exact across ALL occupancy variants of a kernel (one PTX, caps only);
  * denoisers within 1e-5 absolute of the double oracle on [0,1] pixels, with the
    ambiguous-pixel rule (reading R-AMB) for weights within the fp32 band of a threshold;
  * stencil bit-exact vs the oracle's fp32 form, within 2e-6 relative of its f64 form;
  * level lists verified by the driver's occupancy API (orion_build_variants);
  * generator GPU == numpy bit for bit; row-sharded output == full output bit for bit.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

TOL = 1e-5


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.init()
    return torch.device("cuda:0")


_VARIANTS = {}


def variants(kernel, threads=0):
    key = (kernel, threads)
    if key not in _VARIANTS:
        _VARIANTS[key] = O.build_all_levels(0, kernel, threads)
    return _VARIANTS[key]


def stream():
    return torch.cuda.current_stream().cuda_stream


def to_dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def run_denoise(kernel, img, threads=0, level=None, params=None):
    """Run every level (or one) on img; return list of outputs (H, W, 4) float32."""
    v, _ = variants(kernel, threads)
    H, W = img.shape[:2]
    src = to_dev(img)
    outs = []
    levels = range(len(v)) if level is None else [level]
    for i in levels:
        dst = torch.full((H, W, 4), float("nan"), device="cuda", dtype=torch.float32)
        v.launch(i, O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H, params=params), stream())
        torch.cuda.synchronize()
        outs.append(dst.cpu().numpy())
    return outs


def check_vs_oracle(gpu, out, alt, amb):
    g = gpu[..., :3].astype(np.float64)
    ok = (np.abs(g - out) <= TOL).all(-1) | (amb & (np.abs(g - alt) <= TOL).all(-1))
    bad = np.argwhere(~ok)
    assert bad.size == 0, (len(bad), bad[:5], np.abs(g - out).max())
    assert (gpu[..., 3] == 0).all()
    return int(amb.sum())


def test_query_limits_match_b200(dev):
    d = O.query_limits(0)
    n = O.b200_limits()
    for f, _ in O.DeviceLimits._fields_:
        assert getattr(d, f) == getattr(n, f), f


@pytest.mark.parametrize("kernel,threads", [("knn_f4", 128), ("knn_f4", 64), ("knn_f4", 256), ("knn_f4_p1", 128),
                                            ("knn_f4_t16", 128),
                                            ("nlm_f4", 128),
                                            ("nlm_f4_w", 128), ("nlm_f4_direct", 128), ("nlm_f4_regheavy", 128),
                                            ("hotspot_f32", 256),
                                            ("hotspot_f32", 128), ("hotspot2h_f32", 256),
                                            ("hotspot4h_f32", 256), ("srad_f32", 256)])
def test_every_level_realised_and_verified(dev, kernel, threads):
    v, res = variants(kernel, threads)
    planned = O.levels(O.b200_limits(), res)
    assert len(v) == len(planned) and len(v) >= 1
    assert [v.level(i).ctas_per_sm for i in range(len(v))] == list(range(1, len(v) + 1))
    for i in range(len(v)):
        inf = v.info(i)
        assert inf.verified_ctas == inf.level.ctas_per_sm            # driver occupancy API == k
        if planned[i].reg_cap:
            assert inf.regs <= planned[i].reg_cap


def test_generator_bit_identical(dev):
    W, H = 333, 149
    for seed, sigma in ((1, 0.13), (7, 0.2)):
        full = torch.empty((H, W, 4), device="cuda")
        O.generate_rgba(0, full.data_ptr(), W, H, seed=seed, sigma=sigma, stream=stream())
        slab = torch.empty((40, W, 4), device="cuda")
        O.generate_rgba(0, slab.data_ptr(), W, H, 60, 100, seed=seed, sigma=sigma, stream=stream())
        torch.cuda.synchronize()
        ref = synth.noisy_rgba(W, H, seed=seed, sigma=sigma)
        assert np.array_equal(full.cpu().numpy(), ref)
        assert np.array_equal(slab.cpu().numpy(), ref[60:100])
    t0 = torch.empty((97, 211), device="cuda")
    pw = torch.empty((97, 211), device="cuda")
    O.generate_thermal(0, t0.data_ptr(), pw.data_ptr(), 211, 97, seed=3, stream=stream())
    torch.cuda.synchronize()
    rt, rp = synth.thermal_inputs(211, 97, seed=3)
    assert np.array_equal(t0.cpu().numpy(), rt) and np.array_equal(pw.cpu().numpy(), rp)


@pytest.mark.parametrize("kernel,threads", [("knn_f4", 128), ("knn_f4", 64), ("knn_f4", 256), ("knn_f4_p1", 128),
                                            ("knn_f4_p1", 64), ("knn_f4_t16", 128)])
def test_knn_c1_all_levels(dev, kernel, threads):
    # C1: KNN 64x64 RGBA, radius 3, all feasible occupancy levels vs the oracle
    img = synth.noisy_rgba(64, 64, seed=1, sigma=0.2)
    outs = run_denoise(kernel, img, threads)
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])                               # bit-exact across levels
    out, alt, amb = oracle.denoise("knn", img)
    check_vs_oracle(outs[0], out, alt, amb)


@pytest.mark.parametrize("shape", [(203, 77), (1, 1), (5, 300), (300, 5), (33, 17)])
def test_knn_ragged_and_degenerate(dev, shape):
    W, H = shape
    img = synth.noisy_rgba(W, H, seed=5, sigma=0.2)
    v, _ = variants("knn_f4")
    outs = run_denoise("knn_f4", img, level=len(v) - 1) + run_denoise("knn_f4", img, level=0)
    assert np.array_equal(outs[0], outs[1])
    v1, _ = variants("knn_f4_p1")                     # one pixel per thread: the same bits
    assert np.array_equal(run_denoise("knn_f4_p1", img, level=len(v1) - 1)[0], outs[0])
    out, alt, amb = oracle.denoise("knn", img)
    for k in ("knn_f4_t16",):                        # taps split over 16 lanes: same counts, sums reordered
        vk, _ = variants(k)
        tk = run_denoise(k, img, level=len(vk) - 1) + run_denoise(k, img, level=0)
        assert np.array_equal(tk[0], tk[1])
        check_vs_oracle(tk[0], out, alt, amb)
    check_vs_oracle(outs[0], out, alt, amb)


@pytest.mark.parametrize("kernel", ["nlm_f4", "nlm_f4_w"])
@pytest.mark.parametrize("sigma", [0.05, 0.13, 0.2])
def test_nlm_box_all_levels(dev, sigma, kernel):
    img = synth.noisy_rgba(250, 131, seed=2, sigma=sigma)
    outs = run_denoise(kernel, img)
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    out, alt, amb = oracle.denoise("nlm", img)
    check_vs_oracle(outs[0], out, alt, amb)


@pytest.mark.parametrize("kernel", ["nlm_f4_direct", "nlm_f4_regheavy"])
def test_nlm_direct_forms_all_levels(dev, kernel):
    img = synth.noisy_rgba(97, 45, seed=4, sigma=0.13)
    outs = run_denoise(kernel, img)
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    out, alt, amb = oracle.denoise("nlm", img)
    check_vs_oracle(outs[0], out, alt, amb)


def test_nlm_forms_agree(dev):
    img = synth.noisy_rgba(130, 70, seed=9, sigma=0.13)
    a = run_denoise("nlm_f4", img, level=0)[0]
    b = run_denoise("nlm_f4_regheavy", img, level=0)[0]
    out, alt, amb = oracle.denoise("nlm", img)
    check_vs_oracle(a, out, alt, amb)
    check_vs_oracle(b, out, alt, amb)
    assert np.abs(a - b).max() <= 2 * TOL


def _sample_points(W, H, n, seed):
    rng = np.random.default_rng(seed)
    xs = list(rng.integers(0, W, n)) + [0, W - 1, 0, W - 1, W // 2, 119, 120, 121]
    ys = list(rng.integers(0, H, n)) + [0, 0, H - 1, H - 1, H // 2, 15, 16, 17]
    return np.array(xs), np.array(ys)


@pytest.mark.parametrize("kernel,size", [("nlm_f4", 2048), ("nlm_f4_w", 2048), ("knn_f4", 2048), ("knn_f4_t16", 2048),
                                         ("nlm_f4_regheavy", 4096)])
def test_full_size_sampled(dev, kernel, size):
    # C2 / C4 sizes, launched as bench.py launches them (max-occupancy and original levels)
    W = H = size
    v, _ = variants(kernel)
    src = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, seed=1, sigma=0.13, stream=stream())
    dsts = []
    for i in (0, len(v) - 1):
        dst = torch.empty((H, W, 4), device="cuda")
        v.launch(i, O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H), stream())
        dsts.append(dst)
    torch.cuda.synchronize()
    assert torch.equal(dsts[0], dsts[1])
    xs, ys = _sample_points(W, H, 150, 0)
    img = synth.noisy_rgba(W, H, seed=1, sigma=0.13)
    out, alt, amb = oracle.denoise_points("knn" if kernel.startswith("knn") else "nlm", img, xs, ys)
    g = dsts[0].cpu().numpy()[ys, xs]
    check_vs_oracle(g[None], out[None], alt[None], amb[None])


def _hotspot_run(v, level, t0, pw, steps):
    H, W = t0.shape
    a, b = to_dev(t0), torch.empty_like(to_dev(t0))
    p = to_dev(pw)
    for _ in range(steps):
        v.launch(level, O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H), stream())
        a, b = b, a
    torch.cuda.synchronize()
    return a.cpu().numpy()


@pytest.mark.parametrize("threads", [256, 128])
def test_hotspot_bit_exact_fp32_form_all_levels(dev, threads):
    t0, pw = synth.thermal_inputs(300, 203, seed=2)
    v, _ = variants("hotspot_f32", threads)
    ref = oracle.hotspot(t0, pw, 20, precision="f32")
    for i in range(len(v)):
        assert np.array_equal(_hotspot_run(v, i, t0, pw, 20), ref), i


def test_hotspot_vs_f64_100_steps(dev):
    t0, pw = synth.thermal_inputs(256, 256, seed=1)
    v, _ = variants("hotspot_f32")
    g = _hotspot_run(v, len(v) - 1, t0, pw, 100)
    d = oracle.hotspot(t0, pw, 100)
    assert np.max(np.abs(g - d) / np.abs(d)) < 2e-6


def test_hotspot_full_size_crops(dev):
    # C3 size, one step, checked on crops whose 1-cell margin makes the interior exact
    W = H = 8192
    v, _ = variants("hotspot_f32")
    t = torch.empty((H, W), device="cuda")
    p = torch.empty((H, W), device="cuda")
    o = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, t.data_ptr(), p.data_ptr(), W, H, seed=1, stream=stream())
    v.launch(len(v) - 1, O.hotspot_args(t.data_ptr(), o.data_ptr(), p.data_ptr(), W, H), stream())
    torch.cuda.synchronize()
    t0, pw = synth.thermal_inputs(W, H, seed=1)
    g = o.cpu().numpy()
    for (y0, y1, x0, x1) in ((0, 40, 0, 40), (H - 40, H, W - 40, W), (4000, 4040, 127, 170), (0, 30, 8100, W)):
        cy0, cy1, cx0, cx1 = max(0, y0 - 1), min(H, y1 + 1), max(0, x0 - 1), min(W, x1 + 1)
        ref = oracle.hotspot(t0[cy0:cy1, cx0:cx1], pw[cy0:cy1, cx0:cx1], 1, precision="f32")
        assert np.array_equal(g[y0:y1, x0:x1], ref[y0 - cy0:y1 - cy0, x0 - cx0:x1 - cx0])


@pytest.mark.parametrize("kernel", ["hotspot2h_f32", "hotspot4h_f32"])
def test_hotspot2_full_size_crops(dev, kernel):
    # C3 size, one two-step launch at the level bench.py settles on and at max occupancy,
    # checked on crops whose 2-cell margin makes the interior exact (every column block border
    # of both kernels falls inside some crop: 120 / 128-column warps)
    W = H = 8192
    v, _ = variants(kernel)
    t = torch.empty((H, W), device="cuda")
    p = torch.empty((H, W), device="cuda")
    o = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, t.data_ptr(), p.data_ptr(), W, H, seed=1, stream=stream())
    t0, pw = synth.thermal_inputs(W, H, seed=1)
    for lvl in (1 if len(v) > 1 else 0, len(v) - 1):
        v.launch(lvl, O.hotspot_args(t.data_ptr(), o.data_ptr(), p.data_ptr(), W, H), stream())
        torch.cuda.synchronize()
        g = o.cpu().numpy()
        n = O.STEPS_PER_LAUNCH[kernel]
        for (y0, y1, x0, x1) in ((0, 40, 0, 40), (H - 40, H, W - 40, W), (4000, 4040, 110, 140),
                                 (255, 290, 230, 262), (0, 30, 8100, W), (8150, H, 3830, 3850)):
            cy0, cy1, cx0, cx1 = max(0, y0 - n), min(H, y1 + n), max(0, x0 - n), min(W, x1 + n)
            ref = oracle.hotspot(t0[cy0:cy1, cx0:cx1], pw[cy0:cy1, cx0:cx1], n, precision="f32")
            assert np.array_equal(g[y0:y1, x0:x1], ref[y0 - cy0:y1 - cy0, x0 - cx0:x1 - cx0]), (lvl, y0, x0)


def test_row_sharded_bit_identical_to_full(dev):
    # C5 logic on one GPU: P slabs, each generated in place with its 6-row halo
    W, H, P = 700, 256, 4
    v, _ = variants("nlm_f4")
    full_in = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, full_in.data_ptr(), W, H, seed=3, sigma=0.13, stream=stream())
    full_out = torch.empty((H, W, 4), device="cuda")
    v.launch(len(v) - 1, O.denoise_args("nlm_f4", full_in.data_ptr(), full_out.data_ptr(), W, H), stream())
    parts = []
    for r in range(P):
        r0, r1 = r * H // P, (r + 1) * H // P
        s0, s1 = max(0, r0 - 6), min(H, r1 + 6)
        slab = torch.empty((s1 - s0, W, 4), device="cuda")
        O.generate_rgba(0, slab.data_ptr(), W, H, s0, s1, seed=3, sigma=0.13, stream=stream())
        out = torch.empty((r1 - r0, W, 4), device="cuda")
        v.launch(r % len(v), O.denoise_args("nlm_f4", slab.data_ptr(), out.data_ptr(), W, H, r0, r1, s0, s1, r0),
                 stream())
        parts.append(out)
    torch.cuda.synchronize()
    assert torch.equal(torch.cat(parts), full_out)


def test_launch_argument_errors(dev):
    v, _ = variants("knn_f4")
    src = torch.empty((32, 32, 4), device="cuda")
    dst = torch.empty((32, 32, 4), device="cuda")
    n0 = O.launch_count()
    v.launch(0, O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), 32, 32, 5, 5), stream())   # empty: no-op
    assert O.launch_count() == n0
    with pytest.raises(O.OrionError) as e:   # slab misses the 3-row halo
        v.launch(0, O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), 32, 64, 10, 20, 10, 20, 10), stream())
    assert e.value.status == -1
    with pytest.raises(O.OrionError):
        v.launch(len(v), O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), 32, 32), stream())


def test_tuner_walks_ladder_and_settles(dev):
    W = H = 512
    v, res = variants("nlm_f4_regheavy")
    src = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, seed=1, sigma=0.13, stream=stream())
    ref = torch.empty((H, W, 4), device="cuda")
    v.launch(0, O.denoise_args("nlm_f4_regheavy", src.data_ptr(), ref.data_ptr(), W, H), stream())
    t = O.Tuner(v)
    direction, ladder = t.ladder()
    assert direction == O.DIR_INCREASING and ladder[0] == max(
        (i for i in range(len(v)) if v.planned[i].reg_cap == 0), key=lambda i: v.planned[i].ctas_per_sm)
    dst = torch.empty((H, W, 4), device="cuda")
    ran = []
    for _ in range(len(ladder) + 4):
        r = t.step(O.denoise_args("nlm_f4_regheavy", src.data_ptr(), dst.data_ptr(), W, H), stream())
        ran.append(r.level_idx)
    torch.cuda.synchronize()
    final, it = t.final()
    assert final >= 0 and it <= len(ladder)
    assert ran[: it] == ladder[: it] and ran[-1] == final
    assert torch.equal(dst, ref)
    # the same iteration end to end from pinned host buffers
    host_in = src.cpu().pin_memory()
    host_out = torch.empty((H, W, 4)).pin_memory()
    a = O.denoise_args("nlm_f4_regheavy", host_in.data_ptr(), host_out.data_ptr(), W, H)
    rep, hi, ho = t.step_host(a, src.data_ptr(), dst.data_ptr(), stream=stream())
    assert hi == ho == W * H * 16 and rep.level_idx == final
    assert torch.equal(host_out, ref.cpu())


def test_sweep_times_every_level(dev):
    W = H = 1024
    v, _ = variants("knn_f4")
    src = torch.empty((H, W, 4), device="cuda")
    dst = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, stream=stream())
    ms = v.sweep(O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), W, H), stream(), rounds=3)
    assert len(ms) == len(v) and all(m > 0 for m in ms)


@pytest.mark.parametrize("shape", [(1, 1), (5, 300), (300, 5), (33, 17), (129, 24), (128, 23)])
@pytest.mark.parametrize("kernel", ["nlm_f4_w", "nlm_f4_regheavy"])
def test_nlm_ragged_and_degenerate(dev, shape, kernel):
    # degenerate frames (a single pixel, one-pixel-wide strips: every window and patch clamps onto
    # the edge) and shapes one pixel past / exactly at a tile (128 x 23 for nlm_f4_w)
    W, H = shape
    img = synth.noisy_rgba(W, H, seed=11, sigma=0.13)
    v, _ = variants(kernel)
    outs = run_denoise(kernel, img, level=0) + run_denoise(kernel, img, level=len(v) - 1)
    assert np.array_equal(outs[0], outs[1])
    out, alt, amb = oracle.denoise("nlm", img)
    check_vs_oracle(outs[0], out, alt, amb)


def test_tune_step_empty_band_is_not_an_iteration(dev):
    W = H = 64
    v, _ = variants("nlm_f4_w")
    src = torch.empty((H, W, 4), device="cuda")
    dst = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, stream=stream())
    t = O.Tuner(v)
    n0 = O.launch_count()
    r = t.step(O.denoise_args("nlm_f4_w", src.data_ptr(), dst.data_ptr(), W, H, 10, 10), stream())
    assert (r.iteration, r.level_idx, r.phase) == (-1, -1, -1) and O.launch_count() == n0
    assert all(x < 0 for x in t.tried())                   # nothing reached Fig. 9
    r = t.step(O.denoise_args("nlm_f4_w", src.data_ptr(), dst.data_ptr(), W, H), stream())
    assert r.iteration == 0 and r.phase == 0               # the first real iteration is iteration 0
    ms = v.sweep(O.denoise_args("nlm_f4_w", src.data_ptr(), dst.data_ptr(), W, H, 7, 7), stream())
    assert ms == [0.0] * len(v)                            # an empty sweep times nothing
