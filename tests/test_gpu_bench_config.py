"""Parity at the configured sizes IN THE LAUNCH CONFIGURATION bench.py times: the same kernels,
realisation (MIN_CARVEOUT), tuner configuration (Fig. 9, 2 samples per level), programmatic
dependent launch and issue mode as the timed loops --

* C2: a stream of three independent 2048^2 frames (ORION_ARGS_INDEPENDENT: each frame's CTAs
  start in the previous frame's last wave) through the tuner, exploration included; the whole
  of one frame and 48 sampled rows of the others against the double oracle.
* C3: the 8192^2 grid advanced 100 steps as 25 CHAINED `hotspot4h_f32` launches (orion_chain:
  tile-level waits) through the tuner while it explores (levels change inside the chain):
  bit-identical to 25 unchained launches at one level, and within 2e-6 of O3's f64 form on
  crops whose 100-cell margin holds the dependency cone.
* SRAD: the 8192^2 grid, 3 chained `srad_f32hs` iterations (statistics fused) through the tuner
  against O5 (double) over the WHOLE grid, <= 1e-5 relative.
* C1: batches of 64 64^2 KNN frames (orion_args.batch; `knn_f4`, 256-thread CTAs) tuned without
  PDL, then the settled iterations of 6 independent batches captured as one CUDA graph WITH
  programmatic edges and replayed: all 384 frames against the double oracle.
* C4: two independent 4096^2 frames of `nlm_f4_regheavy` through the tuner (its 16-level ladder
  explored); one whole frame against the double oracle.
"""
import numpy as np
import pytest

import oracle
import oracle_par
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

from test_gpu_fullsize import check  # noqa: E402

ROI = (0, 127, 0, 127)          # bench.py's SRAD ROI (reading R-SRAD)


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


def sp():
    return torch.cuda.current_stream().cuda_stream


def bench_tuner(v):
    return O.Tuner(v, O.default_cfg(samples_per_level=2))


def test_c2_independent_frame_stream_vs_oracle(dev):
    W = H = 2048
    nframes = 3                  # bench.py: a pool of frames larger than L2 (3 x 64 MiB)
    v, _ = O.build_all_levels(0, "nlm_f4_w", mode=O.REALISE_MIN_CARVEOUT)
    srcs = [torch.empty((H, W, 4), device="cuda") for _ in range(nframes)]
    dsts = [torch.full((H, W, 4), float("nan"), device="cuda") for _ in range(nframes)]
    for f, t in enumerate(srcs):
        O.generate_rgba(0, t.data_ptr(), W, H, seed=1 + f, sigma=0.13, stream=sp())
    t = bench_tuner(v)
    s = 0
    while s < 12 or t.final()[0] < 0:        # exploration, then settled frames
        f = s % nframes
        t.step(O.denoise_args("nlm_f4_w", srcs[f].data_ptr(), dsts[f].data_ptr(), W, H, independent=True), sp())
        s += 1
        assert s < 200
    torch.cuda.synchronize()
    rng = np.random.default_rng(2)
    for f in range(nframes):
        g = dsts[f].cpu().numpy()
        img = synth.noisy_rgba(W, H, seed=1 + f, sigma=0.13)
        if f == 0:
            out, alt, amb = oracle_par.denoise_rows("nlm", img, H, 0, 0, H)
            check(g, out, alt, amb, "C2 stream, frame 0 (whole)")
        else:
            rows = sorted(set([0, 1, 2, H - 3, H - 2, H - 1]) | set(int(x) for x in rng.integers(0, H, 42)))

            def one(y):
                return oracle.denoise("nlm", img, height=H, row0=0, y_begin=y, y_end=y + 1)
            res = oracle_par.map_threads(one, rows)
            out = np.concatenate([r[0] for r in res])
            alt = np.concatenate([r[1] for r in res])
            amb = np.concatenate([r[2] for r in res])
            check(g[rows], out, alt, amb, f"C2 stream, frame {f} ({len(rows)} rows)")
    t.close()
    v.close()


def test_c3_chained_tuned_100_steps(dev):
    W = H = 8192
    S = 100
    v, _ = O.build_all_levels(0, "hotspot4h_f32", mode=O.REALISE_MIN_CARVEOUT)
    t0 = torch.empty((H, W), device="cuda")
    pw = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, t0.data_ptr(), pw.data_ptr(), W, H, seed=1, stream=sp())
    # the bench's loop: chained launches under the Fig. 9 tuner (its exploration switches levels
    # inside the chain)
    a, b = t0.clone(), torch.empty_like(t0)
    ch = O.Chain(v, W, H)
    t = bench_tuner(v)
    levels = []
    for _ in range(S // 4):
        r = t.step(O.hotspot_args(a.data_ptr(), b.data_ptr(), pw.data_ptr(), W, H, chain=ch), sp())
        levels.append(r.level_idx)
        a, b = b, a
    torch.cuda.synchronize()
    ch.close()
    t.close()
    assert len(set(levels)) > 1, levels          # the chain really crossed level switches
    got = a
    # unchained, one level
    c, d = t0.clone(), torch.empty_like(t0)
    for _ in range(S // 4):
        v.launch(0, O.hotspot_args(c.data_ptr(), d.data_ptr(), pw.data_ptr(), W, H), sp())
        c, d = d, c
    torch.cuda.synchronize()
    assert torch.equal(got, c)
    g = got.cpu().numpy()
    t0h, pwh = synth.thermal_inputs(W, H, seed=1)
    assert np.array_equal(t0.cpu().numpy(), t0h)
    crops = [(0, 80, 0, 80), (H - 80, H, W - 80, W), (0, 48, 4000, 4200), (5000, 5064, W - 130, W),
             (3000, 3070, 2000, 2150), (H - 40, H, 7000, 7200)]

    def one(cr):
        y0, y1, x0, x1 = cr
        cy0, cy1, cx0, cx1 = max(0, y0 - S), min(H, y1 + S), max(0, x0 - S), min(W, x1 + S)
        ref = oracle.hotspot(t0h[cy0:cy1, cx0:cx1], pwh[cy0:cy1, cx0:cx1], S)
        return ref[y0 - cy0:y1 - cy0, x0 - cx0:x1 - cx0]
    for (y0, y1, x0, x1), ref in zip(crops, oracle_par.map_threads(one, crops)):
        rel = np.abs(g[y0:y1, x0:x1] - ref) / np.abs(ref)
        assert rel.max() <= 2e-6, ((y0, x0), float(rel.max()))
    v.close()


def test_srad_chained_tuned_whole_grid(dev):
    W = H = 8192
    iters = 3
    v, _ = O.build_all_levels(0, "srad_f32hs", mode=O.REALISE_MIN_CARVEOUT)
    extra = O.SRAD_STATS_FLOATS
    fa = torch.empty(H * W + extra, device="cuda")
    fb = torch.empty(H * W + extra, device="cuda")
    pw = torch.empty((H, W), device="cuda")
    O.generate_thermal(0, fa.data_ptr(), pw.data_ptr(), W, H, seed=1, stream=sp())
    O.srad_stats_init(0, fa.data_ptr(), W, H, ROI, sp())
    ch = O.Chain(v, W, H)
    t = bench_tuner(v)
    levels = []
    for _ in range(iters):
        r = t.step(O.srad_args(fa.data_ptr(), fb.data_ptr(), 0, W, H, roi=ROI, chain=ch), sp())
        levels.append(r.level_idx)
        fa, fb = fb, fa
    torch.cuda.synchronize()
    ch.close()
    t.close()
    g = fa[:H * W].view(H, W).cpu().numpy()
    j0, _ = synth.thermal_inputs(W, H, seed=1)
    ref, _ = oracle.srad(j0.astype(np.float64), iters, 0.5, ROI)
    rel = np.abs(g - ref) / np.abs(ref)
    assert rel.max() < 1e-5, (levels, float(rel.max()))
    v.close()


def test_c1_graph_of_independent_batches_vs_oracle(dev):
    # bench.py's C1: batches of 64x64 frames (orion_args.batch) through knn_f4 with 256-thread CTAs,
    # tuned without PDL, then the settled iterations captured as a CUDA graph with programmatic
    # edges and replayed; every frame of every batch against the double oracle
    W = H = 64
    B, nb = 64, 6
    v, _ = O.build_all_levels(0, "knn_f4", 256, mode=O.REALISE_MIN_CARVEOUT)
    imgs = np.stack([synth.noisy_rgba(W, H, seed=1 + f, sigma=0.2) for f in range(B * nb)])
    src = torch.from_numpy(imgs).cuda().view(nb, B, H, W, 4)
    dst = torch.full_like(src, float("nan"))
    args = [O.denoise_args("knn_f4", src[b].data_ptr(), dst[b].data_ptr(), W, H, independent=True, batch=B)
            for b in range(nb)]
    prev = O.set_pdl(False)                  # bench.py: the sweep and the exploration run without PDL
    try:
        t = bench_tuner(v)
        s = 0
        while s < 12 or t.final()[0] < 0:
            t.step(args[s % nb], sp())
            s += 1
            assert s < 400
        torch.cuda.synchronize()
        dst.fill_(float("nan"))
        O.set_pdl(True)                      # the timed graph keeps programmatic edges
        g = t.capture(args)
        for _ in range(3):
            g.launch(sp())
        torch.cuda.synchronize()
        g.close()
        t.close()
    finally:
        O.set_pdl(prev)
    res = oracle_par.map_threads(lambda im: oracle.denoise("knn", im), list(imgs))
    got = dst.view(B * nb, H, W, 4).cpu().numpy()
    for f in range(B * nb):
        out, alt, amb = res[f]
        g_ = got[f]
        e = np.abs(g_[..., :3].astype(np.float64) - out).max(-1)
        ok = (e <= 1e-5) | (amb & (np.abs(g_[..., :3].astype(np.float64) - alt).max(-1) <= 1e-5))
        assert ok.all(), (f, int((~ok).sum()), float(e.max()))
        assert (g_[..., 3] == 0).all(), f
    v.close()


def test_c4_independent_frames_through_the_tuner_vs_oracle(dev):
    W = H = 4096
    v, _ = O.build_all_levels(0, "nlm_f4_regheavy", mode=O.REALISE_MIN_CARVEOUT)
    srcs = [torch.empty((H, W, 4), device="cuda") for _ in range(2)]
    dsts = [torch.full((H, W, 4), float("nan"), device="cuda") for _ in range(2)]
    for f, t_ in enumerate(srcs):
        O.generate_rgba(0, t_.data_ptr(), W, H, seed=1 + f, sigma=0.13, stream=sp())
    t = bench_tuner(v)
    s = 0
    while s < 4 or t.final()[0] < 0:
        t.step(O.denoise_args("nlm_f4_regheavy", srcs[s % 2].data_ptr(), dsts[s % 2].data_ptr(), W, H,
                              independent=True), sp())
        s += 1
        assert s < 60
    t.step(O.denoise_args("nlm_f4_regheavy", srcs[0].data_ptr(), dsts[0].data_ptr(), W, H, independent=True), sp())
    torch.cuda.synchronize()
    g = dsts[0].cpu().numpy()
    img = synth.noisy_rgba(W, H, seed=1, sigma=0.13)
    out, alt, amb = oracle_par.denoise_rows("nlm", img, H, 0, 0, H)
    check(g, out, alt, amb, "C4 frames through the tuner, frame 0 (whole)")
    t.close()
    v.close()
