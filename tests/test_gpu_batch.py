"""Batched denoiser launches (orion_args.batch): B whole frames stacked in src / dst filtered by one
launch (grid z = frame) -- configuration C1's small frames (BASELINE.json configs[0]) one batch
per tuner iteration.  Every denoiser at its first and last level: the batch equals B single-frame
launches bit for bit (those are held against the oracle by test_gpu_parity.py), one frame is
also checked against the oracle directly; the tuner counts every frame of a batch as work
(P:L975); misuse is refused; a batch stays inside its buffers (guard zones)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402

DENOISERS = ["knn_f4", "knn_f4_p1", "knn_f4_t16", "nlm_f4", "nlm_f4_w", "nlm_f4_direct", "nlm_f4_regheavy"]


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


def sp():
    return torch.cuda.current_stream().cuda_stream


def frames(W, H, B, sigma, seed0=30):
    return np.stack([synth.noisy_rgba(W, H, seed=seed0 + f, sigma=sigma) for f in range(B)])


@pytest.mark.parametrize("kernel", DENOISERS)
@pytest.mark.parametrize("W,H,B", [(64, 64, 5), (70, 45, 3), (1, 1, 4)])
def test_batch_equals_single_frames(dev, kernel, W, H, B):
    v, _ = O.build_all_levels(0, kernel)
    sigma = 0.2 if kernel.startswith("knn") else 0.13
    src = torch.from_numpy(frames(W, H, B, sigma)).cuda()
    for lvl in sorted({0, len(v) - 1}):
        dst = torch.full_like(src, float("nan"))
        v.launch(lvl, O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H, batch=B), sp())
        ref = torch.full_like(src, float("nan"))
        for f in range(B):
            v.launch(lvl, O.denoise_args(kernel, src[f].data_ptr(), ref[f].data_ptr(), W, H), sp())
        torch.cuda.synchronize()
        assert torch.equal(dst, ref), (kernel, lvl)


def test_batch_frame_vs_oracle(dev):
    W = H = 64
    B = 16
    imgs = frames(W, H, B, 0.2, seed0=1)
    v, _ = O.build_all_levels(0, "knn_f4_t16")
    src = torch.from_numpy(imgs).cuda()
    dst = torch.full_like(src, float("nan"))
    v.launch(len(v) - 1, O.denoise_args("knn_f4_t16", src.data_ptr(), dst.data_ptr(), W, H, batch=B), sp())
    torch.cuda.synchronize()
    g = dst.cpu().numpy()
    for f in (0, 7, B - 1):
        out, alt, amb = oracle.denoise("knn", imgs[f])
        e = np.abs(g[f, ..., :3].astype(np.float64) - out).max(-1)
        ok = (e <= 1e-5) | (amb & (np.abs(g[f, ..., :3].astype(np.float64) - alt).max(-1) <= 1e-5))
        assert ok.all(), (f, float(e.max()))
        assert (g[f, ..., 3] == 0).all()


def test_batches_through_the_tuner_and_a_graph(dev):
    # the bench's C1 loop: independent batches through Fig. 9, then the settled iterations replayed
    # as a CUDA graph with programmatic edges; every frame == a single-frame launch at the final level
    W = H = 64
    B, nb = 8, 6
    v, _ = O.build_all_levels(0, "knn_f4_t16", mode=O.REALISE_MIN_CARVEOUT)
    src = torch.from_numpy(frames(W, H, B * nb, 0.2)).cuda().view(nb, B, H, W, 4)
    dst = torch.zeros_like(src)
    args = [O.denoise_args("knn_f4_t16", src[b].data_ptr(), dst[b].data_ptr(), W, H, independent=True, batch=B)
            for b in range(nb)]
    prev = O.set_pdl(False)
    try:
        t = O.Tuner(v, O.default_cfg(samples_per_level=2))
        s = 0
        while t.final()[0] < 0:
            r = t.step(args[s % nb], sp())
            if r.phase == 0:
                assert r.ms > 0
            s += 1
            assert s < 300
        final = t.final()[0]
        dst.zero_()
        O.set_pdl(True)
        g = t.capture(args)
        g.launch(sp())
        torch.cuda.synchronize()
        g.close()
        t.close()
    finally:
        O.set_pdl(prev)
    ref = torch.zeros_like(src)
    for b in range(nb):
        for f in range(B):
            v.launch(final, O.denoise_args("knn_f4_t16", src[b, f].data_ptr(), ref[b, f].data_ptr(), W, H), sp())
    torch.cuda.synchronize()
    assert torch.equal(dst, ref)


def test_batch_misuse_refused(dev):
    W = H = 64
    buf = torch.zeros((4, H, W, 4), device="cuda")
    v, _ = O.build_all_levels(0, "knn_f4_t16")
    bad = [O.denoise_args("knn_f4_t16", buf.data_ptr(), buf.data_ptr(), W, H, 0, 32, batch=2),            # a band
           O.with_fanout(O.denoise_args("knn_f4_t16", buf.data_ptr(), buf.data_ptr(), W, H, batch=2),
                         [buf.data_ptr()]),                                                               # fan-out
           O.denoise_args("knn_f4_t16", buf.data_ptr(), buf.data_ptr(), W, H, batch=70000)]                # too many
    for a in bad:
        with pytest.raises(O.OrionError) as e:
            v.launch(0, a)
        assert e.value.status == -1
    vh, _ = O.build_all_levels(0, "hotspot_f32")
    t = torch.zeros((2, 16, 128), device="cuda")
    a = O.hotspot_args(t.data_ptr(), t[1].data_ptr(), t.data_ptr(), 128, 16)
    a.batch = 2
    with pytest.raises(O.OrionError):
        vh.launch(0, a)


def test_batch_from_host_buffers(dev):
    # orion_tune_step_host and orion_host_pipe_submit copy a batch as one block each way
    W = H = 64
    B = 6
    imgs = frames(W, H, B, 0.2)
    v, _ = O.build_all_levels(0, "knn_f4_t16")
    hin = torch.from_numpy(imgs).pin_memory()
    hout = torch.zeros_like(hin).pin_memory()
    din = torch.empty(hin.shape, device="cuda")
    dout = torch.empty(hin.shape, device="cuda")
    t = O.Tuner(v)
    t.step_host(O.denoise_args("knn_f4_t16", hin.data_ptr(), hout.data_ptr(), W, H, batch=B), din.data_ptr(),
                dout.data_ptr())
    ref = torch.empty(hin.shape, device="cuda")
    dsrc = hin.cuda()
    refs = []
    for l_ in range(len(v)):
        v.launch(l_, O.denoise_args("knn_f4_t16", dsrc.data_ptr(), ref.data_ptr(), W, H, batch=B), sp())
        torch.cuda.synchronize()
        refs.append(ref.cpu().clone())
    assert all(torch.equal(refs[0], r) for r in refs)      # every level gives the same bits
    assert torch.equal(hout, refs[0])
    pipe = O.HostPipe(t, W, B * H, depth=2)
    outs = [torch.zeros_like(hin).pin_memory() for _ in range(2)]
    for k in range(4):
        pipe.submit(O.denoise_args("knn_f4_t16", hin.data_ptr(), outs[k % 2].data_ptr(), W, H, batch=B))
    pipe.drain()
    for o in outs:
        assert torch.equal(o, refs[0])
    with pytest.raises(O.OrionError):       # a slot too small for the batch
        small = O.HostPipe(t, W, H, depth=2)
        small.submit(O.denoise_args("knn_f4_t16", hin.data_ptr(), outs[0].data_ptr(), W, H, batch=B))
    pipe.close()
    t.close()


@pytest.mark.parametrize("kernel", ["knn_f4_t16", "nlm_f4_w", "nlm_f4_regheavy"])
def test_batch_stays_in_bounds(dev, kernel):
    # the batch inside NaN (input) / sentinel (output) guard zones: no read or write outside
    W, H, B = 70, 45, 3
    n = B * H * W * 4
    G = 8192
    img = torch.from_numpy(frames(W, H, B, 0.13)).cuda()
    sbuf = torch.full((G + n + G,), float("nan"), device="cuda")
    sbuf[G:G + n] = img.reshape(-1)
    dbuf = torch.full((G + n + G,), -7.25e30, device="cuda")
    v, _ = O.build_all_levels(0, kernel)
    ref = torch.empty_like(img)
    v.launch(len(v) - 1, O.denoise_args(kernel, img.data_ptr(), ref.data_ptr(), W, H, batch=B), sp())
    v.launch(len(v) - 1, O.denoise_args(kernel, sbuf[G:].data_ptr(), dbuf[G:].data_ptr(), W, H, batch=B), sp())
    torch.cuda.synchronize()
    assert bool((dbuf[:G] == -7.25e30).all() and (dbuf[G + n:] == -7.25e30).all())
    assert bool(torch.isnan(sbuf[:G]).all() and torch.isnan(sbuf[G + n:]).all())
    got = dbuf[G:G + n].view(B, H, W, 4)
    assert torch.isfinite(got).all()
    assert torch.equal(got, ref)
