"""Independent launches (orion.h ORION_ARGS_INDEPENDENT): a stream of frames, each in its own
buffers, launched with programmatic dependent launch and without waiting for the previous
frame's grid -- the next frame's CTAs start in the previous grid's last wave (one frame per
application iteration, PAPER.md P:L605-P:L607).  The bits must be those of ordinary launches, and
of the oracle; stencil launches (each reads its predecessor's output) must refuse the flag."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def sp():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    prev = O.set_pdl(True)
    yield torch.cuda.current_stream().cuda_stream
    O.set_pdl(prev)


def frames(n, W, H, sigma):
    out = []
    for f in range(n):
        t = torch.empty((H, W, 4), device="cuda")
        O.generate_rgba(0, t.data_ptr(), W, H, seed=11 + f, sigma=sigma, stream=torch.cuda.current_stream().cuda_stream)
        out.append(t)
    return out


@pytest.mark.parametrize("kernel,W,H", [("nlm_f4_w", 700, 301), ("knn_f4_t16", 257, 131), ("nlm_f4", 256, 97)])
def test_independent_frames_bit_identical(sp, kernel, W, H):
    v, _ = O.build_all_levels(0, kernel)
    srcs = frames(4, W, H, 0.13)
    ref = [torch.empty_like(s) for s in srcs]
    for f in range(4):
        v.launch(len(v) - 1, O.denoise_args(kernel, srcs[f].data_ptr(), ref[f].data_ptr(), W, H), sp)
    torch.cuda.synchronize()
    dst = [torch.full_like(s, float("nan")) for s in srcs]
    for n in range(24):            # frames cycled; levels alternate so consecutive grids differ
        f = n % 4
        v.launch((n % len(v)), O.denoise_args(kernel, srcs[f].data_ptr(), dst[f].data_ptr(), W, H, independent=True), sp)
    torch.cuda.synchronize()
    for f in range(4):
        assert torch.equal(dst[f], ref[f]), f


def test_independent_frames_through_the_tuner_match_the_oracle(sp):
    # the tuned loop as bench.py runs it (independent frames), one frame checked against O2
    kernel, W, H = "nlm_f4_w", 300, 170
    v, _ = O.build_all_levels(0, kernel)
    t = O.Tuner(v)
    imgs = [synth.noisy_rgba(W, H, seed=20 + f, sigma=0.13) for f in range(3)]
    srcs = [torch.from_numpy(i).cuda() for i in imgs]
    dst = [torch.empty_like(s) for s in srcs]
    for n in range(30):
        f = n % 3
        t.step(O.denoise_args(kernel, srcs[f].data_ptr(), dst[f].data_ptr(), W, H, independent=True), sp)
    torch.cuda.synchronize()
    g = dst[1].cpu().numpy()[..., :3].astype(np.float64)
    out, alt, amb = oracle.denoise("nlm", imgs[1])
    tol = 1e-5                                   # tests/test_gpu_parity.py's TOL
    ok = (np.abs(g - out) <= tol).all(-1) | (amb & (np.abs(g - alt) <= tol).all(-1))
    assert ok.all(), np.argwhere(~ok)[:5]
    t.close()


def test_independent_split_bands(sp):
    # orion_tune_split's bands of one frame are mutually independent: same bits with the flag
    kernel, W, H = "nlm_f4_w", 640, 301
    v, _ = O.build_all_levels(0, kernel)
    src = frames(1, W, H, 0.13)[0]
    ref = torch.empty_like(src)
    v.launch(0, O.denoise_args(kernel, src.data_ptr(), ref.data_ptr(), W, H), sp)
    t = O.Tuner(v)
    dst = torch.full_like(src, float("nan"))
    t.split(O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H, independent=True), 9, sp)
    torch.cuda.synchronize()
    assert torch.equal(dst, ref)
    t.close()


def test_host_pipe_ignores_the_flag(sp):
    kernel, W, H = "knn_f4_t16", 128, 64
    v, _ = O.build_all_levels(0, kernel)
    t = O.Tuner(v)
    src = frames(1, W, H, 0.13)[0]
    ref = torch.empty_like(src)
    v.launch(0, O.denoise_args(kernel, src.data_ptr(), ref.data_ptr(), W, H), sp)
    torch.cuda.synchronize()
    hin = src.cpu().pin_memory()
    hout = torch.empty_like(hin).pin_memory()
    pipe = O.HostPipe(t, W, H, depth=2)
    pipe.submit(O.denoise_args(kernel, hin.data_ptr(), hout.data_ptr(), W, H, independent=True))
    pipe.drain()
    torch.cuda.synchronize()
    assert torch.equal(hout, ref.cpu())
    pipe.close()
    t.close()


def test_flag_rejected_where_launches_depend(sp):
    W, H = 64, 16
    t = torch.zeros((H, W), device="cuda")
    for kernel in ("hotspot_f32", "hotspot4h_f32"):
        v, _ = O.build_all_levels(0, kernel)
        a = O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H)
        a.flags = O.ARGS_INDEPENDENT
        with pytest.raises(O.OrionError) as e:
            v.launch(0, a, sp)
        assert e.value.status == -1
    v, _ = O.build_all_levels(0, "srad_f32h")
    a = O.srad_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H)
    a.flags = O.ARGS_INDEPENDENT
    with pytest.raises(O.OrionError):
        v.launch(0, a, sp)
    v, _ = O.build_all_levels(0, "nlm_f4_w")
    img = torch.zeros((H, W, 4), device="cuda")
    a = O.denoise_args("nlm_f4_w", img.data_ptr(), img.data_ptr(), W, H)
    a.flags = 2                                                     # unknown bit
    with pytest.raises(O.OrionError):
        v.launch(0, a, sp)
