"""Kernel splitting (NEXT-1): one frame processed as row bands, each a
tuning iteration with work-normalised timing -- output bit-identical to one unsplit launch,
and the tuner reaches its final kernel inside a single frame."""
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def sp():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.cuda.current_stream().cuda_stream


@pytest.mark.parametrize("kernel,bands", [("nlm_f4_regheavy", 16), ("nlm_f4", 7), ("knn_f4", 5)])
def test_split_frame_equals_unsplit_and_converges(sp, kernel, bands):
    W, H = 640, 301
    v, _ = O.build_all_levels(0, kernel)
    src = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, seed=4, sigma=0.13, stream=sp)
    ref = torch.empty_like(src)
    v.launch(0, O.denoise_args(kernel, src.data_ptr(), ref.data_ptr(), W, H), sp)
    t = O.Tuner(v)
    _, ladder = t.ladder()
    dst = torch.full_like(src, float("nan"))
    reps = t.split(O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H), bands, sp)
    torch.cuda.synchronize()
    assert torch.equal(dst, ref)
    assert [r.iteration for r in reps if r.iteration >= 0] == list(range(len([r for r in reps if r.iteration >= 0])))
    if bands >= len(ladder) + 2:
        final, it = t.final()
        assert final >= 0 and it < bands


def test_split_more_bands_than_rows(sp):
    W, H = 64, 5
    v, _ = O.build_all_levels(0, "knn_f4")
    src = torch.empty((H, W, 4), device="cuda")
    O.generate_rgba(0, src.data_ptr(), W, H, seed=2, stream=sp)
    ref = torch.empty_like(src)
    v.launch(0, O.denoise_args("knn_f4", src.data_ptr(), ref.data_ptr(), W, H), sp)
    t = O.Tuner(v)
    dst = torch.empty_like(src)
    reps = t.split(O.denoise_args("knn_f4", src.data_ptr(), dst.data_ptr(), W, H), 8, sp)
    torch.cuda.synchronize()
    assert torch.equal(dst, ref)
    assert sum(r.iteration >= 0 for r in reps) == 5 and reps[-1].iteration == -1


@pytest.mark.parametrize("kernel,bands", [("nlm_f4_regheavy", 16), ("nlm_f4_w", 7), ("knn_f4_t16", 5)])
def test_split_frame_vs_oracle(sp, kernel, bands):
    # NEXT-1 output against the oracle itself (not only the unsplit launch): every pixel of the
    # banded frame, whatever level each band ran at
    import numpy as np
    import oracle
    import synth
    W, H = 333, 170
    v, _ = O.build_all_levels(0, kernel)
    img = synth.noisy_rgba(W, H, seed=6, sigma=0.2 if kernel.startswith("knn") else 0.13)
    src = torch.from_numpy(img).cuda()
    dst = torch.full_like(src, float("nan"))
    t = O.Tuner(v)
    reps = t.split(O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H), bands, sp)
    torch.cuda.synchronize()
    assert len({r.level_idx for r in reps if r.iteration >= 0}) >= 2      # the bands ran different levels
    g = dst.cpu().numpy()
    out, alt, amb = oracle.denoise("knn" if kernel.startswith("knn") else "nlm", img)
    gg = g[..., :3].astype(np.float64)
    ok = (np.abs(gg - out) <= 1e-5).all(-1) | (amb & (np.abs(gg - alt) <= 1e-5).all(-1))
    assert ok.all() and (g[..., 3] == 0).all()
