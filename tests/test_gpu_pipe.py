"""orion_host_pipe: pipelined host->device->kernel->host iterations give the same bytes as
device-resident launches, for several frames in flight (depth 2 and 3), and reject frames
that do not fit."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def nlm():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return O.build_all_levels(0, "nlm_f4")


@pytest.mark.parametrize("depth", [1, 2, 3])
def test_pipe_matches_device_launch(nlm, depth):
    v, _ = nlm
    W, H, F = 300, 97, 5
    frames = [synth.noisy_rgba(W, H, seed=10 + f, sigma=0.13) for f in range(F)]
    refs = []
    sp = torch.cuda.current_stream().cuda_stream
    for img in frames:
        s = torch.from_numpy(img).cuda()
        d = torch.empty_like(s)
        v.launch(len(v) - 1, O.denoise_args("nlm_f4", s.data_ptr(), d.data_ptr(), W, H), sp)
        refs.append(d)
    torch.cuda.synchronize()
    t = O.Tuner(v)
    pipe = O.HostPipe(t, W, H, depth=depth)
    hin = [torch.from_numpy(f).pin_memory() for f in frames]
    hout = [torch.full((H, W, 4), -1.0).pin_memory() for _ in frames]
    for f in range(F):
        _, hi, ho = pipe.submit(O.denoise_args("nlm_f4", hin[f].data_ptr(), hout[f].data_ptr(), W, H))
        assert hi == ho == W * H * 16
    pipe.drain()
    for f in range(F):
        assert torch.equal(hout[f], refs[f].cpu())
    with pytest.raises(O.OrionError):
        pipe.submit(O.denoise_args("nlm_f4", hin[0].data_ptr(), hout[0].data_ptr(), W + 1, H))
    pipe.close()


def test_pipe_row_band(nlm):
    # a band of rows with its halo: output lands at the band's rows of the host frame
    v, _ = nlm
    W, H = 256, 120
    img = synth.noisy_rgba(W, H, seed=3, sigma=0.13)
    full = torch.from_numpy(img).cuda()
    ref = torch.empty_like(full)
    sp = torch.cuda.current_stream().cuda_stream
    v.launch(0, O.denoise_args("nlm_f4", full.data_ptr(), ref.data_ptr(), W, H), sp)
    torch.cuda.synchronize()
    t = O.Tuner(v)
    pipe = O.HostPipe(t, W, 60, depth=2)
    r0, r1 = 40, 80
    slab = torch.from_numpy(np.ascontiguousarray(img[r0 - 6:r1 + 6])).pin_memory()
    out = torch.zeros((H, W, 4)).pin_memory()
    a = O.denoise_args("nlm_f4", slab.data_ptr(), out.data_ptr(), W, H, r0, r1, r0 - 6, r1 + 6, 0)
    pipe.submit(a)
    pipe.drain()
    assert torch.equal(out[r0:r1], ref[r0:r1].cpu())
    assert (out[:r0] == 0).all() and (out[r1:] == 0).all()
