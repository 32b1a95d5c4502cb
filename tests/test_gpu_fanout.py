"""Fan-out epilogue (orion_args.fanout): a row-sharded frame gathered by the kernels' own
stores into every rank's full image (C5 without a separate all-gather).  Here the "ranks" are
row bands launched on one GPU and the fan-out buffers are plain device buffers -- the same
stores a peer pointer receives over NVLink.  Results must equal the unsharded launch bit for
bit in every buffer."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402
from paper_conf_middleware_hayeslcsz16_b200 import shard  # noqa: E402


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return 0


@pytest.mark.parametrize("kernel,halo", [("nlm_f4", 6), ("knn_f4", 3), ("knn_f4_t16", 3), ("nlm_f4_w", 6)])
@pytest.mark.parametrize("P", [2, 3])
def test_fanout_gathers_bands_bit_exact(dev, kernel, halo, P):
    W, H = 250, 131
    sp = torch.cuda.current_stream().cuda_stream
    v, _ = O.build_all_levels(0, kernel)
    img = torch.from_numpy(synth.noisy_rgba(W, H, seed=3, sigma=0.13)).cuda()
    full_ref = torch.empty_like(img)
    v.launch(len(v) - 1, O.denoise_args(kernel, img.data_ptr(), full_ref.data_ptr(), W, H), sp)
    fulls = [torch.full_like(img, -1.0) for _ in range(P)]
    for r in range(P):
        b = shard.band(r, P, H, halo)
        if not b.rows:
            continue
        slab = img[b.src_begin:b.src_end].contiguous()
        band = torch.empty((b.rows, W, 4), device="cuda")
        a = O.denoise_args(kernel, slab.data_ptr(), band.data_ptr(), W, H, b.row_begin, b.row_end, b.src_begin,
                           b.src_end, b.row_begin)
        v.launch(r % len(v), O.with_fanout(a, [f.data_ptr() for f in fulls]), sp)
        torch.cuda.synchronize()
        assert torch.equal(band, full_ref[b.row_begin:b.row_end])
    torch.cuda.synchronize()
    for f in fulls:
        assert torch.equal(f, full_ref)


def test_fanout_rejected_where_unsupported(dev):
    v, _ = O.build_all_levels(0, "hotspot_f32")
    t = torch.zeros((16, 128), device="cuda")
    a = O.with_fanout(O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), 128, 16), [t.data_ptr()])
    with pytest.raises(O.OrionError) as e:
        v.launch(0, a)
    assert e.value.status == -1
