"""orion_tuner_cfg.async_timing = 1: the Fig. 9 walk (PAPER.md P:L605-P:L653) with its event
pairs read by polling instead of a host synchronisation.  The walk must still settle, every
iteration's output must stay bit-exact (any level is a correct kernel), and the levels it
ran must follow the ladder order (the original first, each level repeated only while its
measurement is in flight)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def hs():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return O.build_all_levels(0, "hotspot_f32", mode=O.REALISE_MIN_CARVEOUT)[0]


@pytest.mark.parametrize("samples", [1, 2])
def test_async_walk_settles_and_stays_exact(hs, samples):
    W, H = 2048, 1024
    t0, pw = synth.thermal_inputs(W, H, seed=3)
    a = torch.from_numpy(t0).cuda()
    b = torch.empty_like(a)
    p = torch.from_numpy(pw).cuda()
    sp = torch.cuda.current_stream().cuda_stream
    tuner = O.Tuner(hs, O.default_cfg(async_timing=1, samples_per_level=samples))
    direction, ladder = tuner.ladder()
    ran, measured = [], []
    iters = 0
    for it in range(400):
        r = tuner.step(O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H), sp)
        a, b = b, a
        iters += 1
        ran.append(r.level_idx)
        if r.ms >= 0:
            measured.append(r.ms)
        if r.final_level_idx >= 0 and it > 20:
            break
        if it % 16 == 15:
            torch.cuda.synchronize()        # let measurements land now and then
    torch.cuda.synchronize()
    final, _ = tuner.final()
    assert final >= 0 and len(measured) >= 2
    # levels appear in ladder order: the sequence of distinct levels run is a prefix walk
    distinct = [ran[0]] + [x for i, x in enumerate(ran[1:], 1) if x != ran[i - 1]]
    assert distinct[0] == ladder[0]
    assert np.array_equal(a.cpu().numpy(), oracle.hotspot(t0, pw, iters, precision="f32"))


def test_async_cfg_validated():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    v, _ = O.build_all_levels(0, "knn_f4")
    with pytest.raises(O.OrionError):
        O.Tuner(v, O.default_cfg(async_timing=2))
