"""The carveout axis (NEXT-2, Table 3 analogue): levels realised with
the smallest shared-memory configuration are verified by the driver occupancy API, compute
the same bytes as the max-shared-memory realisation, and the LOWEST_WITHIN_TOL selection
(NEXT-3) picks a level no slower than 2 % of the best it measured."""
import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def sp():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.cuda.current_stream().cuda_stream


@pytest.mark.parametrize("kernel", ["hotspot_f32", "nlm_f4_regheavy", "knn_f4", "nlm_f4"])
def test_min_carveout_levels_verified_and_bit_exact(sp, kernel):
    vmin, res = O.build_all_levels(0, kernel, mode=O.REALISE_MIN_CARVEOUT)
    vmax, _ = O.build_all_levels(0, kernel, mode=O.REALISE_MAX_SMEM)
    assert len(vmin) == len(vmax)
    for i in range(len(vmin)):
        inf = vmin.info(i)
        assert inf.verified_ctas == inf.level.ctas_per_sm
        assert 0 < vmin.level(i).carveout_kb <= 228
    if kernel == "hotspot_f32":
        W, H = 512, 300
        t = torch.empty((H, W), device="cuda")
        p = torch.empty((H, W), device="cuda")
        O.generate_thermal(0, t.data_ptr(), p.data_ptr(), W, H, stream=sp)
        outs = []
        for v in (vmin, vmax):
            for i in range(len(v)):
                o = torch.empty_like(t)
                v.launch(i, O.hotspot_args(t.data_ptr(), o.data_ptr(), p.data_ptr(), W, H), sp)
                outs.append(o)
    else:
        W, H = 300, 130
        s = torch.from_numpy(synth.noisy_rgba(W, H, seed=3, sigma=0.13)).cuda()
        outs = []
        for v in (vmin, vmax):
            for i in range(len(v)):
                o = torch.empty_like(s)
                v.launch(i, O.denoise_args(kernel, s.data_ptr(), o.data_ptr(), W, H), sp)
                outs.append(o)
    torch.cuda.synchronize()
    for o in outs[1:]:
        assert torch.equal(o, outs[0])


def test_lowest_within_tol_selection(sp):
    W = H = 2048
    v, _ = O.build_all_levels(0, "hotspot_f32", mode=O.REALISE_MIN_CARVEOUT)
    t = torch.empty((H, W), device="cuda")
    p = torch.empty((H, W), device="cuda")
    o = torch.empty_like(t)
    O.generate_thermal(0, t.data_ptr(), p.data_ptr(), W, H, stream=sp)
    tu = O.Tuner(v, O.default_cfg(select_mode=O.SELECT_LOWEST_WITHIN_TOL))
    times = {}
    for _ in range(20):
        r = tu.step(O.hotspot_args(t.data_ptr(), o.data_ptr(), p.data_ptr(), W, H), sp)
        if r.phase == 0:
            times[r.level_idx] = r.ms
    final, _ = tu.final()
    assert final >= 0
    best = min(times.values())
    assert times[final] <= best * 1.02 + 1e-9
    within = [i for i, ms in times.items() if ms <= best * 1.02]
    assert v.level(final).ctas_per_sm == min(v.level(i).ctas_per_sm for i in within)
    np.testing.assert_array_equal(o.shape, t.shape)
