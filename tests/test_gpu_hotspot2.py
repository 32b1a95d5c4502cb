"""hotspot2h_f32 (two explicit steps per launch, the intermediate step kept in registers, whole
halo lanes) and hotspot4h_f32 (four steps per launch, a 4-stage register pipeline on the
halo-lane warps):
bit-identical to two launches of the one-step kernel and to the oracle's fp32 form, at every
occupancy level, on ragged heights and at the image borders."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module", params=["hotspot2h_f32", "hotspot4h_f32"])
def v2(request):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    v = O.build_all_levels(0, request.param, mode=O.REALISE_MIN_CARVEOUT)[0]
    v.spl = O.STEPS_PER_LAUNCH[request.param]
    return v


def run(v, level, t0, pw, launches):
    sp = torch.cuda.current_stream().cuda_stream
    H, W = t0.shape
    a = torch.from_numpy(t0).cuda()
    b = torch.empty_like(a)
    p = torch.from_numpy(pw).cuda()
    for _ in range(launches):
        v.launch(level, O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H), sp)
        a, b = b, a
    torch.cuda.synchronize()
    return a.cpu().numpy()


@pytest.mark.parametrize("shape", [(300, 203), (128, 1), (132, 2), (260, 3), (512, 129), (4, 37), (120, 9),
                                   (124, 40), (244, 33), (8, 70)])
def test_two_steps_bit_exact_vs_oracle_fp32(v2, shape):
    W, H = shape
    t0, pw = synth.thermal_inputs(W, H, seed=5)
    ref = oracle.hotspot(t0, pw, 5 * v2.spl, precision="f32")
    for lvl in (0, len(v2) - 1):
        assert np.array_equal(run(v2, lvl, t0, pw, 5), ref), (shape, lvl)


def test_all_levels_identical(v2):
    t0, pw = synth.thermal_inputs(520, 300, seed=1)
    outs = [run(v2, i, t0, pw, 3) for i in range(len(v2))]
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])
    assert np.array_equal(outs[0], oracle.hotspot(t0, pw, 3 * v2.spl, precision="f32"))


def test_unaligned_width_rejected(v2):
    t0, pw = synth.thermal_inputs(130, 20, seed=1)
    with pytest.raises(O.OrionError) as e:
        run(v2, 0, np.ascontiguousarray(t0[:, :129]), np.ascontiguousarray(pw[:, :129]), 1)
    assert e.value.status == -1
