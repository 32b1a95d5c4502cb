"""The live tuner on the GPU replayed through the oracle's independent Fig. 9 (O4 pin 1,
SURVEY §8(c); Fig. 9 P:L605-P:L643, P:L687-P:L689; work normalisation P:L975;
kernel splitting P:L691).

Each case runs real iterations through orion_tune_step / orion_tune_split, then:
  1. reads the runtime table Fig. 9 observed (orion_tuner_tried: ns per output element,
     fastest of samples_per_level samples);
  2. in synchronous mode, re-derives every entry of that table from the per-iteration
     reports (raw event ms / output elements, min over the level's samples), so the table
     is what the kernels measured;
  3. replays the table through oracle.tuner.Fig9 (O4) and asserts the same decisions: the
     same levels measured in the same order (O4's insertion order into `tried`; the live
     sequence with repeated samples / async re-launches collapsed) and the same final level.
"""
import numpy as np
import pytest

from oracle import occupancy as OC
from oracle import tuner as OT

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_middleware_hayeslcsz16_b200 import orion as O  # noqa: E402


@pytest.fixture(scope="module")
def sp():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.cuda.current_stream().cuda_stream


def _oracle_levels(v):
    return [OC.Level(l.ctas_per_sm, l.warps_per_sm, l.occupancy_permille, l.reg_cap, l.smem_pad_bytes, l.limiter,
                     l.carveout_kb) for l in v.planned]


def _collapse(seq):
    out = []
    for x in seq:
        if not out or out[-1] != x:
            out.append(x)
    return out


def _check_replay(v, res, cfg, tuner, reports, works, sync):
    tried = tuner.tried()
    table = [t if t >= 0 else float("inf") for t in tried]
    if sync:   # the table is what the event pairs measured, per output element, best of the samples
        per_level = {}
        for r, w in zip(reports, works):
            if r.phase == 0 and r.ms >= 0:
                per_level.setdefault(r.level_idx, []).append(np.float32(float(r.ms) * 1e6 / w))
        for lvl, vals in per_level.items():
            assert np.float32(tried[lvl]) == min(vals), (lvl, tried[lvl], vals)
        assert set(per_level) == {i for i, t in enumerate(tried) if t >= 0}
    ocfg = OT.TunerCfg(maxlive_threshold=cfg.maxlive_threshold, slowdown_tol=cfg.slowdown_tol,
                       worse_eps=cfg.worse_eps, select_mode=cfg.select_mode,
                       allow_direction_switch=bool(cfg.allow_direction_switch))
    f9 = OT.Fig9(_oracle_levels(v), res.regs_per_thread, ocfg)
    for _ in range(len(reports) + 4):
        f9.step(lambda i: table[i])
    live_measured = _collapse([r.level_idx for r in reports if r.phase == 0])
    assert live_measured == list(f9.tried.keys()), (live_measured, list(f9.tried.keys()), table)
    final, _ = tuner.final()
    assert final >= 0 and final == f9.final, (final, f9.final, table)
    return live_measured, final


@pytest.mark.parametrize("kernel,W,H,samples,async_t,select", [
    ("nlm_f4_regheavy", 512, 512, 1, 0, O.SELECT_FASTEST),
    ("nlm_f4_regheavy", 512, 512, 2, 0, O.SELECT_FASTEST),
    ("nlm_f4_regheavy", 512, 512, 2, 1, O.SELECT_FASTEST),
    ("nlm_f4_regheavy", 512, 512, 2, 0, O.SELECT_LOWEST_WITHIN_TOL),
    ("knn_f4", 1024, 1024, 2, 0, O.SELECT_FASTEST),
    ("nlm_f4_w", 1024, 1024, 2, 0, O.SELECT_FASTEST),
])
def test_live_walk_replays_through_o4(sp, kernel, W, H, samples, async_t, select):
    v, res = O.build_all_levels(0, kernel, mode=O.REALISE_MIN_CARVEOUT)
    src = torch.empty((H, W, 4), device="cuda")
    dst = torch.empty_like(src)
    O.generate_rgba(0, src.data_ptr(), W, H, seed=1, sigma=0.13, stream=sp)
    cfg = O.default_cfg(samples_per_level=samples, async_timing=async_t, select_mode=select)
    t = O.Tuner(v, cfg)
    a = O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H)
    reports = []
    for i in range(400):
        reports.append(t.step(a, sp))
        if t.final()[0] >= 0 and reports[-1].phase == 1:
            break
        if async_t and i % 8 == 7:
            # an application that syncs now and then (async timing never blocks; a measurement
            # lands once the GPU has caught up with the host)
            torch.cuda.synchronize()
    torch.cuda.synchronize()
    seq, final = _check_replay(v, res, cfg, t, reports, [W * H] * len(reports), sync=not async_t)
    assert len(seq) >= 2
    t.close()
    v.close()


def test_split_frame_walk_replays_through_o4(sp):
    # unequal bands (301 rows in 40 bands: 37 x 8 + 5, then two empty ones): only work
    # normalisation makes them comparable
    kernel, W, H, bands = "nlm_f4_regheavy", 640, 301, 40
    v, res = O.build_all_levels(0, kernel, mode=O.REALISE_MIN_CARVEOUT)
    src = torch.empty((H, W, 4), device="cuda")
    dst = torch.empty_like(src)
    O.generate_rgba(0, src.data_ptr(), W, H, seed=4, sigma=0.13, stream=sp)
    cfg = O.default_cfg(samples_per_level=1)
    t = O.Tuner(v, cfg)
    reports = t.split(O.denoise_args(kernel, src.data_ptr(), dst.data_ptr(), W, H), bands, sp)
    torch.cuda.synchronize()
    per = -(-H // bands)
    works = [(min(H, (b + 1) * per) - min(H, b * per)) * W for b in range(bands)]
    live = [(r, w) for r, w in zip(reports, works) if r.iteration >= 0]
    assert len(live) == 38 and live[-1][1] != live[0][1]
    _check_replay(v, res, cfg, t, [r for r, _ in live], [w for _, w in live], sync=True)
    t.close()
    v.close()
