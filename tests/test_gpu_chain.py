"""orion_chain (orion.h): consecutive stencil iterations on one grid, each launch waiting for the
previous one tile by tile instead of grid-wide, so iteration n+1 fills iteration n's last wave
(the iterations of PAPER.md P:L605-P:L607, overlapped).  The bits must be exactly those of
ordinary launches -- the f32 oracle for the thermal stencil (reading R-HS-S), the unchained
kernel for SRAD -- over many launches, alternating levels, through the tuner, with foreign
liborion kernels in between, and with PDL off; misuse must be refused."""
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


@pytest.fixture(scope="module")
def hs():
    return O.build_all_levels(0, "hotspot4h_f32", mode=O.REALISE_MIN_CARVEOUT)[0]


@pytest.fixture(scope="module")
def sr():
    return O.build_all_levels(0, "srad_f32hs", mode=O.REALISE_MIN_CARVEOUT)[0]


def hotspot_run(v, t0, pw, launches, sp, chained=True, levels=None, between=None):
    H, W = t0.shape
    a = torch.from_numpy(t0).cuda()
    b = torch.full_like(a, float("nan"))
    p = torch.from_numpy(pw).cuda()
    ch = O.Chain(v, W, H) if chained else None
    for n in range(launches):
        lvl = levels[n % len(levels)] if levels else len(v) - 1
        v.launch(lvl, O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H, chain=ch), sp)
        if between is not None:
            between(n)
        a, b = b, a
    torch.cuda.synchronize()
    if ch is not None:
        assert ch.info()[0] == launches
        ch.close()
    return a.cpu().numpy()


@pytest.mark.parametrize("W,H", [(1000, 1100), (484, 2000), (2048, 1537), (124, 9), (8, 600)])
def test_chained_hotspot_equals_oracle_fp32(sp, hs, W, H):
    t0, pw = synth.thermal_inputs(W, H, seed=3)
    got = hotspot_run(hs, t0, pw, 25, sp, levels=list(range(len(hs))))
    assert np.array_equal(got, oracle.hotspot(t0, pw, 100, precision="f32"))


def test_chained_hotspot_many_tiles_matches_unchained(sp, hs):
    # 35 x 8 tiles, 60 launches: a missed dependency would show as a difference somewhere
    W, H = 4096, 4000
    t0, pw = synth.thermal_inputs(W, H, seed=9)
    assert np.array_equal(hotspot_run(hs, t0, pw, 60, sp), hotspot_run(hs, t0, pw, 60, sp, chained=False))


def test_chained_hotspot_with_foreign_kernels_between(sp, hs):
    # another liborion kernel on the stream between two chained launches: the next one waits
    # grid-wide (orion_launch tracks the stream's last kernel)
    W, H = 1000, 1100
    t0, pw = synth.thermal_inputs(W, H, seed=4)
    junk_t = torch.empty((H, W), device="cuda")
    junk_p = torch.empty((H, W), device="cuda")

    def between(n):
        if n % 3 == 1:
            O.generate_thermal(0, junk_t.data_ptr(), junk_p.data_ptr(), W, H, seed=n, stream=sp)

    got = hotspot_run(hs, t0, pw, 12, sp, between=between)
    assert np.array_equal(got, oracle.hotspot(t0, pw, 48, precision="f32"))


def test_chained_hotspot_without_pdl(sp, hs):
    W, H = 1000, 1100
    t0, pw = synth.thermal_inputs(W, H, seed=5)
    prev = O.set_pdl(False)
    try:
        got = hotspot_run(hs, t0, pw, 10, sp)
    finally:
        O.set_pdl(prev)
    assert np.array_equal(got, oracle.hotspot(t0, pw, 40, precision="f32"))


def srad_run(v, j0, iters, sp, roi, chained=True, levels=None):
    H, W = j0.shape
    n = H * W + O.SRAD_STATS_FLOATS
    a = torch.zeros(n, device="cuda")
    b = torch.zeros(n, device="cuda")
    a[:H * W] = torch.from_numpy(np.ascontiguousarray(j0, dtype=np.float32).ravel()).cuda()
    O.srad_stats_init(0, a.data_ptr(), W, H, roi, sp)
    ch = O.Chain(v, W, H) if chained else None
    for k in range(iters):
        lvl = levels[k % len(levels)] if levels else len(v) - 1
        v.launch(lvl, O.srad_args(a.data_ptr(), b.data_ptr(), 0, W, H, roi=roi, chain=ch), sp)
        a, b = b, a
    torch.cuda.synchronize()
    if ch is not None:
        ch.close()
    return a[:H * W].reshape(H, W).cpu().numpy()


@pytest.mark.parametrize("W,H,roi", [(1000, 1100, (0, 127, 0, 127)), (2048, 1500, (5, 700, 100, 290)),
                                     (484, 800, (300, 799, 400, 483))])
def test_chained_srad_equals_unchained(sp, sr, W, H, roi):
    j0, _ = synth.thermal_inputs(W, H, seed=6)
    lv = list(range(len(sr)))
    got = srad_run(sr, j0, 20, sp, roi, levels=lv)
    ref = srad_run(sr, j0, 20, sp, roi, chained=False)
    assert np.array_equal(got, ref)
    o, _ = oracle.srad(j0.astype(np.float64), 20, 0.5, roi)
    assert (np.abs(got - o) / np.abs(o)).max() < 1e-5


def test_chained_launches_through_the_tuner(sp, hs):
    # the Fig. 9 walk switches levels between chained iterations; the bits stay the oracle's
    W, H = 2048, 1200
    t0, pw = synth.thermal_inputs(W, H, seed=8)
    a = torch.from_numpy(t0).cuda()
    b = torch.empty_like(a)
    p = torch.from_numpy(pw).cuda()
    t = O.Tuner(hs, O.default_cfg(samples_per_level=1))
    ch = O.Chain(hs, W, H)
    for _ in range(30):
        t.step(O.hotspot_args(a.data_ptr(), b.data_ptr(), p.data_ptr(), W, H, chain=ch), sp)
        a, b = b, a
    torch.cuda.synchronize()
    assert t.final()[0] >= 0
    assert np.array_equal(a.cpu().numpy(), oracle.hotspot(t0, pw, 120, precision="f32"))
    ch.close()
    t.close()


def test_chain_misuse_refused(sp, hs, sr):
    W, H = 256, 600
    t = torch.zeros((H, W), device="cuda")
    ch = O.Chain(hs, W, H)
    for kernel in ("hotspot_f32", "srad_f32h", "nlm_f4_w"):             # families without chains
        v, _ = O.build_all_levels(0, kernel)
        with pytest.raises(O.OrionError):
            O.Chain(v, W, H)
    bad = [O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H, row_begin=0, row_end=300, chain=ch),
           O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W + 4, H, chain=ch),
           O.with_fanout(O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H, chain=ch), [None, None])]
    flagged = O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H, chain=ch)
    flagged.flags = O.ARGS_INDEPENDENT
    bad.append(flagged)
    for a in bad:
        with pytest.raises(O.OrionError) as e:
            hs.launch(0, a, sp)
        assert e.value.status == -1
    ok = O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H, chain=ch)
    with pytest.raises(O.OrionError):                                    # another family's chain
        sr.launch(0, O.srad_args(t.data_ptr(), t.data_ptr(), 0, W, H, roi=(0, 10, 0, 10), chain=ch), sp)
    with pytest.raises(O.OrionError):                                    # the sweep repeats one launch
        hs.sweep(ok, sp, rounds=1)
    hs.launch(0, ok, sp)
    other = torch.cuda.Stream()
    with pytest.raises(O.OrionError):                                    # one stream per chain
        hs.launch(0, ok, other.cuda_stream)
    torch.cuda.synchronize()
    assert ch.info()[0] == 1
    tu = O.Tuner(hs, O.default_cfg(samples_per_level=1))
    plain = O.hotspot_args(t.data_ptr(), t.data_ptr(), t.data_ptr(), W, H)
    for _ in range(40):
        tu.step(plain, sp)
        if tu.final()[0] >= 0:
            break
    torch.cuda.synchronize()
    with pytest.raises(O.OrionError):                                    # graphs bake the epochs in
        tu.capture([ok, ok], sp)
    tu.close()
    ch.close()
