"""Pins for oracle O1 (occupancy calculator + levels) -- PAPER.md Eq. (1).

The oracle is pinned to things other than itself:
  * SURVEY.md Appendix A hand-worked tables (B200, cc 10.0);
  * NVIDIA's header-only cudaOccMaxActiveBlocksPerMultiprocessor (an independent
    implementation, compiled from cuda_occupancy.h by tests/helpers/occ_ref.cpp);
  * the Kepler GTX680 case behind Fig. 1 (P:L91 best at 50 %, P:L713 platform,
    Table 2 P:L733 imageDenoising 63 registers).
"""
import itertools

import pytest

from oracle import occupancy as O

# regs/thread -> CTAs/SM at T = 64, 128, 256.
APPENDIX_A = {
    32: (32, 16, 8), 40: (24, 12, 6), 48: (20, 10, 5), 56: (18, 9, 4), 64: (16, 8, 4),
    72: (14, 7, 3), 80: (12, 6, 3), 88: (10, 5, 2), 96: (10, 5, 2), 104: (8, 4, 2),
    128: (8, 4, 2), 136: (6, 3, 1), 168: (6, 3, 1), 176: (4, 2, 1), 255: (4, 2, 1),
}
# Appendix A: dynamic bytes pinning exactly k CTAs/SM at T=64, no static smem.
APPENDIX_A_PAD = {1: 115840, 2: 76928, 3: 57472, 4: 45696, 8: 24960, 12: 17024, 16: 12800,
                  24: 8320, 31: 6400, 32: 0}


@pytest.mark.parametrize("regs", sorted(APPENDIX_A))
def test_appendix_a_register_table(regs):
    for T, want in zip((64, 128, 256), APPENDIX_A[regs]):
        assert O.ctas_per_sm(O.B200, T, regs) == want, (T, regs)


@pytest.mark.parametrize("k", sorted(APPENDIX_A_PAD))
def test_appendix_a_pad_table(k):
    pad = O.pad_for(O.B200, 64, 32, 0, 0, k)
    assert pad == APPENDIX_A_PAD[k]
    assert O.ctas_per_sm(O.B200, 64, 32, 0, pad) == k
    if pad > 0:  # minimal: 128 bytes less admits k+1
        assert O.ctas_per_sm(O.B200, 64, 32, 0, pad - 128) == k + 1


def test_against_nvidia_header_grid(occ_ref):
    cases = []
    for T in (32, 64, 96, 128, 160, 256, 384, 512, 1024):
        for regs in (16, 24, 32, 37, 39, 40, 48, 56, 63, 64, 72, 80, 96, 128, 168, 200, 255):
            for sst, sdyn in ((0, 0), (0, 4096), (2048, 10000), (8192, 0), (0, 45000), (0, 100000),
                              (1024, 226000)):
                cases.append((T, regs, sst, sdyn))
    want = occ_ref(cases)
    got = [O.ctas_per_sm(O.B200, *c) for c in cases]
    bad = [(c, g, w) for c, g, w in zip(cases, got, want) if g != w]
    assert not bad, bad[:10]


@pytest.mark.parametrize("T,natural,need", [(64, 39, 0), (128, 255, 0), (128, 39, 8704), (256, 20, 0),
                                            (128, 200, 30000), (256, 96, 2048), (64, 255, 4096)])
def test_every_level_realises_k_per_nvidia_header(occ_ref, T, natural, need):
    lv = O.levels(O.B200, T, natural, 0, need)
    assert [l.ctas_per_sm for l in lv] == sorted({l.ctas_per_sm for l in lv})
    cases = [(T, natural if l.reg_cap == 0 else l.reg_cap, 0, need + l.smem_pad_bytes) for l in lv]
    assert occ_ref(cases) == [l.ctas_per_sm for l in lv]
    # k_max is reached and every k below it is feasible (reading R-A10)
    assert [l.ctas_per_sm for l in lv] == list(range(1, lv[-1].ctas_per_sm + 1))


def test_register_ladder_255_regs_T128():
    lv = {l.ctas_per_sm: l for l in O.levels(O.B200, 128, 255)}
    rungs = {k: l.reg_cap for k, l in lv.items() if l.smem_pad_bytes == 0}
    assert rungs == {2: 0, 3: 168, 4: 128, 5: 96, 6: 80, 7: 72, 8: 64, 9: 56, 10: 48, 12: 40, 16: 32}
    assert lv[1].reg_cap == 0 and lv[1].smem_pad_bytes > 0
    assert lv[11].reg_cap == 40 and lv[11].smem_pad_bytes > 0
    assert O.original_level_index(list(lv.values())) == 1


def test_kepler_gtx680_fig1_sanity():
    # imageDenoising 63 regs (Table 2) at 256 threads -> 4 CTAs = 32 warps = 50 % (Fig. 1 best).
    assert O.ctas_per_sm(O.GTX680, 256, 63) == 4
    assert O.occupancy(O.GTX680, 256, 4) == 0.5
    assert O.ctas_per_sm(O.GTX680, 64, 63) == 16  # 16-CTA Kepler limit binds at 8x8 CTAs
    caps = {32: 1.0, 40: 0.75, 48: 0.625, 56: 0.5}
    for r, occ in caps.items():
        assert O.occupancy(O.GTX680, 256, O.ctas_per_sm(O.GTX680, 256, r)) == occ
    # 0.875 is unreachable by register caps (absent from Fig. 1's axis)
    reach = {O.occupancy(O.GTX680, 256, O.ctas_per_sm(O.GTX680, 256, r)) for r in range(16, 64)}
    assert 0.875 not in reach


def test_limiter_mask_and_eq1_upper_bound():
    # Eq. (1) without granularity is an upper bound of the calculator's answer.
    for T, regs, smem in itertools.product((64, 128, 256), (24, 40, 64, 128, 255), (0, 8192, 40000)):
        k = O.ctas_per_sm(O.B200, T, regs, 0, smem)
        eq1_threads = min(65536 / regs, 233472 / ((smem + 1024) / T))
        assert k * T <= eq1_threads + 1e-9
        m = O.limiter_mask(O.B200, T, regs, 0, smem)
        assert m != 0


CARVEOUT_PCTS = (-1, 0, 3, 7, 14, 28, 43, 50, 57, 71, 85, 99, 100)


def test_carveout_preferences_against_nvidia_header(occ_ref):
    # the unified L1 / shared-memory carveout (small vs large cache, Table 3)
    cases = []
    for T in (64, 128, 256):
        for regs in (24, 40, 64, 128):
            for sdyn in (0, 3000, 9000, 30000, 60000, 120000):
                for pct in CARVEOUT_PCTS:
                    cases.append((T, regs, 0, sdyn, pct))
    want = occ_ref(cases)
    got = [O.ctas_per_sm(O.B200, T, r, s, d, None if p < 0 else p) for (T, r, s, d, p) in cases]
    bad = [(c, g, w) for c, g, w in zip(cases, got, want) if g != w]
    assert not bad, bad[:10]


def test_carveout_percent_maps_to_each_configuration():
    for kb in O.CARVEOUT_KB[1:]:
        pct = O.carveout_pct_for(O.B200, kb)
        assert O.carveout_budget(O.B200, pct) == kb * 1024
        if pct < 100:
            assert O.carveout_budget(O.B200, pct + 1) > kb * 1024


@pytest.mark.parametrize("T,natural,need", [(256, 46, 0), (128, 255, 11264), (128, 56, 13376), (128, 255, 108756)])
def test_min_carveout_levels_realise_k_per_nvidia_header(occ_ref, T, natural, need):
    lmax = O.levels(O.B200, T, natural, 0, need)
    lmin = O.levels(O.B200, T, natural, 0, need, mode=O.REALISE_MIN_CARVEOUT)
    assert [l.ctas_per_sm for l in lmin] == [l.ctas_per_sm for l in lmax]
    assert [l.reg_cap for l in lmin] == [l.reg_cap for l in lmax]
    cases = [(T, natural if l.reg_cap == 0 else l.reg_cap, 0, need + l.smem_pad_bytes,
              O.carveout_pct_for(O.B200, l.carveout_kb)) for l in lmin]
    assert occ_ref(cases) == [l.ctas_per_sm for l in lmin]
    for a, b in zip(lmin, lmax):        # never a larger shared-memory carve-out than MAX_SMEM
        assert 0 < a.carveout_kb <= 228
        assert a.carveout_kb * 1024 <= max(b.carveout_kb * 1024, O.B200.smem_per_sm)
    # a kernel without shared memory keeps almost all of the array as L1 at every level
    if need == 0:
        assert max(l.carveout_kb for l in lmin) <= 100


# cuda_occupancy.h's OCC_LIMIT_* bits -> the oracle's (orion.h's) LIM_* bits
_HDR_TO_ORACLE = {0x01: O.LIM_WARPS, 0x02: O.LIM_REGS, 0x04: O.LIM_SMEM, 0x08: O.LIM_BLOCKS}


def _from_header_mask(m):
    return sum(v for b, v in _HDR_TO_ORACLE.items() if m & b)


def test_limiter_mask_against_nvidia_limiting_factors(occ_ref):
    # The limiter bitmask of a level is pinned to cudaOccResult.limitingFactors:
    # every limit that equals the final CTA count, ties included (warps + registers, etc.).
    cases = []
    for T in (32, 64, 128, 256, 512, 1024):
        for regs in (16, 32, 40, 48, 64, 72, 128, 168, 255):
            for sst, sdyn in ((0, 0), (0, 6144), (0, 12800), (2048, 30000), (0, 76928), (0, 115840)):
                for pct in (-1, 28, 100):
                    cases.append((T, regs, sst, sdyn, pct))
    want = occ_ref(cases, mask=True)
    bad = []
    for (T, r, s, d, p), (k, m) in zip(cases, want):
        pct = None if p < 0 else p
        if O.ctas_per_sm(O.B200, T, r, s, d, pct) != k or \
                O.limiter_mask(O.B200, T, r, s, d, pct) != _from_header_mask(m):
            bad.append(((T, r, s, d, p), O.limiter_mask(O.B200, T, r, s, d, pct), _from_header_mask(m)))
    assert not bad, bad[:10]
    # the grid exercises every limiter alone and the common ties
    masks = {_from_header_mask(m) for _, m in want}
    for bit in (O.LIM_REGS, O.LIM_SMEM, O.LIM_WARPS, O.LIM_BLOCKS):
        assert bit in masks
    assert any(m & (m - 1) for m in masks)


def test_every_level_limiter_against_nvidia_header(occ_ref):
    # the limiter field of each realised level equals the header's answer for that realisation
    for T, natural, need in [(64, 39, 0), (128, 255, 0), (128, 39, 8704), (256, 96, 2048)]:
        for mode in (O.REALISE_MAX_SMEM, O.REALISE_MIN_CARVEOUT):
            lv = O.levels(O.B200, T, natural, 0, need, mode=mode)
            cases = [(T, natural if l.reg_cap == 0 else l.reg_cap, 0, need + l.smem_pad_bytes,
                      O.carveout_pct_for(O.B200, l.carveout_kb) if l.carveout_kb > 0 else -1) for l in lv]
            got = occ_ref(cases, mask=True)
            assert [(l.ctas_per_sm, l.limiter) for l in lv] == [(k, _from_header_mask(m)) for k, m in got]
