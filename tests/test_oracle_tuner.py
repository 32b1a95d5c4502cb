"""Pins for oracle O4 -- Fig. 8 candidate prune and Fig. 9 dynamic selection
(PAPER.md P:L583-L693).

Pins: SURVEY §8(c) O4 traces V1-V5 (Fig. 1 V-shape, Fig. 2 plateau, monotone,
ties), Principle 1 (one local minimum) as a brute-force property
-- on any strictly unimodal runtime table the increasing walk ends at the
global argmin of its ladder -- and Fig. 8's ladder shapes.
"""
import random

from hypothesis import given, settings, strategies as st

from oracle import occupancy as O
from oracle import tuner as TU


def ladder_ks(lv, ladder):
    return [lv[i].ctas_per_sm for i in ladder]


def run(lv, natural, ladder_times, iterations, cfg=None, default=9.9):
    cfg = cfg or TU.TunerCfg()
    d, ladder, _ = TU.candidates(lv, natural, cfg)
    ms = [default] * len(lv)
    for i, t in zip(ladder, ladder_times):
        ms[i] = t
    return d, ladder, TU.replay(lv, natural, cfg, ms, iterations)


def test_fig8_ladders():
    lv = O.levels(O.B200, 128, 255)
    d, ladder, other = TU.candidates(lv, 255, TU.TunerCfg())
    assert d == TU.INCREASING
    assert ladder_ks(lv, ladder) == [2, 3, 4, 5, 6, 7, 8, 9, 10, 12, 16]   # original, conservative .. max
    assert ladder_ks(lv, other) == [2, 1]                                   # fail-safe: pad down
    lv = O.levels(O.B200, 256, 20)
    d, ladder, other = TU.candidates(lv, 20, TU.TunerCfg())
    assert d == TU.DECREASING                                               # MAXLIVE < 32
    assert ladder_ks(lv, ladder) == [8, 7, 6, 5, 4, 3, 2, 1]
    assert ladder_ks(lv, other) == [8]                                      # already at max


def test_v1_fig1_vshape_increasing():
    lv = O.levels(O.B200, 128, 56)            # ladder 9, 10, 12, 16
    d, ladder, tr = run(lv, 56, [1.00, 1.30, 1.80, 2.60], 6)
    assert d == TU.INCREASING and len(ladder) == 4
    assert tr.final == ladder[0] and tr.final_iteration == 1
    assert tr.ran == [ladder[0], ladder[1]] + [ladder[0]] * 4


def test_v2_improve_then_worse():
    lv = O.levels(O.B200, 128, 56)
    _, ladder, tr = run(lv, 56, [1.00, 0.90, 0.85, 0.95], 7)
    assert tr.ran[:4] == ladder[:4]
    assert tr.final == ladder[2] and tr.final_iteration == 3
    assert tr.ran[4:] == [ladder[2]] * 3


def test_v3_fig2_plateau_decreasing_both_modes():
    lv = O.levels(O.B200, 256, 20, 0, 45000)   # smem-limited original at 5 CTAs -> 5,4,3,2,1
    times = [1.000, 1.005, 1.010, 1.015, 1.030]
    d, ladder, tr = run(lv, 20, times, 8)
    assert d == TU.DECREASING and ladder_ks(lv, ladder) == [5, 4, 3, 2, 1]
    assert tr.ran[:5] == ladder and tr.final == ladder[0] and tr.final_iteration == 4
    _, _, tr2 = run(lv, 20, times, 8, TU.TunerCfg(select_mode=TU.LOWEST_WITHIN_TOL))
    assert tr2.final == ladder[3]


def test_v4_monotone_exhausts_ladder():
    lv = O.levels(O.B200, 128, 48)             # ladder 10, 12, 16
    _, ladder, tr = run(lv, 48, [1.0, 0.9, 0.8], 5)
    assert len(ladder) == 3
    assert tr.ran == ladder + [ladder[2]] * 2
    assert tr.final == ladder[2] and tr.final_iteration == 3


def test_v5_ties_prefer_lower_occupancy():
    lv = O.levels(O.B200, 128, 40)             # ladder 12, 16
    _, ladder, tr = run(lv, 40, [1.0, 1.0], 4)
    assert len(ladder) == 2
    assert tr.ran[:2] == ladder               # a tie is not "worse": the walk continues
    assert tr.final == ladder[0]              # Principle 2: lower occupancy on a tie


def test_cantune_false_runs_original():
    lv = O.levels(O.B200, 128, 255)
    cfg = TU.TunerCfg(expected_iterations=5)   # < |ladder| + 2
    _, ladder, tr = run(lv, 255, [1.0] * 11, 5, cfg)
    assert tr.ran == [ladder[0]] * 5


def test_direction_switch_failsafe():
    lv = O.levels(O.B200, 128, 56)             # up: 9,10,12,16 ; down: 9,8,...,1
    cfg = TU.TunerCfg(allow_direction_switch=True)
    d, ladder, other = TU.candidates(lv, 56, cfg)
    ms = [9.9] * len(lv)
    ks = {l.ctas_per_sm: i for i, l in enumerate(lv)}
    for k, t in {9: 1.0, 10: 1.2, 8: 0.9, 7: 0.8, 6: 0.85}.items():
        ms[ks[k]] = t
    tr = TU.replay(lv, 56, cfg, ms, 8)
    assert [lv[i].ctas_per_sm for i in tr.ran[:5]] == [9, 10, 8, 7, 6]
    assert lv[tr.final].ctas_per_sm == 7


@settings(max_examples=300, deadline=None)
@given(st.integers(min_value=0, max_value=10), st.integers(min_value=0, max_value=2**31 - 1))
def test_principle1_unimodal_walk_finds_global_argmin(argmin_pos, seed):
    lv = O.levels(O.B200, 128, 255)
    _, ladder, _ = TU.candidates(lv, 255, TU.TunerCfg())
    n = len(ladder)
    rng = random.Random(seed)
    # strictly decreasing to argmin_pos, strictly increasing after it
    t = [0.0] * n
    t[argmin_pos] = 1.0
    for p in range(argmin_pos - 1, -1, -1):
        t[p] = t[p + 1] + rng.uniform(0.01, 0.5)
    for p in range(argmin_pos + 1, n):
        t[p] = t[p - 1] + rng.uniform(0.01, 0.5)
    ms = [50.0] * len(lv)
    for i, x in zip(ladder, t):
        ms[i] = x
    tr = TU.replay(lv, 255, TU.TunerCfg(), ms, n + 3)
    brute = min(ladder, key=lambda i: ms[i])   # exhaustive search over the ladder
    assert tr.final == brute
    assert TU.regret(ms[tr.final], ms[brute]) == 0.0
    # iterations spent exploring: up to the first worse level (or the whole ladder)
    assert tr.final_iteration == min(argmin_pos + 1, n - 1) + (1 if argmin_pos == n - 1 else 0)


def test_fig8_ladders_under_min_carveout_realisation():
    # the smallest-carveout realisation leaves some capped levels unpadded; the ladders are
    # defined by register caps, so they do not change with the realisation
    for T, natural, need in ((256, 30, 9256), (128, 255, 11264), (256, 46, 0)):
        a = O.levels(O.B200, T, natural, 0, need)
        b = O.levels(O.B200, T, natural, 0, need, mode=O.REALISE_MIN_CARVEOUT)
        ca, cb = TU.candidates(a, natural, TU.TunerCfg()), TU.candidates(b, natural, TU.TunerCfg())
        assert ca[0] == cb[0]
        assert ladder_ks(a, ca[1]) == ladder_ks(b, cb[1]) and ladder_ks(a, ca[2]) == ladder_ks(b, cb[2])
        assert O.original_level_index(a) == O.original_level_index(b)
