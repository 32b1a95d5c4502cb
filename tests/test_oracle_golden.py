"""Golden pins: values PAPER.md prints, reproduced by the oracle's O1 (occupancy calculator) and
O4 (Fig. 8 prune) -- and by liborion's independent host-only implementation -- on the paper's own
GTX680 platform.  Each fixture under tests/golden/ carries its citations."""
import json
import os

import pytest

from oracle import occupancy as OC
from oracle import tuner as OT
from paper_conf_middleware_hayeslcsz16_b200 import orion as O

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def _gtx680_product_limits():
    d = O.DeviceLimits()
    for k, v in OC.GTX680.as_dict().items():
        setattr(d, k, v)
    return d


def _oracle_ladders(regs, T):
    lv = OC.levels(OC.GTX680, T, regs)
    direction, ladder, other = OT.candidates(lv, regs, OT.TunerCfg())    # Fig. 8: walk + fail-safe
    return lv, direction, ladder, other


def test_fig1_occupancy_axis_and_best():
    g = load("paper_fig1_gtx680_imagedenoising.json")
    lv, direction, ladder, other = _oracle_ladders(g["registers"], g["block_threads"])
    assert direction == OT.INCREASING
    # the levels Orion generates for imageDenoising: the register-cap rungs of the increasing
    # ladder and the padding levels of its fail-safe (decreasing) ladder
    occ = sorted({lv[i].occupancy_permille / 1000 for i in ladder + other})
    assert [round(o + 1e-9, g["printed_decimals"]) for o in occ] == g["occupancy_axis_printed"]
    # the best point of Fig. 1 is the original (natural-register) build's occupancy
    assert OC.occupancy(OC.GTX680, g["block_threads"],
                        OC.ctas_per_sm(OC.GTX680, g["block_threads"], g["registers"])) == g["best_occupancy_printed"]
    # liborion's host-only calculator agrees with the oracle level by level on the GTX680
    res = O.KernelResources(g["block_threads"], g["registers"], 0, 0, 16)
    prod = O.levels(_gtx680_product_limits(), res)
    assert [(l.ctas_per_sm, l.reg_cap, l.smem_pad_bytes) for l in prod] == \
           [(l.ctas_per_sm, l.reg_cap, l.smem_pad_bytes) for l in lv]


@pytest.mark.parametrize("bench", sorted(load("paper_table2_tuning_directions.json")["registers"]))
def test_table2_direction_split_and_candidate_bound(bench):
    g = load("paper_table2_tuning_directions.json")
    regs, T = g["registers"][bench], g["block_threads"]
    lv, direction, ladder, other = _oracle_ladders(regs, T)
    if bench in g["increase"]:
        assert direction == OT.INCREASING
        assert len(ladder) <= g["max_candidate_versions"]
        assert OC.occupancy(OC.GTX680, T, OC.ctas_per_sm(OC.GTX680, T, regs)) < 1.0
    else:
        assert bench in g["decrease"]
        assert direction == OT.DECREASING
        # their natural build already runs at the hardware's maximum occupancy
        assert OC.occupancy(OC.GTX680, T, OC.ctas_per_sm(OC.GTX680, T, regs)) == 1.0
    # the product's Fig. 8 (host replay on a flat table: only the first iteration matters here)
    res = O.KernelResources(T, regs, 0, 0, 16)
    prod = O.levels(_gtx680_product_limits(), res)
    ran, _, _ = O.tuner_replay(O.default_cfg(allow_direction_switch=0), prod, regs, [1.0] * len(prod), 1)
    assert ran[0] == ladder[0]                                           # the original runs first


def test_golden_sets_are_table2():
    g = load("paper_table2_tuning_directions.json")
    assert sorted(g["increase"] + g["decrease"]) == sorted(g["registers"])
    assert len(g["increase"]) == 7 and len(g["decrease"]) == 5
