"""The C-ABI library on the CPU: it loads, exports every symbol include/orion.h declares,
and its host-only entry points agree with the oracle:

* orion_levels / orion_ctas_per_sm  == oracle O1, field by field (bit-exact integers);
* orion_tuner_replay (the product's Fig. 8 + Fig. 9 state machine) == oracle O4's decision
  sequence on the SURVEY O4 vectors and on random runtime tables;
* the embedded ptxas honours every register cap (regs <= cap) -- the realisation of a level.
No compute call runs here (no GPU).
"""
import itertools
import os
import random
import re

import pytest
from hypothesis import given, settings, strategies as st

from oracle import occupancy as OC
from oracle import tuner as OT
from paper_conf_middleware_hayeslcsz16_b200 import orion as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_symbols():
    txt = open(os.path.join(ROOT, "include", "orion.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(orion_[a-z0-9_]+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    lib = O.lib()
    syms = header_symbols()
    assert len(syms) >= 29
    missing = [s for s in syms if not hasattr(lib, s)]
    assert not missing, missing
    assert O.version().startswith("liborion")


def _to_oracle_dev(d: O.DeviceLimits) -> OC.Device:
    return OC.Device(**{n: getattr(d, n) for n, _ in O.DeviceLimits._fields_})


def test_b200_limits_match_oracle_device():
    assert _to_oracle_dev(O.b200_limits()) == OC.B200


def test_ctas_per_sm_matches_oracle_grid():
    d = O.b200_limits()
    for T, r, s, dyn in itertools.product((32, 64, 96, 128, 256, 512, 1024), (16, 24, 32, 40, 56, 64, 96, 128, 200, 255),
                                          (0, 4096), (0, 3000, 45000, 120000, 231424)):
        k, lim = O.ctas_per_sm(d, T, r, s, dyn)
        assert k == OC.ctas_per_sm(OC.B200, T, r, s, dyn), (T, r, s, dyn)
        assert lim == OC.limiter_mask(OC.B200, T, r, s, dyn), (T, r, s, dyn)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("T", [64, 128, 256, 512])
@pytest.mark.parametrize("natural", [16, 24, 32, 37, 39, 46, 56, 63, 64, 72, 96, 128, 168, 200, 241, 255])
@pytest.mark.parametrize("smem", [(0, 0), (0, 13376), (1024, 8192), (0, 52544), (0, 100000)])
def test_levels_bit_exact_vs_oracle(T, natural, smem, mode):
    d = O.b200_limits()
    got = [l.as_tuple() for l in O.levels(d, O.resources(T, natural, smem[0], smem[1]), mode)]
    want = [(l.ctas_per_sm, l.warps_per_sm, l.occupancy_permille, l.reg_cap, l.smem_pad_bytes, l.limiter,
             l.carveout_kb) for l in OC.levels(OC.B200, T, natural, smem[0], smem[1], mode=mode)]
    assert got == want


def test_ctas_per_sm_carveout_matches_oracle():
    d = O.b200_limits()
    for T, r, dyn, pct in itertools.product((64, 128, 256), (24, 64, 128), (0, 3000, 30000, 120000),
                                            (-1, 0, 3, 14, 28, 43, 71, 100)):
        k, lim = O.ctas_per_sm(d, T, r, 0, dyn, pct)
        p = None if pct < 0 else pct
        assert k == OC.ctas_per_sm(OC.B200, T, r, 0, dyn, p), (T, r, dyn, pct)
        assert lim == OC.limiter_mask(OC.B200, T, r, 0, dyn, p)


def test_levels_capacity_protocol():
    import ctypes
    d = O.b200_limits()
    res = O.resources(128, 255)
    n = ctypes.c_int()
    arr = (O.Level * 3)()
    st_ = O.lib().orion_levels(ctypes.byref(d), ctypes.byref(res), arr, 3, ctypes.byref(n))
    assert st_ == -2 and n.value == 16
    bad = O.resources(0, 40)
    assert O.lib().orion_levels(ctypes.byref(d), ctypes.byref(bad), arr, 3, ctypes.byref(n)) == -1
    assert "bad kernel resources" in O.lib().orion_last_error().decode()


def _o_levels(T, natural, need=0, mode=0):
    ol = OC.levels(OC.B200, T, natural, 0, need, mode=mode)
    return ol, [O.Level(*[getattr(l, f) for f, _ in O.Level._fields_]) for l in ol]



def _replay_both(T, natural, need, ms, iters, mode=0, **cfgkw):
    ol, pl = _o_levels(T, natural, need, mode)
    ocfg = OT.TunerCfg(**{k: v for k, v in cfgkw.items()})
    pcfg = O.default_cfg(**{k: (int(v) if isinstance(v, bool) else v) for k, v in cfgkw.items()})
    tr = OT.replay(ol, natural, ocfg, ms, iters)
    ran, fin, fit = O.tuner_replay(pcfg, pl, natural, ms, iters)
    return tr, ran, fin, fit


@pytest.mark.parametrize("T,natural,need,ladder_ms,mode", [
    (128, 56, 0, [1.00, 1.30, 1.80, 2.60], 0),                 # V1
    (128, 56, 0, [1.00, 0.90, 0.85, 0.95], 0),                 # V2
    (256, 20, 45000, [1.000, 1.005, 1.010, 1.015, 1.030], 0),  # V3 FASTEST
    (256, 20, 45000, [1.000, 1.005, 1.010, 1.015, 1.030], 1),  # V3 LOWEST_WITHIN_TOL
    (128, 48, 0, [1.0, 0.9, 0.8], 0),                          # V4
    (128, 40, 0, [1.0, 1.0], 0),                               # V5
])
def test_replay_vectors_match_oracle(T, natural, need, ladder_ms, mode):
    ol, _ = _o_levels(T, natural, need)
    _, ladder, _ = OT.candidates(ol, natural, OT.TunerCfg())
    ms = [9.5] * len(ol)
    for i, t in zip(ladder, ladder_ms):
        ms[i] = t
    tr, ran, fin, fit = _replay_both(T, natural, need, ms, 10, select_mode=mode, allow_direction_switch=False)
    assert ran == tr.ran and fin == tr.final and fit == tr.final_iteration


@settings(max_examples=200, deadline=None)
@given(st.sampled_from([(128, 255, 0), (128, 56, 0), (256, 20, 0), (256, 46, 0), (128, 128, 52544), (64, 39, 13376)]),
       st.integers(0, 2**31 - 1), st.sampled_from([0, 1]), st.booleans(), st.integers(0, 20), st.sampled_from([0, 1]))
def test_replay_random_tables_match_oracle(shape, seed, mode, switch, expected, realise):
    T, natural, need = shape
    ol, _ = _o_levels(T, natural, need, realise)
    rng = random.Random(seed)
    ms = [round(rng.uniform(0.5, 2.0), 3) for _ in ol]
    tr, ran, fin, fit = _replay_both(T, natural, need, ms, 25, realise, select_mode=mode,
                                     allow_direction_switch=switch, expected_iterations=expected)
    assert ran == tr.ran
    assert fin == (tr.final if tr.final is not None else -1)
    assert fit == (tr.final_iteration if tr.final_iteration is not None else -1)


@pytest.mark.parametrize("kernel", ["knn_f4", "nlm_f4", "nlm_f4_regheavy", "hotspot_f32", "hotspot2h_f32", "hotspot4h_f32", "srad_f32"])
def test_embedded_ptxas_honours_register_caps(kernel):
    res = O.kernel_probe(kernel)
    assert res.regs_per_thread > 0 and res.block_threads in (64, 128, 256)
    for l in O.levels(O.b200_limits(), res):
        if l.reg_cap:
            info = O.compile_info(kernel, res.block_threads, l.reg_cap)
            assert info["regs"] <= l.reg_cap


def test_device_entry_points_fail_cleanly_without_gpu():
    if os.path.exists("/dev/nvidia0"):
        pytest.skip("a GPU is present")
    with pytest.raises(O.OrionError) as e:
        O.query_limits(0)
    assert e.value.status == -5


def test_default_params_match_the_oracles_constants():
    # liborion's method parameters (orion_default_params, C++) and the oracle's (Python) are
    # written independently; they must agree to fp32 (the kernels' parameter precision)
    import numpy as np
    import oracle
    f32 = np.float32
    for k in ("knn_f4", "knn_f4_t16"):
        p = O.default_params(k)
        assert p[:4] == (f32(oracle.KNN["noise"]), f32(oracle.KNN["lerpc"]), f32(oracle.KNN["wthr"]),
                         f32(oracle.KNN["lthr"]))
    for k in ("nlm_f4_w", "nlm_f4_regheavy"):
        p = O.default_params(k)
        assert p[:4] == (f32(oracle.NLM["noise"]), f32(oracle.NLM["lerpc"]), f32(oracle.NLM["wthr"]),
                         f32(oracle.NLM["lthr"]))
    c = oracle.hotspot_constants()
    for k in ("hotspot_f32", "hotspot4h_f32"):
        assert O.default_params(k)[:5] == tuple(f32(c[n]) for n in ("sdc", "rx", "ry", "rz", "amb"))
    assert O.default_params("srad_f32h")[0] == 0.5
    with pytest.raises(O.OrionError):
        O.default_params("no_such_kernel")


def test_every_header_entry_cites_its_passage():
    # each declaration in include/orion.h is preceded by a comment citing the passage (PAPER.md
    # line, figure / equation, SURVEY section or DESIGN reading) that defines the operation
    txt = open(os.path.join(ROOT, "include", "orion.h")).read()
    missing = []
    for m in re.finditer(r"\n(orion_status|void|const char \*|long long) (orion_[a-z0-9_]+)\(", txt):
        before = txt[:m.start()].rstrip()
        end = before.rfind("*/")
        if before[end:].count(";") > 2:        # no comment block within the last declarations
            missing.append(m.group(2))
            continue
        com = before[before.rfind("/*", 0, end):end]
        if not re.search(r"P:L|SURVEY|reading|Fig\.|Eq\.", com):
            missing.append(m.group(2))
    assert not missing, missing


def test_set_pdl_switch_host_only():
    prev = O.set_pdl(False)
    try:
        assert O.set_pdl(True) is False          # returns the setting it replaces
        assert O.set_pdl(True) is True
        import ctypes
        assert O.lib().orion_set_pdl(2, None) == -1   # ORION_E_INVALID
    finally:
        O.set_pdl(prev)


def test_ctypes_structs_match_the_header_layout(tmp_path):
    # the binding's ctypes mirrors (orion.py) against the C compiler's layout of include/orion.h
    import ctypes
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    structs = {"orion_args": O.Args, "orion_tuner_cfg": O.TunerCfg, "orion_step_report": O.StepReport,
               "orion_device_limits": O.DeviceLimits, "orion_kernel_resources": O.KernelResources,
               "orion_level": O.Level}
    src = ["#include <stdio.h>", "#include <stddef.h>", '#include "orion.h"', "int main(void) {"]
    for cname, cls in structs.items():
        src.append(f'printf("{cname} %zu\\n", sizeof({cname}));')
        for f in cls._fields_:
            src.append(f'printf("{cname}.{f[0]} %zu\\n", offsetof({cname}, {f[0]}));')
    src += ["return 0; }"]
    c = tmp_path / "layout.c"
    c.write_text("\n".join(src))
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-I", os.path.join(root, "include"), str(c), "-o", str(exe)], check=True)
    got = dict(l.rsplit(" ", 1) for l in subprocess.run([str(exe)], capture_output=True, text=True,
                                                         check=True).stdout.split("\n") if l)
    for cname, cls in structs.items():
        assert int(got[cname]) == ctypes.sizeof(cls), cname
        for f in cls._fields_:
            assert int(got[f"{cname}.{f[0]}"]) == getattr(cls, f[0]).offset, (cname, f[0])
    assert O.ARGS_INDEPENDENT == 1
