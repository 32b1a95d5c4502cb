"""Mutation checks of the oracle's pins ("a deliberately wrong coefficient fails a CPU pin").

Each case rebuilds liboracle from a copy of oracle/*.c with ONE plausible mistake (a dropped term,
a wrong constant, a swapped operand or index) and runs that oracle part's pin module against the
mutant (ORACLE_LIB_OVERRIDE) in a subprocess: the module must FAIL.  The unmodified oracle passes
the same modules in the normal suite.
"""
import os
import subprocess
import sys

import pytest

import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# (file, exact original text, mutated text, pin module, what the mistake is)
MUTATIONS = [
    # O5 SRAD: the diffusion coefficient
    ("srad.c", "(1.0 / 16.0) * (L * L)", "(1.0 / 8.0) * (L * L)", "test_oracle_srad.py",
     "srad: wrong 1/16 in q^2"),
    ("srad.c", "double den = 1.0 + 0.25 * L;", "double den = 1.0 + 0.5 * L;", "test_oracle_srad.py",
     "srad: wrong 1 + L/4"),
    ("srad.c", "den = (qsqr - q0sqr) / (q0sqr * (1.0 + q0sqr));",
     "den = (q0sqr - qsqr) / (q0sqr * (1.0 + q0sqr));", "test_oracle_srad.py", "srad: swapped q^2 - q0^2"),
    ("srad.c", "den = (qsqr - q0sqr) / (q0sqr * (1.0 + q0sqr));",
     "den = (qsqr - q0sqr) / (q0sqr);", "test_oracle_srad.py", "srad: dropped (1 + q0^2)"),
    ("srad.c", "double cW = cN, cE = C[(size_t)i * W + jE];", "double cW = cN, cE = cN;",
     "test_oracle_srad.py", "srad: east flux with the cell's own c"),
    ("srad.c", "double G2 = (dN * dN + dS * dS + dW * dW + dE * dE) / (Jc * Jc);",
     "double G2 = (dN * dN + dS * dS + dW * dW + dE * dE) / Jc;", "test_oracle_srad.py",
     "srad: G2 not normalised by J^2"),
    ("srad.c", "double var = sum2 / size - mean * mean;", "double var = sum2 / size;",
     "test_oracle_srad.py", "srad: ROI variance without the mean term"),
    # O2 denoise
    ("denoise.c", "(double)(i * i + j * j) / (double)A", "(double)(i * i + j * j) / (double)(2 * R + 1)",
     "test_oracle_denoise.py", "denoise: spatial term over the diameter, not A"),
    ("denoise.c", "sample(img, W, H, row0, x + m, y + n, b);", "sample(img, W, H, row0, x + n, y + m, b);",
     "test_oracle_denoise.py", "denoise: transposed centre patch index"),
    ("denoise.c", "out[c] = clr[c] + (c00[c] - clr[c]) * q;", "out[c] = c00[c] + (clr[c] - c00[c]) * q;",
     "test_oracle_denoise.py", "denoise: lerp toward the mean instead of the centre"),
    ("denoise.c", "int above = w > p->wthr;", "int above = w >= 2.0 * p->wthr;", "test_oracle_denoise.py",
     "denoise: wrong weight threshold"),
    ("denoise.c", "return dx * dx + dy * dy + dz * dz;", "return dx * dx + dy * dy;", "test_oracle_denoise.py",
     "denoise: dropped blue channel from the distance"),
    # O3 hotspot
    ("stencil.c", "(P + (S + N - 2.0 * T) * p->ry", "(P + (S + N - T) * p->ry", "test_oracle_stencil.py",
     "hotspot f64: dropped factor 2 of the centre term"),
    ("stencil.c", "b[(size_t)y * W + x] = T + p->sdc * (P", "b[(size_t)y * W + x] = T + p->sdc * (2.0 * P",
     "test_oracle_stencil.py", "hotspot f64: doubled power term"),
    ("stencil.c", "+ (p->amb - T) * p->rz);", "+ (T - p->amb) * p->rz);", "test_oracle_stencil.py",
     "hotspot f64: sink sign"),
    ("stencil.c", "float Wv = a[(size_t)y * W + clampi(x - 1, 0, W - 1)];",
     "float Wv = a[(size_t)y * W + clampi(x - 2, 0, W - 1)];", "test_oracle_stencil.py",
     "hotspot f32: wrong west index"),
]


def _build_mutant(tmp_path, fname, old, new):
    srcs = []
    for s in oracle._SOURCES:
        text = open(s).read()
        if os.path.basename(s) == fname:
            assert text.count(old) == 1, (fname, old)
            text = text.replace(old, new)
        dst = tmp_path / os.path.basename(s)
        dst.write_text(text)
        srcs.append(str(dst))
    lib = tmp_path / "liboracle_mutant.so"
    subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fPIC", "-shared",
                           "-o", str(lib), *srcs, "-lm"])
    return str(lib)


@pytest.mark.parametrize("fname,old,new,module,why", MUTATIONS, ids=[m[4] for m in MUTATIONS])
def test_mutation_is_caught_by_pins(tmp_path, fname, old, new, module, why):
    lib = _build_mutant(tmp_path, fname, old, new)
    env = dict(os.environ, ORACLE_LIB_OVERRIDE=lib)
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", module)], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 1, f"the pins in {module} do not catch: {why}\n{r.stdout[-2000:]}"
