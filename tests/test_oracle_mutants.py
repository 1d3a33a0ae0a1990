"""Mutation test of the oracle pins (CPU).

Each mutant is oracle/oracle.c with one plausible mistake (a dropped term, a
wrong sign, a transposed or shifted index, a skipped k, float accumulation, a
wrong |A||B|).  It is compiled to a temporary liboracle.so and the pin suite
(tests/test_oracle_pins.py) is run against it in a subprocess (ORACLE_LIB);
every mutant must make at least one pin fail (or crash).  The unmutated
source must pass.
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = open(os.path.join(ROOT, "oracle", "oracle.c")).read()

MUTANTS = {
    "dropped_first_term": ("acc[j] += a * b[j];", "acc[j] += (k ? a * b[j] : 0.0);"),
    "sign_flip": ("acc[j] += a * b[j];", "acc[j] -= a * b[j];"),
    "transposed_A_index": ("((const double *)A)[i * K + k]", "((const double *)A)[k * M_ + i]"),
    "shifted_B_row": ("const double *b = (const double *)B + k * N;",
                      "const double *b = (const double *)B + (k + (k + 1 < K)) * N;"),
    "skipped_last_k": ("for (int64_t k = 0; k < K; ++k) {", "for (int64_t k = 0; k + 1 < K; ++k) {"),
    "float_accumulation_f32": ("acc[j] += a * bj;", "acc[j] = (float)(acc[j] + a * bj);"),
    "signed_mag": ("mag[j] += aa * fabs(b[j]);", "mag[j] += aa * b[j];"),
    "mag_not_abs_a": ("double aa = fabs(a);", "double aa = a;"),
    "no_zero_init": ("for (int64_t j = 0; j < N; ++j) { acc[j] = 0.0; mag[j] = 0.0; }",
                     "for (int64_t j = 0; j < N; ++j) { mag[j] = 0.0; }"),
}

PIN_SUBSET = "p1 or p2 or p3 or p4 or p5 or p6 or p8 or float32 or rows_subset"


def _build(src, out):
    c = os.path.join(os.path.dirname(out), "oracle_mut.c")
    with open(c, "w") as f:
        f.write(src)
    subprocess.check_call(["gcc", "-O1", "-fopenmp", "-ffp-contract=off", "-shared", "-fPIC", "-o", out, c, "-lm"])


def _run_pins(lib):
    env = dict(os.environ, ORACLE_LIB=lib, OMP_NUM_THREADS="2")
    r = subprocess.run([sys.executable, "-m", "pytest", os.path.join(ROOT, "tests", "test_oracle_pins.py"), "-x",
                        "-q", "-k", PIN_SUBSET, "-p", "no:cacheprovider"], capture_output=True, text=True, env=env,
                       timeout=600, cwd=ROOT)
    return r.returncode, r.stdout[-800:]


def test_unmutated_passes(tmp_path):
    src = SRC.replace("static void one_row(", "#define M_ 0\nstatic void one_row(", 1)
    lib = str(tmp_path / "liboracle_ok.so")
    _build(src, lib)
    rc, out = _run_pins(lib)
    assert rc == 0, out


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_mutant_is_killed(name, tmp_path):
    old, new = MUTANTS[name]
    assert old in SRC, f"mutation anchor for {name} not found"
    src = SRC.replace(old, new, 1)
    if "M_" in new:
        # give the transposed index a row count to (wrongly) use
        src = src.replace("static void one_row(int dtype, const void *A, const void *B, int64_t i,\n"
                          "                    int64_t N, int64_t K, double *acc, double *mag)",
                          "static int64_t M_ = 1;\nstatic void one_row(int dtype, const void *A, const void *B, "
                          "int64_t i,\n                    int64_t N, int64_t K, double *acc, double *mag)", 1)
        src = src.replace("    if (nrows == 0 || N == 0) return 0;", "    if (nrows == 0 || N == 0) return 0;\n    M_ = M;", 1)
    lib = str(tmp_path / f"liboracle_{name}.so")
    _build(src, lib)
    rc, out = _run_pins(lib)
    assert rc != 0, f"mutant {name} survived the pins:\n{out}"
