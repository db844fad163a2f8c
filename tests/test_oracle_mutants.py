"""Mutation self-test of the oracle pins (CPU only).

Each mutant is oracle.c with one plausible mistake (a dropped term, a wrong
sign or index, a transposed operand, a wrong bandwidth form).  The pin suite
in test_oracle_pins.py must reject every one of them: at least one pin fails.
"""
import os
import subprocess
import tempfile

import pytest

import oracle
from tests import test_oracle_pins as pins

SRC = os.path.join(os.path.dirname(oracle.__file__), "oracle.c")

MUTANTS = {
    # Q1 bandwidth forms
    "den_h2": ("const double den = 2.0 * h * h;", "const double den = h * h;"),
    "den_2h_sq": ("const double den = 2.0 * h * h;", "const double den = 4.0 * h * h;"),
    "den_2h": ("const double den = 2.0 * h * h;", "const double den = 2.0 * h;"),
    # sign of the exponent
    "exp_sign": ("exp(-d2 / den)", "exp(d2 / den)"),
    # norm instead of squared norm
    "sqrt_d2": ("exp(-d2 / den)", "exp(-sqrt(d2) / den)"),
    # dropped last source / first source
    "drop_last_source": ("for (int64_t i = 0; i < M; ++i)", "for (int64_t i = 0; i < M - 1; ++i)"),
    "drop_first_source": ("for (int64_t i = 0; i < M; ++i)", "for (int64_t i = 1; i < M; ++i)"),
    # dropped last coordinate
    "drop_last_dim": ("for (int d = 0; d < K; ++d)", "for (int d = 0; d < K - 1; ++d)"),
    # difference replaced by sum
    "sum_not_diff": ("(double)b[d] - (double)a[d]", "(double)b[d] + (double)a[d]"),
    # weight indexed by the target instead of the source (Q2/Q5)
    "W_by_target": ("const float *w = W + i * (int64_t)R;", "const float *w = W + (j % M) * (int64_t)R;"),
    # weight column index fixed at 0
    "W_col0": ("v[r] += k * (double)w[r];", "v[r] += k * (double)w[0];"),
    # |W| instead of W
    "abs_W": ("v[r] += k * (double)w[r];", "v[r] += k * fabs((double)w[r]);"),
    # target subset ignored
    "J_ignored": ("const int64_t j = J ? J[t] : t;", "const int64_t j = t;"),
    # self term dropped (Q14)
    "no_self": ("const double k = exp(-d2 / den); /* Eq.1 */",
                "const double k = (d2 == 0.0) ? 0.0 : exp(-d2 / den);"),
    # kernel truncated (a cutoff the paper does not have)
    "cutoff": ("const double k = exp(-d2 / den); /* Eq.1 */",
               "const double k = (d2 > den) ? 0.0 : exp(-d2 / den);"),
    # single-precision exponent
    "float_exp": ("const double k = exp(-d2 / den); /* Eq.1 */",
                  "const double k = (double)expf((float)(-d2 / den));"),
}

PIN_TESTS = [
    pins.test_hand_cases, pins.test_hand_case_literals, pins.test_self_interaction_is_one,
    pins.test_coincident_sources_sum, pins.test_h_to_infinity, pins.test_h_to_zero_identity,
    pins.test_cancellation_exact, pins.test_symmetry_bitwise, pins.test_adjoint_identity,
    pins.test_scaling_bitwise, pins.test_translation_bitwise, pins.test_rotations,
    pins.test_source_permutation, pins.test_linearity_and_columns, pins.test_sampling_bitwise,
    pins.test_separable_headline_shape,
]


@pytest.mark.parametrize("name", sorted(MUTANTS))
def test_pins_reject_mutant(name, tmp_path):
    old, new = MUTANTS[name]
    src = open(SRC).read()
    assert src.count(old) >= 1, f"mutation anchor missing: {old!r}"
    msrc = tmp_path / "mut.c"
    msrc.write_text(src.replace(old, new))
    lib = tmp_path / "libmut.so"
    subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
                           "-fPIC", "-shared", "-std=c11", str(msrc), "-o", str(lib), "-lm"])
    mod = oracle.Variant(str(lib))
    failed = []
    for t in PIN_TESTS:
        try:
            t(mod)
        except (AssertionError, ValueError):
            failed.append(t.__name__)
    assert failed, f"mutant {name} passed every pin"
