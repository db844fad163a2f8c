"""Pins for the CPU oracle (SS4).  CPU only.

The oracle is the plain definition of Eq.1-2.  It is
trusted because it reproduces things that the paper and mathematics fix
independently of it:

* hand cases with closed-form values (tests/golden/hand_cases.json);
* closed forms: coincident sources (V = sum W), h -> inf (V -> sum W),
  h -> 0 (K = I), exact cancellation;
* invariants: symmetry of K, the adjoint identity, scaling, translation,
  sign flips / axis permutations, source permutation, linearity in W,
  column independence, target-subset sampling, thread-count independence;
* a separable closed form at the headline shape (M = 65,536, K = 32);
* an independent FP64 formulation of Alg.1 (norms + GEMM + exp + GEMV).

Each catches a plausible oracle bug: a wrong denominator (h^2 vs 2h^2 vs
(2h)^2) fails the hand cases; a dropped/duplicated source fails the closed
forms; an index swap (alpha/beta, i/j) fails symmetry/adjoint/separable;
a wrong sign fails cancellation and h -> 0.
"""
import json
import math
import os

import numpy as np
import pytest

import workloads
from tests.parity import e_norm

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hand_cases.json")


def ev(oracle_mod, a, W, b, h, **kw):
    return oracle_mod.oracle_eval(np.asarray(a, np.float32), np.asarray(W, np.float32),
                                  np.asarray(b, np.float32), h, **kw)


# ---------------------------------------------------------------- hand cases
def test_hand_cases(oracle_mod):
    gold = json.load(open(GOLD))
    for c in gold["cases"]:
        V = ev(oracle_mod, c["alpha"], c["W"], c["beta"], c["h"])
        exp = np.array(c["expected"], dtype=np.float64)
        if c.get("exact"):
            assert np.array_equal(V, exp), c["name"]
        else:
            np.testing.assert_allclose(V, exp, rtol=1e-15, atol=1e-16, err_msg=c["name"])


def test_hand_case_literals(oracle_mod):
    # the printed constants, independent of math.exp (SURVEY SS8(c) pin table)
    V = ev(oracle_mod, [[0.0, 0.0]], [[1.0]], [[3.0, 4.0]], 5.0)
    assert abs(V[0, 0] - 0.6065306597126334) < 1e-16
    V = ev(oracle_mod, [[1, 0, 0], [0, 1, 0], [0, 0, 1]], [[1.0], [2.0], [3.0]], [[0, 0, 0]], 1.0)
    assert abs(V[0, 0] - 3.6391839582758005) < 4e-16


# ---------------------------------------------------------------- closed forms
def test_self_interaction_is_one(oracle_mod):
    """exp(0) = 1 (Q14): beta == alpha, one-hot W = e_j -> V_j = 1 exactly."""
    a = workloads.uniform_points(64, 5, 7)
    for j in (0, 17, 63):
        W = np.zeros((64, 1), np.float32)
        W[j] = 1.0
        V = ev(oracle_mod, a, W, a, 0.3)
        assert V[j, 0] == 1.0
        # and V_t = K(alpha_j, alpha_t) = K(alpha_t, alpha_j): one row of the kernel matrix
        assert np.all(V[:, 0] <= 1.0) and np.all(V[:, 0] > 0.0)


def test_coincident_sources_sum(oracle_mod):
    """All sources equal the target: every K = 1, V = sum_i W_i, bitwise equal
    to a plain ascending FP64 sum."""
    b = workloads.uniform_points(3, 6, 11)
    a = np.repeat(b[1:2], 500, axis=0)
    W = workloads.weights(500, 2, "signed", 12)
    V = ev(oracle_mod, a, W, b[1:2], 0.7)
    for r in range(2):
        s = 0.0
        for i in range(500):
            s += float(W[i, r])
        assert V[0, r] == s


def test_h_to_infinity(oracle_mod):
    a, W, b, _ = workloads.custom(300, 20, 4, 1, 1.0, wkind="signed", seed=3)
    V = ev(oracle_mod, a, W, b, 1e8)
    sw = float(np.abs(W).sum())
    assert np.max(np.abs(V[:, 0] - W[:, 0].astype(np.float64).sum())) / sw <= 1e-15


def test_h_to_zero_identity(oracle_mod):
    """beta == alpha, distinct points on a 2^-6 grid, h = 1e-4: K = I -> V = W bitwise."""
    g = workloads.rng(5)
    pts = np.unique(g.integers(0, 64, size=(200, 3)), axis=0)[:150]
    a = (pts / 64.0).astype(np.float32)
    W = workloads.weights(a.shape[0], 1, "signed", 6)
    V = ev(oracle_mod, a, W, a, 1e-4)
    assert np.array_equal(V[:, 0], W[:, 0].astype(np.float64))


def test_cancellation_exact(oracle_mod):
    V = ev(oracle_mod, [[1.0, 2.0], [-1.0, 2.0]], [[1.0], [-1.0]], [[0.0, 2.0]], 0.9)
    assert V[0, 0] == 0.0


def test_empty_sources_and_targets(oracle_mod):
    V = oracle_mod.oracle_eval(np.zeros((0, 3), np.float32), np.zeros((0, 2), np.float32),
                               workloads.uniform_points(5, 3, 1), 1.0)
    assert V.shape == (5, 2) and np.all(V == 0.0)
    V = oracle_mod.oracle_eval(workloads.uniform_points(5, 3, 1), np.ones((5, 1), np.float32),
                               np.zeros((0, 3), np.float32), 1.0)
    assert V.shape == (0, 1)


# ---------------------------------------------------------------- invariants
def test_symmetry_bitwise(oracle_mod):
    """K(alpha_i, beta_j) = K(beta_j, alpha_i): one-hot weights both ways, bitwise."""
    a = workloads.uniform_points(40, 7, 21)
    b = workloads.uniform_points(30, 7, 22)
    for i, j in ((0, 0), (39, 29), (13, 5)):
        Wa = np.zeros((40, 1), np.float32); Wa[i] = 1
        Wb = np.zeros((30, 1), np.float32); Wb[j] = 1
        v_ab = ev(oracle_mod, a, Wa, b, 0.8)[j, 0]
        v_ba = ev(oracle_mod, b, Wb, a, 0.8)[i, 0]
        assert v_ab == v_ba and v_ab > 0


def test_adjoint_identity(oracle_mod):
    """sum_j U_j V(alpha->beta; W)_j = sum_i W_i V(beta->alpha; U)_i."""
    a, W, b, _ = workloads.custom(200, 150, 6, 1, 0.6, wkind="signed", seed=31)
    U = workloads.weights(150, 1, "signed", 99)
    lhs = float((U[:, 0].astype(np.float64) * ev(oracle_mod, a, W, b, 0.6)[:, 0]).sum())
    rhs = float((W[:, 0].astype(np.float64) * ev(oracle_mod, b, U, a, 0.6)[:, 0]).sum())
    assert abs(lhs - rhs) <= 1e-12 * max(abs(lhs), 1e-300) + 1e-15


def test_scaling_bitwise(oracle_mod):
    """Points x4 and h x4: every difference and the denominator scale by powers
    of two, so V is bitwise unchanged."""
    a, W, b, h = workloads.custom(100, 50, 5, 2, 0.45, seed=41)
    V1 = ev(oracle_mod, a, W, b, float(h))
    V2 = ev(oracle_mod, a * 4, W, b * 4, float(h) * 4)
    assert np.array_equal(V1, V2)


def test_translation_bitwise(oracle_mod):
    g = workloads.rng(51)
    a = (g.integers(-512, 512, size=(80, 4)) / 1024.0).astype(np.float32)
    b = (g.integers(-512, 512, size=(60, 4)) / 1024.0).astype(np.float32)
    W = workloads.weights(80, 1, "signed", 52)
    shift = (g.integers(-64, 64, size=4) / 16.0).astype(np.float32)
    V1 = ev(oracle_mod, a, W, b, 0.3)
    V2 = ev(oracle_mod, a + shift, W, b + shift, 0.3)
    assert np.array_equal(V1, V2)


def test_rotations(oracle_mod):
    a, W, b, _ = workloads.custom(90, 40, 6, 1, 0.5, seed=61)
    V = ev(oracle_mod, a, W, b, 0.5)
    flip = np.array([1, -1, 1, -1, -1, 1], np.float32)
    assert np.array_equal(V, ev(oracle_mod, a * flip, W, b * flip, 0.5))   # sign flips: bitwise
    perm = np.array([3, 0, 5, 1, 4, 2])
    Vp = ev(oracle_mod, a[:, perm], W, b[:, perm], 0.5)                    # axis permutation
    np.testing.assert_allclose(Vp, V, rtol=1e-14, atol=0)


def test_source_permutation(oracle_mod):
    a, W, b, _ = workloads.custom(300, 30, 4, 3, 0.5, seed=71)
    p = workloads.rng(72).permutation(300)
    V = ev(oracle_mod, a, W, b, 0.5)
    Vp = ev(oracle_mod, a[p], W[p], b, 0.5)
    np.testing.assert_allclose(Vp, V, rtol=1e-13, atol=1e-300)


def test_linearity_and_columns(oracle_mod):
    a, W, b, _ = workloads.custom(120, 35, 5, 3, 0.7, wkind="signed", seed=81)
    V = ev(oracle_mod, a, W, b, 0.7)
    for r in range(3):
        assert np.array_equal(ev(oracle_mod, a, W[:, r:r + 1], b, 0.7)[:, 0], V[:, r])
    Wc = (2.0 * W[:, 0:1] - 0.5 * W[:, 1:2]).astype(np.float32)
    Vc = ev(oracle_mod, a, Wc, b, 0.7)[:, 0]
    ref = 2.0 * V[:, 0] - 0.5 * V[:, 1]
    S = ev(oracle_mod, a, np.abs(W), b, 0.7)
    assert np.max(np.abs(Vc - ref) / (2 * S[:, 0] + 0.5 * S[:, 1])) < 1e-7  # Wc rounded to FP32


def test_sampling_bitwise(oracle_mod):
    a, W, b, _ = workloads.custom(200, 100, 3, 2, 0.4, seed=91)
    V = ev(oracle_mod, a, W, b, 0.4)
    J = np.array([0, 5, 99, 42, 42], np.int64)
    assert np.array_equal(ev(oracle_mod, a, W, b, 0.4, J=J), V[J])


def test_thread_count_independent(oracle_mod):
    a, W, b, _ = workloads.custom(500, 300, 8, 1, 0.5, seed=101)
    n = oracle_mod.num_threads()
    try:
        oracle_mod.set_num_threads(1)
        V1 = ev(oracle_mod, a, W, b, 0.5)
        oracle_mod.set_num_threads(max(n, 4))
        V4 = ev(oracle_mod, a, W, b, 0.5)
    finally:
        oracle_mod.set_num_threads(n)
    assert np.array_equal(V1, V4)


# ---------------------------------------------------------------- separable closed form
def separable_closed_form(g, c, w, beta, h):
    """V_j = prod_{d<G} [sum_b w[d,b] exp(-(g[d,b]-beta_jd)^2/2h^2)] * exp(-sum_{d>=G}(c_d-beta_jd)^2/2h^2)."""
    G = g.shape[0]
    bt = beta.astype(np.float64)
    den = 2.0 * h * h
    out = np.ones(beta.shape[0])
    for d in range(G):
        s = np.zeros(beta.shape[0])
        for bb in range(2):
            s += float(w[d, bb]) * np.exp(-(float(g[d, bb]) - bt[:, d]) ** 2 / den)
        out *= s
    rest = ((c.astype(np.float64)[None, :] - bt[:, G:]) ** 2).sum(axis=1)
    return out * np.exp(-rest / den)


def test_separable_headline_shape(oracle_mod):
    """M = 2^16 = 65,536 sources at K = 32 (the headline shape), closed form O(NK)."""
    a, W, g, c, w, _ = workloads.separable_grid(32, 16, seed=111)
    assert a.shape == (65536, 32)
    b = (workloads.uniform_points(24, 32, 112) * 0.5 + 0.25).astype(np.float32)
    h = 0.5
    V, S = oracle_mod.oracle_eval(a, W, b, h, want_S=True)
    ref = separable_closed_form(g, c, w, b, h)
    assert np.all(ref > 0)
    np.testing.assert_allclose(V[:, 0], ref, rtol=1e-11, atol=0)


# ---------------------------------------------------------------- Alg.1 cross-check
def alg1_fp64(a, W, b, h):
    """Alg.1 in FP64: norms, GEMM, R = sqA + sqB - 2C, exp, GEMV.
    Independent of the oracle's direct-difference loop."""
    A = a.astype(np.float64)
    B = b.astype(np.float64)
    va = (A * A).sum(1)
    vb = (B * B).sum(1)
    C = A @ B.T                                   # [M, N]
    Rm = va[:, None] + vb[None, :] - 2.0 * C
    Km = np.exp(-Rm / (2.0 * h * h))
    return Km.T @ W.astype(np.float64)           # V = K^T W  (W on sources, Q2)


@pytest.mark.parametrize("cfg", [1, 2, 3, 5])
def test_alg1_crosscheck(oracle_mod, cfg):
    a, W, b, h = workloads.make(cfg, M=700, N=300, wkind="signed")
    V = ev(oracle_mod, a, W, b, float(h))
    V1 = alg1_fp64(a, W, b, float(h))
    S = ev(oracle_mod, a, np.abs(W), b, float(h))
    assert np.max(np.abs(V - V1) / S) < 1e-12


# ---------------------------------------------------------------- harness self-test
def test_metric_catches_injected_bugs(oracle_mod):
    """The parity metric must FAIL for the bugs a kernel could plausibly have
    (SS4): dropping the last 128-source tile, h off by 1%, 2h^2 -> h^2, a NaN or inf
    output (found by the GPU-side self-test, tests/test_gpu_harness.py: max() skipped NaNs).
    W >= 0 on the cfg3 distribution (the signed-W metric is lenient)."""
    a, W, b, h = workloads.make(3, M=4096, N=128, wkind="pos")
    h = float(h)
    V = ev(oracle_mod, a, W, b, h)
    bugs = {
        "drop_last_tile": ev(oracle_mod, a[:-128], W[:-128], b, h),
        "h_x1.01": ev(oracle_mod, a, W, b, h * 1.01),
        "2h2_to_h2": ev(oracle_mod, a, W, b, h / math.sqrt(2.0)),
    }
    Vn = V.copy()
    Vn[7, 0] = np.nan  # one non-finite output (a kernel reading garbage) -- max() alone skips a NaN
    bugs["one_nan"] = Vn
    Vi = V.copy()
    Vi[0, 0] = np.inf
    bugs["one_inf"] = Vi
    for name, Vb in bugs.items():
        assert e_norm(Vb, V, W) > 1e-5, name
    assert e_norm(V.astype(np.float32), V, W) < 1e-7
