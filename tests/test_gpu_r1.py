"""GPU parity of the dedicated R = 1 kernel (ks_fused_r1.cu; the AUTO path for one weight
column at K <= 58) against the FP64 oracle, bar e_norm <= 1e-5 (BASELINE.json north_star,
DESIGN.md SS4), and its d^2 >= 0 behaviour on coincident points (Q8).

The kernel computes t = sum_d bh_jd a_id + na_i + nb_j in one tcgen05 accumulator (the norms
ride in six FP16 K columns, reading Q26, with the fold shift of reading Q28) and then, per
KS_OPT_R1_EPILOGUE: 0 log-weights (W >= 0, V = Wmax sum 2^t; any W_i < 0 falls back to 1),
1 weights with the clamp t <= 0, 2 weights with t -> -|t|, 3 weights without a clamp.
"""
import numpy as np
import pytest

import workloads
from tests.parity import TOL_3XTF32, e_norm

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402


def run(alpha, W, beta, h, **opts):
    W = np.asarray(W, np.float32)
    if W.ndim == 1:
        W = W[:, None]
    with ks.KernelSum(alpha.shape[1], float(h), "auto", options=opts) as plan:
        plan.set_sources(torch.from_numpy(np.ascontiguousarray(alpha)).cuda(),
                         torch.from_numpy(np.ascontiguousarray(W)).cuda())
        V = plan.eval(torch.from_numpy(np.ascontiguousarray(beta)).cuda())
        torch.cuda.synchronize()
        info = plan.info()
    # the dedicated kernel runs 128-source units
    r1 = opts.get("r1_kernel", 1) and alpha.shape[1] + 6 <= 64
    assert info["path"] == ks.KS_PATH_TC and info["tile_s"] == (128 if r1 else 256)
    return V.cpu().numpy().astype(np.float64)


def check(oracle_mod, a, W, b, h, tol=TOL_3XTF32, **opts):
    V = run(a, W, b, h, **opts)
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    err = e_norm(V, Vr, W)
    assert err <= tol, f"e_norm {err:.3e} > {tol:.0e} ({opts})"
    return V, Vr


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
@pytest.mark.parametrize("wkind", ["pos", "signed"])
def test_epilogue_modes(oracle_mod, mode, wkind):
    a, W, b, h = workloads.make(3, M=3000, N=1000, wkind=wkind)
    check(oracle_mod, a, W, b, h, r1_epilogue=mode)


@pytest.mark.parametrize("npoly", [0, 4, 5, 6, 7, 8])
def test_fma_pipe_exponential_shares(oracle_mod, npoly):
    """NPOLY of every 16 exponential pairs on the FMA pipe (degree-5 polynomial, reading
    Q25), the rest on MUFU.EX2: every share meets the bar."""
    a, W, b, h = workloads.make(3, M=2600, N=700, wkind="pos")
    check(oracle_mod, a, W, b, h, exp_poly=npoly)


@pytest.mark.parametrize("K", [1, 2, 7, 10, 16, 26, 27, 31, 32, 33, 40, 50, 58])
def test_operand_layouts(oracle_mod, K):
    """K + 6 <= 32: one 64-byte operand chunk (hi + lo planes); else two, the second with
    (K > 32) or without (K <= 32) a lo plane; the norm columns start at K."""
    a, W, b, h = workloads.custom(1500 + 3 * K, 700, K, 1, 0.3 * np.sqrt(K) + 0.1, dist="gm", sigma=0.07,
                                  wkind="pos", seed=500 + K)
    check(oracle_mod, a, W, b, h)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("wcase", ["zeros", "all_zero", "one_negative", "tiny", "huge", "one_hot"])
def test_weight_cases(oracle_mod, mode, wcase):
    a, W, b, h = workloads.make(3, M=3000, N=700, wkind="pos")
    W = W.copy()
    if wcase == "zeros":
        W[::3] = 0.0
    elif wcase == "all_zero":
        W[:] = 0.0
    elif wcase == "one_negative":
        W[17] = -0.5
    elif wcase == "tiny":
        W *= np.float32(1e-30)
    elif wcase == "huge":
        W *= np.float32(1e30)
    elif wcase == "one_hot":
        W[:] = 0.0
        W[1234] = 1.0
    V = run(a, W, b, h, r1_epilogue=mode)
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    if wcase == "all_zero":
        assert np.all(V == 0.0)
        return
    assert e_norm(V, Vr, W) <= TOL_3XTF32


@pytest.mark.parametrize("h", [0.004, 0.01, 0.03])
def test_fold_shift_wide_spread(oracle_mod, h):
    """c K amax^2 beyond 2^12 (h down to 0.004 on the unit cube at K = 8: the fold shift s
    grows to 6): the norm pieces are stored as n 2^-s against unit columns 2^s (reading Q28)
    and the layout stays valid; coincident points keep their self term."""
    a, W, b, _ = workloads.custom(2000, 700, 8, 1, h, wkind="pos", seed=61, same_points=True)
    check(oracle_mod, a, W, b, np.float32(h))


def test_far_targets_are_zero(oracle_mod):
    a, W, b, h = workloads.make(3, M=2000, N=600, wkind="pos")
    b = b.copy()
    b[::7] += np.float32(40.0)
    V, _ = check(oracle_mod, a, W, b, h)
    assert np.all(np.abs(V[::7]) <= 2.0**-120 * np.abs(W).sum())


@pytest.mark.parametrize("M,N", [(1, 1), (1, 300), (300, 1), (128, 128), (129, 127), (40000, 90), (100, 70000)])
def test_edge_sizes_and_splits(oracle_mod, M, N):
    """Single points, exact and ragged tiles; N <= 128 with M = 40,000 (every CTA splits the
    one target tile: ~148 stream-K partial slots); M = 100 with 547 target tiles (several
    waves and a remainder)."""
    a, W, b, h = workloads.custom(M, N, 32, 1, 1.0, dist="gm", sigma=0.1, wkind="pos", seed=M + N)
    check(oracle_mod, a, W, b, h)


def test_matches_general_kernel(oracle_mod):
    a, W, b, h = workloads.make(3, M=5000, N=1300, wkind="pos")
    V1, Vr = check(oracle_mod, a, W, b, h)
    V0 = run(a, W, b, h, r1_kernel=0)
    assert np.max(np.abs(V1 - V0)) / np.abs(W).sum() <= 2 * TOL_3XTF32


def test_deterministic_bitwise():
    a, W, b, h = workloads.make(3, M=6000, N=2000, wkind="pos")
    assert np.array_equal(run(a, W, b, h), run(a, W, b, h))


def _lattice(K, n, scale, seed):
    """n distinct points of the lattice {0, 1, 2, 3}^K scaled by `scale`."""
    g = np.random.default_rng(seed)
    pts = g.permutation(np.arange(4 ** K))[:n]
    x = np.zeros((n, K), np.float64)
    for d in range(K):
        x[:, d] = (pts // 4 ** d) % 4
    return (x * scale).astype(np.float32)


@pytest.mark.parametrize("f", [4.0, 40.0])
def test_coincident_points_overshoot_bound(oracle_mod, f):
    """beta == alpha on a lattice of spacing f h (K = 6, W = 1): V_j = 1 + sum of neighbour
    terms (exp(-f^2/2) each).  Mode 0 has no d^2 >= 0 clamp (Q8): the diagonal term
    2^t differs from 1 by the rounding of t, which the Eq.3 cancellation bounds by
    ~2^-22 (c||alpha_hat||^2 + c||beta_hat||^2) (reading Q11) -- f = 40 puts
    c ||alpha_hat||^2 near 2^13, past the accuracy domain, where the test bounds the overshoot;
    f = 4 (c ||alpha_hat||^2 ~ 90) is inside it and meets the 1e-5 bar.  Modes 1 (clamp)
    and 2 (|d^2|) never exceed the exact value by more than the neighbour terms' rounding."""
    K, n, hk = 6, 1024, 0.5
    a = _lattice(K, n, f * hk, 7)
    h = np.float32(hk)
    c = np.log2(np.e) / (2.0 * float(h) ** 2)
    W = np.ones((n, 1), np.float32)
    nrm = c * ((a.astype(np.float64) - a.astype(np.float64).mean(axis=0)) ** 2).sum(axis=1)
    Vr = oracle_mod.oracle_eval(a, W, a, float(h))[:, 0]
    bound = np.log(2) * 2.0**-21 * (2.0 * nrm + 1.0)
    for mode in (0, 1, 2):
        V = run(a, W, a, h, r1_epilogue=mode)[:, 0]
        d = V - Vr
        assert np.all(np.abs(d) <= bound * Vr), (mode, float(np.max(np.abs(d) / (bound * Vr))))
        if mode in (1, 2):  # the diagonal term never exceeds exp(0) = 1
            assert np.all(d <= bound * (Vr - 1.0) + 2.0**-21), (mode, float(d.max()))
        if f == 4.0:
            assert np.max(np.abs(d)) / n <= TOL_3XTF32


def test_reserve_then_graph_capture():
    """ks_reserve(N_max) sizes every per-eval buffer, so an eval with N <= N_max can be
    captured in a CUDA graph and replayed (include/ks.h)."""
    a, W, b, h = workloads.make(3, M=3000, N=2000, wkind="pos")
    ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
    with ks.KernelSum(a.shape[1], float(h), "auto") as plan:
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            plan.set_sources(ta, tw)
            ks.ks_reserve(plan.ctx, 4096)
            V = torch.empty((b.shape[0], 1), device="cuda")
            plan.eval(tb, out=V)
            s.synchronize()
            ref = V.clone()
            V.zero_()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                plan.eval(tb, out=V)
            g.replay()
            s.synchronize()
        assert torch.equal(V, ref)


def test_options_api():
    with ks.KernelSum(32, 1.0) as plan:
        assert plan.get_option("r1_kernel") == 1 and plan.get_option("r1_epilogue") == 0
        plan.set_option("r1_epilogue", 2)
        assert plan.get_option("r1_epilogue") == 2
        with pytest.raises(ks.KsError):
            plan.set_option("r1_epilogue", 9)
        with pytest.raises(ks.KsError):
            ks.ks_set_option(plan.ctx, 99, 0)


@pytest.mark.parametrize("K", [6, 16, 100])
@pytest.mark.parametrize("opts", [{}, {"r1_kernel": 0}, {"r1_kernel": 0, "fold": 0}])
def test_large_magnitudes_stay_finite(oracle_mod, K, opts):
    """Coordinates up to 30 h (c K amax^2 ~ 10^4, beyond the 2^12 fold limit of the general
    kernel): the R = 1 kernel folds with the shift, the general kernel falls back to FP32 norms
    on the device.  Every path stays finite and within the Eq.3 FP32 cancellation bound of
    reading Q11, ~2^-22 c K amax^2 relative (regression: the general kernel's target prep
    dropped the target norm when the fold was requested but inactive -> NaN)."""
    g = np.random.default_rng(K)
    a = g.uniform(-15.0, 15.0, (600, K)).astype(np.float32)
    W = np.ones((600, 1), np.float32)
    h = np.float32(0.5)
    V = run(a, W, a, h, **opts)
    assert np.all(np.isfinite(V))
    Vr = oracle_mod.oracle_eval(a, W, a, float(h))
    cka2 = np.log2(np.e) / (2 * 0.25) * K * float(np.abs(a - a.mean(0)).max()) ** 2
    assert e_norm(V, Vr, W) <= 2.0**-18 * cka2 / 600 + 1e-7


def _run_any(alpha, W, beta, h, **opts):
    with ks.KernelSum(alpha.shape[1], float(h), "auto", options=opts) as plan:
        plan.set_sources(torch.from_numpy(np.ascontiguousarray(alpha)).cuda(),
                         torch.from_numpy(np.ascontiguousarray(W)).cuda())
        V = plan.eval(torch.from_numpy(np.ascontiguousarray(beta)).cuda())
        torch.cuda.synchronize()
        return V.cpu().numpy().astype(np.float64), plan.info()


@pytest.mark.parametrize("K", [1, 4, 10, 16, 26, 32, 58])
@pytest.mark.parametrize("M,R,wkind", [(1, 1, "pos"), (777, 1, "signed"), (70001, 1, "pos"), (5000, 3, "signed"),
                                       (3000, 1, "zero"), (150001, 1, "pos")])
def test_cooperative_source_prep(oracle_mod, K, M, R, wkind):
    """Source statistics + folded source prep in one cooperative launch (option coop_prep, the
    default for the R = 1 and multi-column kernels; a grid barrier between the partial and the
    final statistics) against the separate statistics and prep kernels: the same layout and
    scales, so V agrees to the rounding of mu's FP64 column sums (a different fixed order); the
    result meets the bar and is bitwise reproducible.  Covers one source, ragged counts, more
    rows than one block's share (70,001), blocks whose rows do not fit shared memory at once
    (150,001 at K >= 39: phase 1 in sub-chunks, phase 3 re-reads L2), R > 1 (multi-column kernel,
    no weight statistics), negative weights (the weight mode) and all-zero weights."""
    if wkind == "zero":
        a, W, b, h = workloads.custom(M, 300, K, R, 1.0, dist="gm", sigma=0.1, wkind="pos", seed=K + M)
        W = np.zeros_like(W)
    else:
        a, W, b, h = workloads.custom(M, 300, K, R, 1.0, dist="gm", sigma=0.1, wkind=wkind, seed=K + M)
    Vc, info = _run_any(a, W, b, h)
    assert info["launches"] >= 1
    Vs, _ = _run_any(a, W, b, h, coop_prep=0)
    Vc2, _ = _run_any(a, W, b, h)
    assert np.array_equal(Vc, Vc2)
    den = max(np.abs(W).sum(), 1e-30)
    assert np.max(np.abs(Vc - Vs)) / den <= 1e-6
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    if wkind == "zero":
        assert np.all(Vc == 0.0)
    else:
        assert e_norm(Vc, Vr, W) <= TOL_3XTF32


def test_cooperative_prep_graph_replay():
    """The cooperative source prep's grid barrier resets itself, so ks_set_sources can be
    captured in a CUDA graph and replayed any number of times, interleaved with live calls."""
    a, W, b, h = workloads.make(3, M=9000, N=1000, wkind="pos")
    a2 = a[::-1].copy()
    ta, ta2, tw, tb = (torch.from_numpy(x).cuda() for x in (a, a2, W, b))
    with ks.KernelSum(a.shape[1], float(h), "auto") as plan:
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            plan.set_sources(ta, tw)
            ref = plan.eval(tb).clone()
            plan.set_sources(ta2, tw)
            s.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                plan.set_sources(ta, tw)
            for _ in range(3):
                plan.set_sources(ta2, tw)
                g.replay()
                g.replay()
                V = plan.eval(tb)
                s.synchronize()
                assert torch.equal(V, ref)


@pytest.mark.parametrize("wkind", ["pos", "signed"])
@pytest.mark.parametrize("K", [10, 11, 13, 16, 17, 26, 27, 30, 32, 33, 42])
def test_narrow_planes(oracle_mod, K, wkind):
    """Operand planes with only 16 used columns load as 32-byte rows (SWIZZLE_32B TMA box over the
    same array, their own MMA descriptor layout) instead of 64-byte chunks: at 27 <= K <= 32 the
    second chunk (the six folded norm columns), at 11 <= K <= 16 the lo plane (coordinates in its
    first 16 columns only; the lo.hi / hi.lo MMAs then mix the two layouts).  The MMAs multiply
    the same values in the same order, so V is bitwise the 64-byte layout's (option
    narrow_planes = 0); the neighbouring K (10: 32-byte rows throughout; 17, 26: fold inside chunk
    0; 33, 42: coordinates in chunk 1) are unaffected."""
    a, W, b, h = workloads.custom(3000, 1500, K, 1, 1.0, dist="gm", sigma=0.1, wkind=wkind, seed=K)
    V1 = run(a, W, b, h)
    V0 = run(a, W, b, h, narrow_planes=0)
    assert np.array_equal(V1, V0)
    Vr = oracle_mod.oracle_eval(a, W, b, float(h))
    assert e_norm(V1, Vr, W) <= TOL_3XTF32
