"""GPU parity: the CUDA path (through the C ABI) against the FP64 oracle.

Acceptance (BASELINE.json north_star, SS4):
    e_norm = max_{j,r} |V_gpu - V_ref| / sum_i |W_i|  <= 1e-5  (FP32, 3xTF32)
Inputs come from workloads/ (seeded, the configs' distributions).  Sizes here
span several 128-tiles with ragged tails; the full BASELINE sizes are checked
on sampled targets (the oracle computes them one by one) in the launch
configuration bench.py times, and by a separable closed form at the headline
shape (M = N = 65,536, K = 32).
"""
import numpy as np
import pytest

import workloads
from tests.parity import TOL_FP32, e_norm, e_S

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

# Every test in this module runs on both K<=32 kernels: the FP32 FFMA2 kernel
# and the tcgen05 3xTF32 kernel (the AUTO choice for M > 4096).
_PREC = {"p": "fp32"}


@pytest.fixture(autouse=True, params=["fp32", "3xtf32", "3xf16"])
def precision(request):
    _PREC["p"] = request.param
    yield request.param


def gpu_eval(alpha, W, beta, h, precision=None, host=False, options=None):
    precision = precision or _PREC["p"]
    K = alpha.shape[1]
    W = np.asarray(W, np.float32)
    if W.ndim == 1:
        W = W[:, None]
    with ks.KernelSum(K, float(h), precision) as plan:
        for k, v in (options or {}).items():
            plan.set_option(k, v)
        if host:
            plan.set_sources_host(alpha, W)
            return plan.eval_host(beta).astype(np.float64)
        a = torch.from_numpy(np.ascontiguousarray(alpha)).cuda()
        w = torch.from_numpy(np.ascontiguousarray(W)).cuda()
        b = torch.from_numpy(np.ascontiguousarray(beta)).cuda()
        plan.set_sources(a, w)
        V = plan.eval(b)
        torch.cuda.synchronize()
        return V.cpu().numpy().astype(np.float64)


def check(oracle_mod, alpha, W, beta, h, tol=TOL_FP32, J=None, precision=None, V=None):
    if V is None:
        V = gpu_eval(alpha, W, beta, h, precision)
    Vg = V if J is None else V[J]
    Vr, S = oracle_mod.oracle_eval(alpha, W, beta, float(h), J=J, want_S=True)
    err = e_norm(Vg, Vr, W)
    assert err <= tol, f"e_norm {err:.3e} > {tol:.0e} (e_S {e_S(Vg, Vr, S):.3e})"
    return err


# ---------------------------------------------------------------- configs at reduced / sampled sizes
@pytest.mark.parametrize("wkind", ["pos", "signed"])
def test_cfg1_full(oracle_mod, wkind):
    a, W, b, h = workloads.make(1, wkind=wkind)           # N = M = 1024, K = 4, beta == alpha
    check(oracle_mod, a, W, b, h)


@pytest.mark.parametrize("wkind", ["pos", "signed"])
def test_cfg2_reduced(oracle_mod, wkind):
    a, W, b, h = workloads.make(2, M=5000, N=3001, wkind=wkind)
    check(oracle_mod, a, W, b, h)


@pytest.mark.parametrize("wkind", ["pos", "signed"])
def test_cfg3_reduced(oracle_mod, wkind):
    a, W, b, h = workloads.make(3, M=8192 + 77, N=1000, wkind=wkind)
    check(oracle_mod, a, W, b, h)


def test_cfg3_tight_cluster(oracle_mod):
    """sigma = 0.05 mixture, W >= 0: the case where the bar discriminates (SS4)."""
    a, W, b, h = workloads.make(3, M=6000, N=700, sigma=0.05, wkind="pos")
    check(oracle_mod, a, W, b, h)


def test_cfg5_reduced(oracle_mod):
    a, W, b, h = workloads.make(5, M=20000, N=2000)
    check(oracle_mod, a, W, b, h)


@pytest.mark.parametrize("cfg", [2, 3])
def test_self_variant(oracle_mod, cfg):
    """beta == alpha variant of each config (reading Q20): self terms exp(0) = 1."""
    a, W, b, h = workloads.make(cfg, M=3000, N=3000, same_points=True, wkind="pos")
    check(oracle_mod, a, W, b, h)


# ---------------------------------------------------------------- full BASELINE sizes, sampled targets
@pytest.mark.slow
@pytest.mark.parametrize("cfg,nsamp", [(2, 512), (3, 256), (5, 128)])
def test_full_size_sampled(oracle_mod, cfg, nsamp):
    a, W, b, h = workloads.make(cfg)
    J = workloads.sample_targets(b.shape[0], nsamp, seed=7 + cfg)
    check(oracle_mod, a, W, b, h, J=J)


def test_headline_separable_closed_form():
    """M = 65,536 sources on a product grid at K = 32, N = 65,536 targets: every
    V_j checked against the O(NK) closed form (no oracle needed at full size)."""
    from tests.test_oracle_pins import separable_closed_form
    a, W, g, c, w, _ = workloads.separable_grid(32, 16, seed=111)
    b = (workloads.uniform_points(65536, 32, 113) * 0.5 + 0.25).astype(np.float32)
    h = np.float32(0.5)
    V = gpu_eval(a, W, b, h)[:, 0]
    ref = separable_closed_form(g, c, w, b, float(h))
    err = np.max(np.abs(V - ref)) / float(np.abs(W).sum())
    assert err <= TOL_FP32, err


# ---------------------------------------------------------------- edge cases
@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (1, 300, 3), (129, 1, 5), (128, 128, 4), (255, 257, 17),
                                   (1000, 130, 31), (640, 384, 32), (3000, 128, 8), (130, 5000, 16)])
def test_edge_shapes(oracle_mod, M, N, K):
    a, W, b, h = workloads.custom(M, N, K, 1, 0.8, seed=M * 7 + N + K, wkind="signed")
    check(oracle_mod, a, W, b, h)


def test_single_target_tile_many_splits(oracle_mod):
    """N <= 128 with a long source range: every persistent CTA splits the one
    target tile -> exercises the deterministic cross-CTA fix-up with ~300 slots."""
    a, W, b, h = workloads.make(3, M=65536, N=100, wkind="pos")
    check(oracle_mod, a, W, b, h)


def test_one_hot_weights_at_tile_boundaries(oracle_mod):
    a, _, b, h = workloads.make(3, M=1000, N=300)
    for i in (0, 127, 128, 999):
        W = np.zeros((1000, 1), np.float32)
        W[i] = 1.0
        Vr = oracle_mod.oracle_eval(a, W, b, float(h))
        Vg = gpu_eval(a, W, b, h)
        assert np.max(np.abs(Vg - Vr)) <= 1e-6, i      # a row of the kernel matrix


def test_h_huge_is_plain_sum():
    a, W, b, _ = workloads.custom(3000, 400, 8, 1, 1.0, wkind="signed", seed=5)
    V = gpu_eval(a, W, b, np.float32(1e8))[:, 0]
    assert np.max(np.abs(V - W[:, 0].astype(np.float64).sum())) / np.abs(W).sum() <= TOL_FP32


def test_coincident_sources_clamp():
    """All sources at one point, targets at that point: d^2 = 0 exactly, Eq.3
    cancellation may go negative in FP32 -> the clamp keeps K <= 1."""
    p = workloads.uniform_points(1, 32, 9) * 3.0
    a = np.repeat(p, 2000, axis=0)
    W = workloads.weights(2000, 1, "pos", 10)
    V = gpu_eval(a, W, p.copy(), np.float32(0.05))[0, 0]
    assert abs(V - W.astype(np.float64).sum()) / W.sum() <= TOL_FP32


def test_beta_equals_alpha_self_kernel_one():
    """exp(0) = 1 inside the accuracy domain of Eq.3 in FP32 (reading Q11:
    2h^2 >> 1e5 u (||a||^2 + ||b||^2) after centring)."""
    a = workloads.uniform_points(500, 16, 3)
    W = np.zeros((500, 1), np.float32)
    W[200] = 1.0
    V = gpu_eval(a, W, a, np.float32(0.2))
    assert abs(V[200, 0] - 1.0) <= 1e-5


def test_zero_sources_gives_zeros():
    with ks.KernelSum(4, 1.0, _PREC["p"]) as plan:
        plan.set_sources(torch.zeros((0, 4), device="cuda"), torch.zeros((0, 1), device="cuda"))
        V = plan.eval(torch.rand((300, 4), device="cuda"))
        torch.cuda.synchronize()
        assert V.shape == (300, 1) and torch.all(V == 0)


def test_zero_targets_noop():
    with ks.KernelSum(4, 1.0, _PREC["p"]) as plan:
        plan.set_sources(torch.rand((10, 4), device="cuda"), torch.rand((10, 1), device="cuda"))
        V = plan.eval(torch.zeros((0, 4), device="cuda"))
        assert V.shape == (0, 1)


def test_deterministic_bitwise():
    a, W, b, h = workloads.make(3, M=20000, N=3000)
    assert np.array_equal(gpu_eval(a, W, b, h), gpu_eval(a, W, b, h))


def test_host_api_matches_device_api():
    a, W, b, h = workloads.make(2, M=3000, N=1500)
    assert np.array_equal(gpu_eval(a, W, b, h), gpu_eval(a, W, b, h, host=True))


@pytest.mark.parametrize("N", [20000, 40000 + 77])
def test_host_api_chunked_eval(oracle_mod, N):
    """ks_eval_host splits a large target set into up to 4 chunks (upload of chunk c + 1 and
    download of chunk c - 1 overlap the evaluation of chunk c); the result meets the bar and
    matches the one-piece device evaluation to rounding (the stream-K grouping differs)."""
    a, W, b, h = workloads.make(3, M=3000, N=N, wkind="pos")
    Vd = gpu_eval(a, W, b, h)
    Vh = gpu_eval(a, W, b, h, host=True)
    assert np.max(np.abs(Vh - Vd)) <= 1e-6 * np.abs(W).sum()
    J = workloads.sample_targets(N, 300, seed=5)
    check(oracle_mod, a, W, b, h, J=J, V=Vh)


@pytest.mark.parametrize("chunks,chunk0", [(1, 0), (0, -1), (3, 5), (4, 0), (2, 300), (0, 1000)])
def test_host_api_chunk_schedules(oracle_mod, chunks, chunk0):
    """Every ks_eval_host chunk schedule (one launch; equal chunks; a first chunk of t tiles,
    default one wave of tiles, and the rest in n - 1 chunks; a first chunk past N) gives the
    one-piece device result to rounding and meets the bar.  N = 40,077: > 2 waves of tiles
    on 148 SMs, a ragged last tile."""
    if _PREC["p"] != "3xf16":
        pytest.skip("chunking is independent of the precision")
    a, W, b, h = workloads.make(3, M=2000, N=40077, wkind="pos")
    Vd = gpu_eval(a, W, b, h)
    Vh = gpu_eval(a, W, b, h, host=True, options={"eval_chunks": chunks, "eval_chunk0": chunk0})
    assert np.max(np.abs(Vh - Vd)) <= 1e-6 * np.abs(W).sum()
    J = workloads.sample_targets(40077, 200, seed=6)
    check(oracle_mod, a, W, b, h, J=J, V=Vh)


def test_host_api_buffers_reusable_on_return():
    """ks_set_sources_host returns once alpha and W are uploaded (the preparation
    continues on the stream) and ks_eval_host once V is on the host: overwriting
    the caller's host arrays right after each call must not change any result,
    including across a source replacement and back-to-back evaluations."""
    a, W, b, h = workloads.make(3, M=5000, N=2100, wkind="pos")
    ref = gpu_eval(a, W, b, h)
    a2, W2, b2 = a.copy(), W.copy(), b.copy()
    with ks.KernelSum(a.shape[1], float(h), _PREC["p"]) as plan:
        plan.set_sources_host(a2, W2)
        a2[:] = 7.0
        W2[:] = -3.0
        V1 = plan.eval_host(b2).astype(np.float64)
        b2[:] = 0.0
        V2 = plan.eval_host(b).astype(np.float64)
        plan.set_sources_host(np.ascontiguousarray(a[::-1]), np.ascontiguousarray(W[::-1]))
        V3 = plan.eval_host(b).astype(np.float64)
    assert np.array_equal(V1, ref) and np.array_equal(V2, ref)
    # reversed source order: same sums up to rounding order
    assert np.max(np.abs(V3 - ref)) <= 1e-5 * np.abs(W).sum()


def test_repeated_eval_and_reset_sources(oracle_mod):
    """Counters are left zero across launches; sources can be replaced."""
    a, W, b, h = workloads.make(3, M=4000, N=200, wkind="pos")
    a2, W2, _, _ = workloads.make(3, M=2500, N=10, wkind="signed", seed_offset=9)
    with ks.KernelSum(32, float(h), _PREC["p"]) as plan:
        tb = torch.from_numpy(b).cuda()
        plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
        V1 = [plan.eval(tb).cpu().numpy() for _ in range(3)]
        plan.set_sources(torch.from_numpy(a2).cuda(), torch.from_numpy(W2).cuda())
        V2 = plan.eval(tb).cpu().numpy()
    assert np.array_equal(V1[0], V1[1]) and np.array_equal(V1[0], V1[2])
    check(oracle_mod, a, W, b, h, V=V1[0].astype(np.float64))
    check(oracle_mod, a2, W2, b, h, V=V2.astype(np.float64))


# ---------------------------------------------------------------- API errors on the GPU
def test_api_errors():
    ctx = ks.ks_create(8, 1.0)
    try:
        with pytest.raises(ks.KsError) as e:
            ks.ks_eval(ctx, 0, 10, 0)
        assert e.value.status == ks.KS_ESTATE
        with pytest.raises(ks.KsError) as e:
            ks.ks_set_sources(ctx, 0, 0, 10, 1)
        assert e.value.status == ks.KS_EINVAL
        with pytest.raises(ks.KsError) as e:
            ks.ks_set_sources(ctx, 0, 0, 0, 0)
        assert e.value.status == ks.KS_EINVAL
        with pytest.raises(ks.KsError) as e:
            ks.ks_set_precision(ctx, 9)
        assert e.value.status == ks.KS_EINVAL
    finally:
        ks.ks_destroy(ctx)
    ctx = ks.ks_create(64, 1.0)
    try:
        ks.ks_set_precision(ctx, "fp32")
        a = torch.rand((10, 64), device="cuda")
        w = torch.rand((10, 1), device="cuda")
        with pytest.raises(ks.KsError) as e:
            ks.ks_set_sources(ctx, a.data_ptr(), w.data_ptr(), 10, 1)
        assert e.value.status == ks.KS_EUNSUPPORTED
    finally:
        ks.ks_destroy(ctx)


def test_info_reports_path():
    with ks.KernelSum(32, 1.0, _PREC["p"]) as plan:
        plan.set_sources(torch.rand((1000, 32), device="cuda"), torch.rand((1000, 1), device="cuda"))
        plan.eval(torch.rand((5000, 32), device="cuda"))
        info = plan.info()
        want = ks.KS_PATH_FP32 if _PREC["p"] == "fp32" else ks.KS_PATH_TC
        # 3xf16 at R = 1: the folded layout adds 6 norm columns (K step of their own at K = 32)
        assert info["path"] == want and info["k_pad"] == (64 if info["precision"] == ks.KS_PREC_3XF16 else 32)
        assert info["num_ctas"] >= 1 and info["fused_launches"] == 1


def test_auto_policy():
    """AUTO: the tcgen05 split-FP16 kernel for every source-set size (SS7); the FP32
    kernel on request."""
    for M, want, prec in ((1024, ks.KS_PATH_TC, ks.KS_PREC_3XF16), (8192, ks.KS_PATH_TC, ks.KS_PREC_3XF16)):
        with ks.KernelSum(32, 1.0, "auto") as plan:
            plan.set_sources(torch.rand((M, 32), device="cuda"), torch.rand((M, 1), device="cuda"))
            assert plan.info()["path"] == want and plan.info()["precision"] == prec


# ---------------------------------------------------------------- the paper's grid corners (NEXT-2)
@pytest.mark.parametrize("orient,K", [("paper", 32), ("paper", 256), ("flip", 32), ("flip", 256)])
def test_paper_grid_corners(oracle_mod, orient, K):
    """The corners of the paper's workload grid at M = 524,288 in both
    orientations (reading Q21): 1,024 weighted sources x 524,288 targets (Alg.1's own, 4,096
    target tiles of 8 source tiles) and 524,288 sources x 1,024 targets (8 target tiles swept by
    stream-K), on sampled targets."""
    if _PREC["p"] == "fp32" and K > 32:
        pytest.skip("the FP32 kernel serves K <= 32")
    M = 524288
    ns, nt = (1024, M) if orient == "paper" else (M, 1024)
    a, W, b, h = workloads.custom(ns, nt, K, 1, np.sqrt(K) / 4.0, wkind="pos", seed=K + (1 if orient == "paper" else 2))
    J = workloads.sample_targets(nt, 40 if orient == "paper" else 24, seed=K)
    check(oracle_mod, a, W, b, h, J=J)
