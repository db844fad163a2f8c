"""R > 1 policy sweep at M = N = 65,536 (input to the AUTO choice and DESIGN.md SS6b): fused time per
eval of the multi-column kernel (ks_fused_rv.cu, AUTO for K + 6 <= 64) against the general kernel
with the tensor-core weighted sum (r1_kernel = 0, weighted_sum = 0) and with the CUDA-core one
(weighted_sum = 1, R <= 16).  Prints ms per eval, pairs/s and the fraction of the MUFU-only
exponential bound (one MUFU.EX2 per pair, 16 per clock per SM) at 1965 MHz and, for the
multi-column kernel, at its own measured SM clock (ks_clock_read)."""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

n = int(sys.argv[1]) if len(sys.argv) > 1 else 65536
KS = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [8, 16, 32, 58]
RS = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else [2, 4, 8, 16, 32, 64]
SMS = 148


def run(a, W, b, h, opts, reps=5):
    plan = ks.KernelSum(a.shape[1], float(h), options=dict(opts, measure_clock=1))
    ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
    plan.set_sources(ta, tw)
    V = plan.eval(tb)
    for _ in range(2):
        plan.eval(tb, out=V)
    torch.cuda.synchronize()
    ks.ks_timing_read(plan.ctx, reset=True)
    ks.ks_timing_enable(plan.ctx, True)
    for _ in range(reps):
        plan.eval(tb, out=V)
    kms, _ = ks.ks_timing_read(plan.ctx, reset=True)
    try:
        ghz = ks.ks_clock_read(plan.ctx)[0]
    except ks.KsError:
        ghz = float("nan")
    info = plan.info()
    plan.close()
    return kms / reps, ghz, info


print(f"M = N = {n}; ms per eval (all launches); frac = MUFU-only bound / time", flush=True)
for K in KS:
    for R in RS:
        a, W, b, h = workloads.custom(n, n, K, R, 0.3 * np.sqrt(K) + 0.1, dist="gm", sigma=0.08, seed=K + R,
                                      wkind="signed")
        bound_ms = n * n / (16 * SMS * 1.965e9) * 1e3
        line = f"K={K:3d} R={R:3d}"
        for name, opts in (("rv", {}), ("general-TC", {"r1_kernel": 0, "weighted_sum": 0}),
                           ("general-CC", {"r1_kernel": 0, "weighted_sum": 1})):
            if name == "general-CC" and R > 16:
                continue
            ms, ghz, info = run(a, W, b, h, opts)
            extra = ""
            if name == "rv":
                assert info["kernel"] == 4, info
                extra = f" @{ghz:.2f} GHz frac {bound_ms * 1.965 / ghz / ms:.2f}" if ghz == ghz else ""
            line += f" | {name} {ms:7.3f} ms {n * n / ms / 1e9:6.2f} Tpairs/s frac@1965 {bound_ms / ms:.2f}{extra}"
        print(line, flush=True)
