"""Scratch: R = 1 fused-kernel ms, folded norms (default) vs KS_TC_FOLD=0, by K (M = N = 65,536)."""
import os, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

for K in (16, 32, 48, 64, 96, 128, 192, 256):
    a, W, b, h = workloads.custom(65536, 65536, K, 1, 0.35 * np.sqrt(K), seed=K, wkind="pos")
    plan = ks.KernelSum(K, float(h))
    ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
    plan.set_sources(ta, tw)
    V = plan.eval(tb)
    for _ in range(2): plan.eval(tb, out=V)
    torch.cuda.synchronize()
    ks.ks_timing_read(plan.ctx, reset=True)
    ks.ks_timing_enable(plan.ctx, True)
    for _ in range(5): plan.eval(tb, out=V)
    kms, n = ks.ks_timing_read(plan.ctx, reset=True)
    print(f"FOLD={os.environ.get('KS_TC_FOLD', '1')} K={K} kernel {kms / n:.4f} ms k_pad={plan.info()['k_pad']}", flush=True)
    plan.close()
