"""Scratch: fused-kernel time of the two weighted-sum variants (CUDA-core vs tensor-core V)
over (K, R) at M = N = 65,536 -- input to the AUTO policy.  Run twice: KS_TC_VCC unset / =0."""
import os, sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

for K in (32, 64, 128, 256):
    for R in (2, 4, 8, 16):
        a, W, b, h = workloads.custom(65536, 65536, K, R, 0.35 * np.sqrt(K), seed=K + R, wkind="pos")
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
        ks.ks_timing_enable(plan.ctx, False)
        print(f"VCC={os.environ.get('KS_TC_VCC', 'auto')} K={K} R={R} kernel {kms / n:.4f} ms tile_s={plan.info()['tile_s']}", flush=True)
        plan.close()
