"""Scratch: fused-kernel time of the FP32 kernel vs the tcgen05 kernel for small source sets
(input to the AUTO threshold).  K = 32, R = 1, W >= 0."""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

for N in (1024, 65536):
    for M in (512, 1024, 2048, 4096, 8192):
        a, W, b, h = workloads.custom(M, N, 32, 1, 1.0, seed=M + N, wkind="pos")
        ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
        res = []
        for prec in ("fp32", "3xf16"):
            plan = ks.KernelSum(32, float(h), prec)
            plan.set_sources(ta, tw)
            V = plan.eval(tb)
            for _ in range(3): plan.eval(tb, out=V)
            torch.cuda.synchronize()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for _ in range(20):
                plan.set_sources(ta, tw); plan.eval(tb, out=V)
            e.record(); torch.cuda.synchronize()
            res.append(s.elapsed_time(e) / 20)
            plan.close()
        print(f"N={N} M={M}: fp32 {res[0]:.4f} ms  tc {res[1]:.4f} ms  (set_sources + eval)", flush=True)
