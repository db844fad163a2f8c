"""Scratch timing of ks_eval on one config (not the bench contract)."""
import sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
a, W, b, h = workloads.make(cfg)
prec = sys.argv[3] if len(sys.argv) > 3 else "auto"
plan = ks.KernelSum(a.shape[1], float(h), prec)
ta, tw, tb = (torch.from_numpy(x).cuda() for x in (a, W, b))
plan.set_sources(ta, tw)
V = plan.eval(tb)
for _ in range(3): plan.eval(tb, out=V)
torch.cuda.synchronize()
ks.ks_timing_enable(plan.ctx, True)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
for _ in range(reps): plan.eval(tb, out=V)
e.record(); torch.cuda.synchronize()
ms = s.elapsed_time(e) / reps
kms, n = ks.ks_timing_read(plan.ctx)
pairs = a.shape[0] * b.shape[0]
print(f"cfg{cfg}: {ms:.3f} ms/eval (kernel {kms/n:.3f} ms)  {pairs/ms/1e9:.1f} Gpairs/s  info={plan.info()}")
