"""Scratch: distribution of the host-API end-to-end step time (cfg3) -- mean, median, min, max."""
import sys, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks

a, W, b, h = workloads.make(3)
ha = torch.from_numpy(a).pin_memory().numpy(); hw = torch.from_numpy(W).pin_memory().numpy()
hb = torch.from_numpy(b).pin_memory().numpy(); hv = torch.empty((b.shape[0], 1)).pin_memory().numpy()
plan = ks.KernelSum(a.shape[1], float(h))
for _ in range(5):
    plan.set_sources_host(ha, hw); plan.eval_host(hb, out=hv)
torch.cuda.synchronize()
ms = []
for _ in range(int(sys.argv[1]) if len(sys.argv) > 1 else 60):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    plan.set_sources_host(ha, hw); plan.eval_host(hb, out=hv)
    torch.cuda.synchronize(); ms.append(1e3 * (time.perf_counter() - t0))
ms = np.array(ms)
print("e2e ms: mean %.3f median %.3f min %.3f max %.3f  p90 %.3f" % (ms.mean(), np.median(ms), ms.min(), ms.max(), np.percentile(ms, 90)))
