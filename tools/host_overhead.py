"""Host-side cost of the device API calls (ks_set_sources + ks_eval through the Python binding,
no synchronisation) against the GPU time of the same step, for one BASELINE config.  A
measurement tool.  Usage: tools/host_overhead.py [CFG] [N]"""
import sys
import time

import torch

sys.path.insert(0, ".")
import workloads  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
n = int(sys.argv[2]) if len(sys.argv) > 2 else 200
a, W, b, h = workloads.make(cfg, wkind="pos")
plan = ks.KernelSum(a.shape[1], float(h))
da, dw, db = (torch.from_numpy(x).cuda() for x in (a, W, b))
V = torch.empty((b.shape[0], 1), device="cuda")
for _ in range(5):
    plan.set_sources(da, dw)
    plan.eval(db, out=V)
torch.cuda.synchronize()
t_set = t_ev = 0.0
for _ in range(n):
    t0 = time.perf_counter()
    plan.set_sources(da, dw)
    t1 = time.perf_counter()
    plan.eval(db, out=V)
    t2 = time.perf_counter()
    t_set += t1 - t0
    t_ev += t2 - t1
torch.cuda.synchronize()
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s.record()
for _ in range(n):
    plan.set_sources(da, dw)
    plan.eval(db, out=V)
e.record()
torch.cuda.synchronize()
print(f"cfg{cfg}: host set_sources {1e6 * t_set / n:.1f} us, eval {1e6 * t_ev / n:.1f} us per call; "
      f"back-to-back GPU {1e3 * s.elapsed_time(e) / n:.1f} us per step")
