"""Kernel timeline of device steps (ks_set_sources + ks_eval on resident inputs) from the CUDA
activity trace (torch.profiler / CUPTI): each kernel's start offset from the step's first kernel
and its duration, so the gaps between launches and the time outside the fused kernel show.
A measurement tool, not the bench contract (numbers under a tracer are never bench values).
Usage: tools/step_timeline.py [CFG] [STEPS]  |  tools/step_timeline.py custom M N K h [STEPS]"""
import sys

import torch
from torch.profiler import ProfilerActivity, profile

sys.path.insert(0, ".")
import workloads  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

if len(sys.argv) > 1 and sys.argv[1] == "custom":  # custom M N K h [steps]: uniform points, W ~ U[0,1]
    M, N, K, hh = int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), float(sys.argv[5])
    steps = int(sys.argv[6]) if len(sys.argv) > 6 else 3
    a, W, b, h = workloads.custom(M, N, K, 1, hh, seed=K)
else:
    cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    a, W, b, h = workloads.make(cfg, wkind="pos")
plan = ks.KernelSum(a.shape[1], float(h))
da, dw, db = (torch.from_numpy(x).cuda() for x in (a, W, b))
V = torch.empty((b.shape[0], W.shape[1]), device="cuda")
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
for _ in range(3):
    plan.set_sources(da, dw)
    plan.eval(db, out=V)
torch.cuda.synchronize()
with profile(activities=[ProfilerActivity.CUDA]) as prof:
    for _ in range(steps):
        flush.fill_(1.0)
        plan.set_sources(da, dw)
        plan.eval(db, out=V)
    torch.cuda.synchronize()
ev = sorted((e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA),
            key=lambda e: e.time_range.start)
step, t0, prev_end = [], None, None
for e in ev:
    name = e.name.split("(")[0].replace("void ", "")[:48]
    if "elementwise" in name or "fill" in name.lower():  # the L2 flush starts a step
        if step:
            print(f"  step span {step[-1][1] + step[-1][2]:.1f} us")
        step, t0, prev_end = [], None, e.time_range.end
        print(f"-- step (L2 flush {e.time_range.end - e.time_range.start:.1f} us)")
        continue
    s, d = e.time_range.start, e.time_range.end - e.time_range.start
    if t0 is None:
        print(f"  first kernel starts {s - prev_end:.1f} us after the flush ends")
        t0 = s
    gap = 0.0 if prev_end is None else s - prev_end
    prev_end = e.time_range.end
    step.append((name, s - t0, d))
    print(f"  {s - t0:9.1f} us  dur {d:9.1f} us  gap {gap:6.1f}  {name}")
if step:
    print(f"  step span {step[-1][1] + step[-1][2]:.1f} us")
