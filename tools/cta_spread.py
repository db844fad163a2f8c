"""Per-CTA start / end spread of the R = 1 fused kernel (globaltimer at every CTA's start and end,
KS_CTA_TIMES) for one BASELINE config: how long the launch ramp and the tail are against the
kernel's span.  A measurement tool.  Usage: tools/cta_spread.py [CFG] [EVALS]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
path = "/tmp/ks_cta_times.txt"
if os.path.exists(path):
    os.remove(path)
os.environ["KS_CTA_TIMES"] = path
import workloads  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
n = int(sys.argv[2]) if len(sys.argv) > 2 else 5
a, W, b, h = workloads.make(cfg, wkind="pos")
plan = ks.KernelSum(a.shape[1], float(h))
da, dw, db = (torch.from_numpy(x).cuda() for x in (a, W, b))
V = torch.empty((b.shape[0], 1), device="cuda")
for _ in range(n):
    plan.set_sources(da, dw)
    plan.eval(db, out=V)
torch.cuda.synchronize()
blocks = [blk for blk in open(path).read().split("--") if blk.strip()]
for blk in blocks[-3:]:
    rows = np.array([[int(x) for x in ln.split()[2:6]] for ln in blk.strip().splitlines() if ln.startswith("r1")],
                    dtype=np.float64)
    t0, t1 = rows[:, 0] - rows[:, 0].min(), rows[:, 1] - rows[:, 0].min()
    span = t1.max()
    print(f"cfg{cfg}: span {span / 1e3:.1f} us; CTA start max {t0.max() / 1e3:.2f} us; CTA end min "
          f"{t1.min() / 1e3:.1f} median {np.median(t1) / 1e3:.1f} max {t1.max() / 1e3:.1f} us; "
          f"clock {np.mean((rows[:, 3] - rows[:, 2]) / (rows[:, 1] - rows[:, 0])):.3f} GHz")
if os.environ.get("DETAIL"):
    blk = blocks[-1]
    rows = np.array([[int(x) for x in ln.split()[1:6]] for ln in blk.strip().splitlines() if ln.startswith("r1")],
                    dtype=np.float64)
    clk = (rows[:, 4] - rows[:, 3]) / (rows[:, 2] - rows[:, 1])
    end = (rows[:, 2] - rows[:, 1].min()) / 1e3
    cyc = (rows[:, 4] - rows[:, 3]) / 1e3
    o = np.argsort(end)
    print("per-CTA (cta, end us, clock GHz, kcycles), by end time:")
    for i in list(o[:8]) + list(o[-8:]):
        print(f"  {int(rows[i, 0]):4d} {end[i]:8.1f} {clk[i]:.3f} {cyc[i]:8.1f}")
    print("clock min/median/max", clk.min(), np.median(clk), clk.max(), " kcycles min/median/max", cyc.min(),
          np.median(cyc), cyc.max())
    print("end by CTA parity (even/odd mean):", end[rows[:, 0] % 2 == 0].mean(), end[rows[:, 0] % 2 == 1].mean())
    print("end by CTA half (<74 / >=74):", end[rows[:, 0] < 74].mean(), end[rows[:, 0] >= 74].mean())
