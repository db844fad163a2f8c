"""Time the host-API step (ks_set_sources_host + ks_eval_host, pinned buffers) of a BASELINE
config under several ks_eval_host chunk schedules, beside its pieces: the pinned uploads of
alpha+W and of beta alone, and the device step on resident inputs.  A measurement tool, not the
bench contract.  Usage: tools/e2e_time.py [CFG] [STEPS] [chunks:chunk0 ...]"""
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
import workloads  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
scheds = [tuple(int(x) for x in s.split(":")) for s in sys.argv[3:]] or [(0, 0), (0, -1), (1, 0), (3, 0)]
a, W, b, h = workloads.make(cfg, wkind="pos")
K = a.shape[1]
pairs = a.shape[0] * b.shape[0]
ha, hw, hb = (torch.from_numpy(x).pin_memory() for x in (a, W, b))
hv = torch.empty((b.shape[0], W.shape[1]), dtype=torch.float32).pin_memory()
flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")


def wall(fn, n=steps):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(n):
        flush.fill_(1.0)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        fn()
        torch.cuda.synchronize()
        ts.append(1e3 * (time.perf_counter() - t0))
    return float(np.median(ts)), float(np.mean(ts))


da, dw, db = (torch.empty(x.shape, device="cuda") for x in (ha, hw, hb))
print(f"cfg{cfg}: upload alpha+W {wall(lambda: (da.copy_(ha, non_blocking=True), dw.copy_(hw, non_blocking=True)))[0]:.4f} ms, "
      f"beta {wall(lambda: db.copy_(hb, non_blocking=True))[0]:.4f} ms "
      f"({(ha.numel() + hw.numel() + hb.numel()) * 4 / 1e6:.1f} MB)")
plan = ks.KernelSum(K, float(h))
da.copy_(ha)
dw.copy_(hw)
db.copy_(hb)
V = torch.empty((b.shape[0], W.shape[1]), device="cuda")
print(f"device step (resident inputs): {wall(lambda: (plan.set_sources(da, dw), plan.eval(db, out=V)))[0]:.4f} ms")
an, wn, bn, vn = ha.numpy(), hw.numpy(), hb.numpy(), hv.numpy()
for ch, c0 in scheds:
    plan.set_option("eval_chunks", ch)
    plan.set_option("eval_chunk0", c0)
    med, mean = wall(lambda: (plan.set_sources_host(an, wn), plan.eval_host(bn, out=vn)))
    print(f"e2e chunks={ch} chunk0={c0}: median {med:.4f} ms mean {mean:.4f} ms  {pairs / mean / 1e9:.1f} Gpairs/s")
plan.close()
