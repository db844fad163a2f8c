"""Time ks_eval on one BASELINE config: ms per eval, kernel ms (CUDA events), board energy per eval
and power (NVML over ~1 s of evals), and with KS_CTA_TIMES the effective SM clock of the R = 1
kernel (clock64 over globaltimer per CTA).  Usage: tools/quick_time.py CFG [REPS] [PRECISION].
A measurement tool, not the bench contract."""
import sys, os, time
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 20
prec = sys.argv[3] if len(sys.argv) > 3 else "auto"
wkind = os.environ.get("WKIND", "pos")
a, W, b, h = workloads.make(cfg, wkind=wkind)
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
# energy over ~1 s
import pynvml
pynvml.nvmlInit(); hd = pynvml.nvmlDeviceGetHandleByIndex(0)
nrep = max(5, int(1000 / max(ms, 1e-3))) if not os.environ.get("KS_CTA_TIMES") else 1
torch.cuda.synchronize(); e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(hd); t0 = time.perf_counter()
for _ in range(nrep): plan.eval(tb, out=V)
torch.cuda.synchronize(); e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(hd); t1 = time.perf_counter()
jps = (e1 - e0) / 1e3 / nrep
watts = (e1 - e0) / 1e3 / (t1 - t0)
clk = ""
ctf = os.environ.get("KS_CTA_TIMES")
if ctf and os.path.exists(ctf):
    blocks = open(ctf).read().strip().split("--")
    rows = [l.split() for l in blocks[-2 if blocks[-1].strip() == "" else -1].strip().splitlines() if l.startswith("r1")]
    if rows:
        r = np.array([[int(x) for x in l[2:]] for l in rows], dtype=np.float64)
        f = (r[:, 3] - r[:, 2]) / (r[:, 1] - r[:, 0])
        clk = f" clk {f.mean():.3f} GHz (cta run {((r[:,1]-r[:,0]).max())/1e6:.3f} ms)"
Vr = None
print(f"cfg{cfg} {os.environ.get('TAG','')}: {ms:.4f} ms/eval (kernel {kms/n:.4f} ms) {pairs/ms/1e9:.1f} Gpairs/s "
      f"{jps*1e3:.1f} mJ/eval {watts:.0f} W{clk} info={plan.info()['tile_s']},{plan.info()['stages']}")
