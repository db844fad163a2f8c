"""Per-warp phase clocks of the R = 1 kernel (KS_PROF build: tools/build_debug_lib.sh, run with
KS_LIB=libks_dbg.so KS_CTA_TIMES=file): effective SM clock, MMA-warp and epilogue waits."""
import sys, numpy as np
blocks = open(sys.argv[1]).read().strip().split("--")
blk = blocks[-2 if blocks[-1].strip() == "" else -1]
rows = [l.split() for l in blk.strip().splitlines() if l.startswith("r1")]
a = np.array([[int(x) for x in l[2:]] for l in rows], dtype=np.float64)
print("clock %.3f GHz, run %.3f ms" % (((a[:, 3] - a[:, 2]) / (a[:, 1] - a[:, 0])).mean(), (a[:, 1] - a[:, 0]).mean() / 1e6))
pf = a[:, 4:].reshape(len(a), 20, 4)
if pf.sum() == 0: sys.exit()
tot = pf[:, :, 3]
def show(name, w, labels):
    t = tot[:, w].mean()
    print(f"{name:18s} run {t/1e6:7.3f} Mcyc  " + ", ".join(f"{lab} {pf[:, w, k].mean()/t:.3f}" for k, lab in enumerate(labels)))
show("warp1 MMA", 1, ["wait sempty", "wait full", "issue"])
for w in (4, 5, 8, 12, 16, 19):
    show(f"epi warp {w}", w, ["wait sfull", "unit", "seg end"])
e = pf[:, 4:20, :]
print("epi mean: " + ", ".join(f"{lab} {e[:, :, k].mean()/e[:, :, 3].mean():.3f}" for k, lab in enumerate(["wait sfull", "unit", "seg end"])))
