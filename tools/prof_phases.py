"""Summarise a KS_PROF=1 phase profile (KS_CTA_TIMES file, last block):
mean per-warp clock64 totals of waits / work, as a fraction of the warp's run."""
import sys
import numpy as np

blocks = open(sys.argv[1]).read().strip().split("--")
rows = [list(map(int, l.split())) for l in blocks[-2 if blocks[-1].strip() == "" else -1].strip().splitlines()]
a = np.array(rows, dtype=np.float64)
pf = a[:, 3:].reshape(len(a), 20, 5)
tot = pf[:, :, 4]
def show(name, w, labels):
    t = tot[:, w].mean()
    parts = ", ".join(f"{lab} {pf[:, w, k].mean() / t:.3f}" for k, lab in enumerate(labels))
    print(f"{name:22s} run {t / 1e6:8.3f} Mcyc  {parts}")
show("warp0 operand TMA", 0, ["wait empty"])
show("warp1 MMA", 1, ["wait full", "wait sempty", "issue", "commit+rest"])
show("warp3 norms/W loads", 3, ["wait wempty"])
for w in (4, 5, 6, 7, 8, 12, 16, 19):
    show(f"epilogue warp {w}", w, ["wait wfull", "wait sfull", "compute", "tail"])
e = pf[:, 4:20, :]
print("epilogue mean: " + ", ".join(f"{lab} {e[:, :, k].mean() / e[:, :, 4].mean():.3f}"
                                     for k, lab in enumerate(["wait wfull", "wait sfull", "compute", "tail"])))
print("CTA run spread (globaltimer): min %.3f max %.3f ms" % ((a[:, 2] - a[:, 1]).min() / 1e6, (a[:, 2] - a[:, 1]).max() / 1e6))
