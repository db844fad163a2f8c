"""Unit timeline of CTA 0 of the R = 1 kernel (KS_TRACE build: TRACE=1 PROF=0
tools/build_debug_lib.sh, run with KS_LIB=libks_dbg.so KS_CTA_TIMES=file): MMA issue period,
issue duration, commit-to-epilogue and release-to-reissue latencies."""
import sys, numpy as np
blocks = open(sys.argv[1]).read().strip().split("--")
blk = blocks[-2 if blocks[-1].strip() == "" else -1]
tr = np.array([[int(x) for x in l.split()[1:]] for l in blk.strip().splitlines() if l.startswith("trace")], dtype=np.float64)
q = tr[:, 0]; t = tr[:, 1:] - tr[0, 1]
lo, hi = 200, 240
print("unit  mma_go  mma_done  epi_wake  epi_rel   (cycles from unit 0's MMA start)")
for i in range(lo, hi):
    print("%4d %8.0f %8.0f %8.0f %8.0f" % (q[i], t[i, 0], t[i, 1], t[i, 2], t[i, 3]))
d = np.diff(t[100:1500, 0])
print("MMA issue period (median/mean): %.0f / %.0f" % (np.median(d), d.mean()))
print("issue duration (done-go) median: %.0f" % np.median(t[100:1500, 1] - t[100:1500, 0]))
print("epi wake - mma done median: %.0f" % np.median(t[100:1500, 2] - t[100:1500, 1]))
print("epi release - wake median: %.0f" % np.median(t[100:1500, 3] - t[100:1500, 2]))
nx = t[104:1504, 0] - t[100:1500, 3]
print("MMA go(q+4) - release(q) median: %.0f" % np.median(nx))
