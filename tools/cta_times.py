"""Analyse KS_CTA_TIMES dumps: per-launch CTA start/end spread."""
import sys
import numpy as np
blocks, cur = [], []
for line in open(sys.argv[1]):
    if line.startswith("--"):
        blocks.append(np.array(cur, dtype=np.float64)); cur = []
    else:
        cur.append([float(x) for x in line.split()])
for a in blocks[-2:]:
    t0 = a[:, 1].min(); s = (a[:, 1] - t0) / 1e3; e = (a[:, 2] - t0) / 1e3
    print(f"grid {len(a)}: start spread {s.max():.1f} us, end min {e.min():.1f} med {np.median(e):.1f} max {e.max():.1f} us, "
          f"mean busy {np.mean(e - s):.1f} us; sum(busy)/(G*max) = {np.sum(e - s) / (len(a) * e.max()):.3f}")
    order = np.argsort(e)
    print("  earliest ends:", [(int(a[i, 0]), round(e[i], 1)) for i in order[:6]])
    print("  latest ends:", [(int(a[i, 0]), round(e[i], 1)) for i in order[-6:]])
    print("  latest starts:", [(int(a[i, 0]), round(s[i], 1)) for i in np.argsort(s)[-6:]])
