"""Per-CUDA-source-line warp-stall samples of an ncu report (needs -lineinfo)."""
import csv, io, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hi = next(i for i, r in enumerate(rows[:20]) if "Address" in r)
hdr = rows[hi]
iN = hdr.index("Warp Stall Sampling (Not-issued Samples)"); iA = hdr.index("Warp Stall Sampling (All Samples)")
scols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
cur = None; agg = defaultdict(lambda: [0, 0, defaultdict(int)])
for r in rows[hi + 1:]:
    if r and r[0].strip().isdigit():
        cur = (int(r[0]), r[1].strip()[:80]); continue
    if len(r) > iN and r[iN].isdigit():
        a = agg[cur]; a[0] += int(r[iA]); a[1] += int(r[iN])
        for i in scols:
            if r[i] not in ("", "0"):
                a[2][hdr[i]] += int(r[i])
tot = sum(v[0] for v in agg.values())
for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    rs = sorted(v[2].items(), key=lambda x: -x[1])[:2]
    print(f"{v[0]:8d} {100 * v[0] / tot:5.1f}%  L{k[0]:<4d} {k[1]:80s} {[(a.replace('stall_', ''), b) for a, b in rs]}")
