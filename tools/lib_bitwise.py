"""Evaluate a set of shapes through the library KS_LIB names and save V (npz), or compare two
such files bitwise: a check that a change meant to compute the same bits does.  A tool.
Usage: KS_LIB=libks_x.so tools/lib_bitwise.py save OUT.npz | tools/lib_bitwise.py cmp A.npz B.npz"""
import sys

import numpy as np

sys.path.insert(0, ".")
if sys.argv[1] == "cmp":
    a, b = np.load(sys.argv[2]), np.load(sys.argv[3])
    bad = [k for k in a.files if not np.array_equal(a[k], b[k])]
    print(f"{len(a.files) - len(bad)} of {len(a.files)} cases bitwise equal", bad[:10])
    sys.exit(1 if bad else 0)
import torch  # noqa: E402

import workloads  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402

out = {}
for K in (1, 4, 8, 10, 16, 26, 27, 32, 40, 58):
    for R, wk in ((1, "pos"), (1, "signed"), (3, "signed")):
        for coop in (0, 1):
            a, W, b, h = workloads.custom(3000 + 7 * K, 2100, K, R, 1.0, dist="gm", sigma=0.1, wkind=wk, seed=K)
            with ks.KernelSum(K, float(h), "auto", options={"coop_prep": coop}) as plan:
                plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
                V = plan.eval(torch.from_numpy(b).cuda())
                torch.cuda.synchronize()
                out[f"K{K}_R{R}_{wk}_coop{coop}"] = V.cpu().numpy()
# the general kernel's prep paths (K > 58; R = 1 log-weights, signed W, R = 16; TF32 modes)
for K, R, wk, prec in ((64, 1, "pos", "auto"), (100, 1, "signed", "auto"), (128, 16, "signed", "auto"),
                       (40, 1, "pos", "3xtf32"), (300, 2, "signed", "auto")):
    a, W, b, h = workloads.custom(2500, 1700, K, R, 2.0, dist="uniform", wkind=wk, seed=K + R)
    with ks.KernelSum(K, float(h), prec) as plan:
        plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
        V = plan.eval(torch.from_numpy(b).cuda())
        torch.cuda.synchronize()
        out[f"gen_K{K}_R{R}_{wk}_{prec}"] = V.cpu().numpy()
np.savez(sys.argv[2], **out)
print("saved", len(out))
