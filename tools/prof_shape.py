"""Scratch: one fused evaluation of a custom (M=N, K, R) shape for the phase profile (KS_PROF build,
KS_CTA_TIMES=file).   python tools/prof_shape.py K R [M]"""
import sys
import numpy as np, torch
sys.path.insert(0, '.')
import workloads
import paper_conf_icppw_wangkbgj16_b200 as ks
K, R = int(sys.argv[1]), int(sys.argv[2])
M = int(sys.argv[3]) if len(sys.argv) > 3 else 65536
a, W, b, h = workloads.custom(M, M, K, R, 0.35 * np.sqrt(K), seed=K + R, wkind="pos")
plan = ks.KernelSum(K, float(h))
plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
V = plan.eval(torch.from_numpy(b).cuda())
torch.cuda.synchronize()
print(plan.info())
