"""Determinism + parity spot check of the TC kernel on stream-K-split shapes (scratch)."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import workloads, oracle
import paper_conf_icppw_wangkbgj16_b200 as ks
prec = sys.argv[1] if len(sys.argv) > 1 else "3xtf32"
for (M, N) in [(8192 + 77, 1000), (8192, 1024), (4096 + 128, 256), (20000, 300)]:
    a, W, b, h = workloads.make(3, M=M, N=N, wkind="pos")
    outs = []
    for rep in range(6):
        with ks.KernelSum(32, float(h), prec) as p:
            p.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
            V = p.eval(torch.from_numpy(b).cuda()); torch.cuda.synchronize()
        outs.append(V.cpu().numpy()[:, 0].astype(np.float64))
    Vr = oracle.oracle_eval(a, W, b, float(h))[:, 0]
    errs = [float(np.max(np.abs(o - Vr)) / np.abs(W).sum()) for o in outs]
    same = all(np.array_equal(outs[0], o) for o in outs)
    print(M, N, "bitwise-repeatable", same, "max e_norm %.2e" % max(errs))
