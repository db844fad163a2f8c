import sys, numpy as np, torch
sys.path.insert(0, ".")
import workloads, oracle
import paper_conf_icppw_wangkbgj16_b200 as ks
for (M, N) in [(8192 + 77, 1000), (8192, 1024), (4096 + 128, 256), (20000, 300)]:
    a, W, b, h = workloads.make(3, M=M, N=N, wkind="pos")
    errs = []
    for rep in range(6):
        with ks.KernelSum(32, float(h), "3xtf32") as p:
            p.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
            V = p.eval(torch.from_numpy(b).cuda()); torch.cuda.synchronize()
            info = p.info()
        Vg = V.cpu().numpy()[:, 0].astype(np.float64)
        if rep == 0:
            Vr = oracle.oracle_eval(a, W, b, float(h))[:, 0]
        rel = np.abs(Vg - Vr) / np.abs(W).sum()
        bad = np.where(rel > 1e-6)[0]
        errs.append((rel.max(), len(bad), bad[:8].tolist(), sorted(set((bad // 128).tolist()))[:10]))
    print(M, N, "ctas", info["num_ctas"], errs)
