"""Scratch check of the tensor-core path on small shapes (each case in a
subprocess with a timeout so a pipeline deadlock cannot hang the box)."""
import subprocess, sys, json

CASES = [
    # M, N, K, R, h, precision
    (128, 128, 16, 16, 1.0, "3xtf32"),
    (128, 128, 16, 1, 1.0, "3xtf32"),
    (256, 128, 32, 16, 1.0, "3xtf32"),
    (1000, 300, 64, 16, 1.5, "3xtf32"),
    (1000, 300, 64, 16, 1.5, "tf32"),
    (3000, 700, 256, 16, 2.0, "3xtf32"),
    (2000, 500, 40, 5, 1.0, "3xtf32"),
    (2000, 500, 32, 40, 1.0, "3xtf32"),
    (20000, 100, 64, 16, 2.0, "3xtf32"),
]

CHILD = r'''
import sys, json, numpy as np, torch
sys.path.insert(0, ".")
import workloads, oracle
import paper_conf_icppw_wangkbgj16_b200 as ks
M, N, K, R, h, prec = json.loads(sys.argv[1])
a, W, b, _ = workloads.custom(M, N, K, R, h, seed=M + N + K + R, wkind="signed")
with ks.KernelSum(K, h, prec) as p:
    p.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
    V = p.eval(torch.from_numpy(b).cuda()); torch.cuda.synchronize()
    info = p.info()
Vg = V.cpu().numpy().astype(np.float64)
Vr = oracle.oracle_eval(a, W, b, h)
err = float(np.max(np.abs(Vg - Vr).max(axis=0) / np.abs(W).sum(axis=0)))
print(json.dumps({"case": [M, N, K, R, h, prec], "e_norm": err, "path": info["path"], "ctas": info["num_ctas"],
                  "max_abs_V": float(np.abs(Vr).max()), "sample_gpu": Vg[0, :3].tolist(), "sample_ref": Vr[0, :3].tolist()}))
'''
for c in CASES:
    try:
        r = subprocess.run([sys.executable, "-c", CHILD, json.dumps(c)], capture_output=True, text=True, timeout=120)
        print(r.stdout.strip() or r.stderr.strip()[-800:], flush=True)
    except subprocess.TimeoutExpired:
        print("TIMEOUT", c, flush=True)
