"""NEXT-2 + NEXT-4: the paper's workload grid (K in {32, 64, 128,
256}, one set of 1,024 points, the other from 1,024 to 524,288) on one B200, fused
(libks.so, AUTO) against the unfused cuBLAS design (tools/unfused.py: SGEMM into HBM
+ one pass, the paper's cuBLAS-Unfused made fair), with NVML board energy per
evaluation -- the B200 analog of the paper's Fig. 6 (speedup) and Table III
(energy saving).  Both orientations (reading Q21):
  "paper": 1,024 weighted SOURCES, M = 1,024..524,288 TARGETS -- Alg.1's V = K W with
           W N-dimensional (N = 1,024) and V indexed by the M rows (P:L98, P:L104-110,
           P:L130-132): the fused kernel runs M/128 target tiles of 8 source tiles;
  "flip":  M SOURCES, 1,024 TARGETS: 8 target tiles, long source sweeps (stream-K).

    python tools/grid.py [out_dir]     (GPU; writes grid.json and grid.md)

Inputs: uniform points in [0,1]^K, W ~ U[0,1], h = sqrt(K)/4 (the paper does
not state h; this keeps ||a-b||^2 / 2h^2 ~ 1.3 on average), seeds from
workloads.custom.  One timed evaluation = set_sources + eval (both designs
recompute the norms), CUDA events, median of repeats; energy = NVML total
energy over >= 0.5 s of repeated evaluations.
"""
from __future__ import annotations

import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402
import workloads  # noqa: E402
from unfused import unfused_eval  # noqa: E402

KS = (32, 64, 128, 256)
MS = (1024, 8192, 131072, 524288)
N = 1024


def timed(fn, reps=None, min_s=0.2):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    one = time.perf_counter() - t0
    reps = reps or max(3, min(200, int(min_s / max(one, 1e-5))))
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    for s, e in ev:
        s.record()
        fn()
        e.record()
    torch.cuda.synchronize()
    return float(np.median([s.elapsed_time(e) for s, e in ev]))


def energy(fn, hdl, seconds=0.5):
    import pynvml
    torch.cuda.synchronize()
    e0 = pynvml.nvmlDeviceGetTotalEnergyConsumption(hdl)
    t0 = time.perf_counter()
    n = 0
    while time.perf_counter() - t0 < seconds:
        for _ in range(4):
            fn()
        n += 4
        torch.cuda.synchronize()
    e1 = pynvml.nvmlDeviceGetTotalEnergyConsumption(hdl)
    return (e1 - e0) / 1e3 / n


ORIENT = ("paper", "flip")


def run_point(K, M, orient, dev, hdl):
    h = math.sqrt(K) / 4.0
    ns, nt = (N, M) if orient == "paper" else (M, N)    # (sources, targets)
    a, W, b, h = workloads.custom(ns, nt, K, 1, h, dist="uniform", wkind="pos", seed=1000 * K + M % 997)
    ta, tw, tb = (torch.from_numpy(x).to(dev) for x in (a, W, b))
    plan = ks.KernelSum(K, float(h), "auto")
    V = torch.empty((nt, 1), device=dev)

    def fused():
        plan.set_sources(ta, tw)
        plan.eval(tb, out=V)

    def unf():
        return unfused_eval(ta, tw, tb, float(h))

    t_f = timed(fused)
    t_u = timed(unf)
    e_f = energy(fused, hdl)
    e_u = energy(unf, hdl)
    J = workloads.sample_targets(nt, 16, K + M)
    Vr = oracle.oracle_eval(a, W, b, float(h), J=J)
    fused()
    Vf = V.cpu().numpy().astype(np.float64)[J]
    Vu = unf().cpu().numpy().astype(np.float64)[J]
    sw = np.abs(W).sum()
    info = plan.info()
    plan.close()
    r = {"orient": orient, "K": K, "M": M, "sources": ns, "targets": nt, "h": float(h), "fused_ms": t_f,
         "unfused_ms": t_u, "speedup": t_u / t_f, "fused_j": e_f, "unfused_j": e_u,
         "energy_saving": 1.0 - e_f / e_u, "fused_pairs_per_s": ns * nt / (t_f / 1e3),
         "fused_kernel": {1: "fp32", 2: "tcgen05", 3: "tcgen05 R=1"}.get(info["kernel"]),
         "e_norm_fused": float(np.max(np.abs(Vf - Vr)) / sw), "e_norm_unfused": float(np.max(np.abs(Vu - Vr)) / sw)}
    del ta, tw, tb, V
    torch.cuda.empty_cache()
    return r


def main():
    out_dir = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "r02")
    os.makedirs(out_dir, exist_ok=True)
    import pynvml
    pynvml.nvmlInit()
    hdl = pynvml.nvmlDeviceGetHandleByIndex(0)
    oracle.build()
    dev = torch.device("cuda", 0)
    rows = []
    for orient in ORIENT:
        for K in KS:
            for M in MS:
                r = run_point(K, M, orient, dev, hdl)
                rows.append(r)
                print(json.dumps(r), flush=True)
    json.dump(rows, open(os.path.join(out_dir, "grid.json"), "w"), indent=1)
    lines = []
    for orient in ORIENT:
        title = ("1,024 weighted sources, M targets (the paper's Alg.1 orientation)" if orient == "paper"
                 else "M sources, 1,024 targets")
        lines += [f"### {title}", "",
                  "| K | M | fused ms | unfused ms | speedup | fused mJ | unfused mJ | energy saved | "
                  "fused e_norm | unfused e_norm |", "|---|---|---|---|---|---|---|---|---|---|"]
        for r in rows:
            if r["orient"] != orient:
                continue
            lines.append(f"| {r['K']} | {r['M']:,} | {r['fused_ms']:.4f} | {r['unfused_ms']:.4f} | "
                         f"{r['speedup']:.2f}x | {1e3 * r['fused_j']:.2f} | {1e3 * r['unfused_j']:.2f} | "
                         f"{100 * r['energy_saving']:.0f}% | {r['e_norm_fused']:.1e} | {r['e_norm_unfused']:.1e} |")
        lines.append("")
        lines += [f"Speedup / energy saved ({orient}):", "", "| K | " + " | ".join(f"M={m:,}" for m in MS) + " |",
                  "|---|" + "---|" * len(MS)]
        for K in KS:
            cells = [f"{r['speedup']:.1f}x / {100 * r['energy_saving']:.0f}%" for r in rows
                     if r["orient"] == orient and r["K"] == K]
            lines.append(f"| {K} | " + " | ".join(cells) + " |")
        lines.append("")
    open(os.path.join(out_dir, "grid.md"), "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()
