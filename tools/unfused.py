"""The paper's unfused comparison ("cuBLAS-Unfused"; Alg.1
P:L102-132) on B200, for NEXT-1: norms, a cuBLAS SGEMM for the alpha^T beta
block, the kernel evaluation as PyTorch elementwise passes over the M x N
intermediate in HBM, and a cuBLAS GEMV with W.  It is a measurement baseline,
not part of the product path (which is the fused kernel in libks.so).

Same arithmetic conventions as the fused path where they matter for the
comparison: centring on the source mean (FP64 accumulation), FP32 GEMM with
TF32 disabled (the FP32-equivalent accuracy class of the fused default),
exp2 of a log2(e)-prescaled argument, d^2 clamped at 0.  Targets are
processed in chunks so the intermediate fits a fixed HBM budget.
"""
from __future__ import annotations

import math

import torch


def unfused_eval(ta: torch.Tensor, tw: torch.Tensor, tb: torch.Tensor, h: float,
                 budget_bytes: int = 8 << 30) -> torch.Tensor:
    """V [N, R] = sum_i exp(-||alpha_i - beta_j||^2 / 2h^2) W_i, unfused (Alg.1)."""
    torch.backends.cuda.matmul.allow_tf32 = False
    M, K = ta.shape
    N = tb.shape[0]
    c = math.log2(math.e) / (2.0 * h * h)
    mu = ta.double().mean(0).float()                      # Alg.1 l.3-4: vec_alpha, vec_beta (centred)
    a = ta - mu
    b = tb - mu
    na = (a.double() * a.double()).sum(1).float().mul_(-c)   # -c ||alpha_i||^2
    nb = (b.double() * b.double()).sum(1).float().mul_(-c)
    b2 = b * (2.0 * c)                                    # prescale the small operand, not the M x N block
    V = torch.empty((N, tw.shape[1]), device=ta.device, dtype=torch.float32)
    nc = max(1, min(N, budget_bytes // max(1, 4 * M)))
    for j0 in range(0, N, nc):
        j1 = min(N, j0 + nc)
        G = torch.mm(b2[j0:j1], a.t())                    # Alg.1 l.10: cuBLAS SGEMM, [nc, M] to HBM
        G.add_(na[None, :]).add_(nb[j0:j1, None])         # l.11: + norms (-c d^2 in log2 units)
        G.clamp_(max=0.0).exp2_()                         # l.12-13: d^2 >= 0, exp
        torch.mm(G, tw, out=V[j0:j1])                     # l.16: cuBLAS GEMV/GEMM with W
    return V


def hbm_bytes_per_pair(R: int = 1) -> dict:
    """HBM traffic per (source, target) pair of the intermediate, by design:
    this module's eager version and the best any unfused design can do
    (GEMM writes the block once, one fused exp+GEMV pass reads it once)."""
    eager = 4 + 4 * 2 * 4 + 4          # GEMM write, 4 read+write elementwise passes, GEMM-with-W read
    return {"eager_passes": eager, "best_unfused": 8}
