"""The paper's unfused comparison ("cuBLAS-Unfused"; Alg.1
P:L102-132) on B200, for NEXT-1: norms, a cuBLAS SGEMM for the alpha^T beta
block written to HBM, then the kernel evaluation and the product with W.  It is
a measurement baseline, not part of the product path (which is the fused kernel
in libks.so).

Two versions of the second half:
  "pass"  (default on CUDA tensors) -- ONE kernel (tools/unfused_expw.cu) reads
          each element of the block once: norm add, d^2 >= 0 clamp, exp2, times W,
          row sum.  8 HBM bytes per pair (GEMM write + one read): the best any
          design that materialises the block can do, i.e. the fair comparison.
  "eager" -- PyTorch elementwise passes + a cuBLAS GEMM with W (~40 B per pair);
          also the CPU-tensor path used by tests/test_unfused_baseline.py.

Same arithmetic conventions as the fused path where they matter for the
comparison: centring on the source mean (FP64 accumulation), FP32 GEMM with
TF32 disabled (the FP32-equivalent accuracy class of the fused default),
exp2 of a log2(e)-prescaled argument, d^2 clamped at 0.  Targets are
processed in chunks so the intermediate fits a fixed HBM budget.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "libunfused_expw.so")
_lib = None


def build_lib(force: bool = False) -> str:
    """Compile tools/unfused_expw.cu for sm_100a into tools/libunfused_expw.so (C ABI)."""
    src = os.path.join(_HERE, "unfused_expw.cu")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        nvcc = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call([nvcc, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-shared",
                               "-Xcompiler", "-fPIC", "-cudart", "static", src, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build_lib()
        _lib = ctypes.CDLL(_LIB)
        P, L, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
        _lib.unfused_expw_rows.argtypes = [P, P, P, P, P, L, L, I, P]
        _lib.unfused_expw_rows.restype = I
    return _lib


def unfused_eval(ta: torch.Tensor, tw: torch.Tensor, tb: torch.Tensor, h: float,
                 budget_bytes: int = 24 << 30, mode: str | None = None) -> torch.Tensor:
    """V [N, R] = sum_i exp(-||alpha_i - beta_j||^2 / 2h^2) W_i, unfused (Alg.1)."""
    mode = mode or ("pass" if ta.is_cuda else "eager")
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
    wc = tw.contiguous()
    for j0 in range(0, N, nc):
        j1 = min(N, j0 + nc)
        G = torch.mm(b2[j0:j1], a.t())                    # Alg.1 l.10: cuBLAS SGEMM, [nc, M] to HBM
        if mode == "pass":                                # l.11-16 in one read of G
            st = torch.cuda.current_stream().cuda_stream
            err = _load().unfused_expw_rows(G.data_ptr(), na.data_ptr(), nb[j0:j1].data_ptr(), wc.data_ptr(),
                                            V[j0:j1].data_ptr(), j1 - j0, M, wc.shape[1], ctypes.c_void_p(st))
            if err:
                raise RuntimeError(f"unfused_expw_rows: CUDA error {err}")
            continue
        G.add_(na[None, :]).add_(nb[j0:j1, None])         # l.11: + norms (-c d^2 in log2 units)
        G.clamp_(max=0.0).exp2_()                         # l.12-13: d^2 >= 0, exp
        torch.mm(G, tw, out=V[j0:j1])                     # l.16: cuBLAS GEMV/GEMM with W
    return V


def hbm_bytes_per_pair(R: int = 1) -> dict:
    """HBM traffic per (source, target) pair of the intermediate, by design:
    the eager version and the one-pass version ("pass", the default on the GPU:
    GEMM writes the block once, one fused exp+W pass reads it once)."""
    eager = 4 + 4 * 2 * 4 + 4          # GEMM write, 4 read+write elementwise passes, GEMM-with-W read
    return {"eager_passes": eager, "best_unfused": 8, "pass": 8}
