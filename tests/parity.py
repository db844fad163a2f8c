"""Parity metrics (test infrastructure).

The acceptance metric comes from BASELINE.json:north_star, made concrete in
DESIGN.md SS4:

    e_norm = max_{j,r} |V_gpu[j,r] - V_ref[j,r]| / sum_i |W[i,r]|

bar 1e-5 for the FP32 and 3xTF32 paths, 2e-3 for plain TF32.  If
sum_i |W[i,r]| = 0 the GPU column must be exactly 0.  Diagnostics (not
pass/fail): e_S = max |dV| / S with S = sum_i K |W| from the oracle.
"""
import numpy as np

TOL_FP32 = 1e-5
TOL_3XTF32 = 1e-5
TOL_TF32 = 2e-3


def e_norm(V_gpu, V_ref, W):
    V_gpu = np.asarray(V_gpu, dtype=np.float64).reshape(V_ref.shape)
    W = np.asarray(W, dtype=np.float64)
    if W.ndim == 1:
        W = W[:, None]
    sw = np.abs(W).sum(axis=0)                      # [R]
    d = np.abs(V_gpu - V_ref)                       # [n, R]
    if d.size == 0:
        return 0.0
    if not np.all(np.isfinite(V_gpu)):             # NaN / inf never pass (max() would skip a NaN)
        return float("inf")
    out = 0.0
    for r in range(V_ref.shape[1]):
        if sw[r] == 0.0:
            if np.any(V_gpu[:, r] != 0.0):
                return float("inf")
            continue
        out = max(out, float(d[:, r].max() / sw[r]))
    return out


def e_S(V_gpu, V_ref, S):
    V_gpu = np.asarray(V_gpu, dtype=np.float64).reshape(V_ref.shape)
    with np.errstate(divide="ignore", invalid="ignore"):
        q = np.abs(V_gpu - V_ref) / S
    q = q[np.isfinite(q)]
    return float(q.max()) if q.size else 0.0
