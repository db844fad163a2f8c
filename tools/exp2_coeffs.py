"""Fit the degree-5 polynomial for 2^f on [-0.5, 0.5] used by exp2_poly2
(ks_ptx.cuh): minimax of the relative error with p(0) = 1 fixed (linear
program on a dense Chebyshev grid), then the error of FP32 Horner evaluation."""
import numpy as np
from scipy.optimize import linprog

deg = 5
f = np.unique(np.concatenate([np.cos(np.linspace(0, np.pi, 4001)) * 0.5, [-0.5, 0.5, 0.0]]))
target = 2.0 ** f
A = np.stack([f ** k / target for k in range(1, deg + 1)], 1)
b0 = 1 / target - 1
Aub = np.vstack([np.hstack([A, -np.ones((len(f), 1))]), np.hstack([-A, -np.ones((len(f), 1))])])
r = linprog(np.r_[np.zeros(deg), 1.0], A_ub=Aub, b_ub=np.r_[-b0, b0], bounds=[(None, None)] * (deg + 1),
            method="highs")
co = r.x[:deg].astype(np.float32)
print("minimax relative error %.3e" % r.x[-1])
x = np.random.default_rng(0).uniform(-0.5, 0.5, 2_000_000).astype(np.float32)
fma = lambda a, b, c: np.float32(a.astype(np.float64) * b.astype(np.float64) + np.float64(c))
p = np.full_like(x, co[4])
for k in (3, 2, 1, 0):
    p = fma(p, x, co[k])
p = fma(p, x, np.float32(1))
print("FP32 Horner max relative error %.3e" % np.max(np.abs(p / 2.0 ** x.astype(np.float64) - 1)))
print("coefficients c1..c5:", ", ".join("%.9ef" % c for c in co))
