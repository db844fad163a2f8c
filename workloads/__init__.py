"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NO arithmetic of the method (no distances, exponentials,
norms or sums): it only draws points and weights.  Both the oracle
(``oracle/``) and the product path are fed the same FP32 bytes from here.

The paper states no distributions, h or W (SS IV only
gives sizes; reading Q18 in DESIGN.md), so the recipe is the one in
DESIGN.md SS5 / SURVEY.md SS8(d):

* generator: numpy ``Generator(PCG64(seed))`` -> float32;
* seeds: ``s = 20160 + cfg``: sources s, targets s+1, W s+2, mixture centres s+3;
* uniform points in [0,1]^K; Gaussian mixture: C=16 centres ~ U[0,1]^K,
  component chosen uniformly, point = centre + sigma * N(0, I);
* W ~ U[0,1] ("pos") or U[-1,1] ("signed"), R independent columns.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

SEED_BASE = 20160


@dataclass(frozen=True)
class Config:
    """One BASELINE.json workload.  M sources, N targets (M = N in every config)."""
    cfg: int
    M: int
    N: int
    K: int
    R: int
    h: float
    dist: str            # "uniform" | "gm"
    sigma: float = 0.1   # GM spread
    same_points: bool = False  # cfg1: beta is alpha (reading Q20)

    @property
    def pairs(self) -> int:
        return self.M * self.N


# BASELINE.json "configs", in order (1-based cfg ids as in SURVEY.md SS8(a)).
CONFIGS = {
    1: Config(1, 1024, 1024, 4, 1, 1.0, "uniform", same_points=True),
    2: Config(2, 16384, 16384, 16, 1, 0.5, "uniform"),
    3: Config(3, 65536, 65536, 32, 1, 1.0, "gm", sigma=0.1),
    4: Config(4, 262144, 262144, 256, 16, 2.0, "uniform"),
    5: Config(5, 1048576, 1048576, 8, 1, 0.25, "uniform"),
}


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def uniform_points(n: int, K: int, seed: int) -> np.ndarray:
    return rng(seed).random((n, K), dtype=np.float64).astype(np.float32)


def mixture_centres(K: int, C: int, seed: int) -> np.ndarray:
    return rng(seed).random((C, K), dtype=np.float64)


def gm_points(n: int, K: int, centres: np.ndarray, sigma: float, seed: int) -> np.ndarray:
    g = rng(seed)
    comp = g.integers(0, centres.shape[0], size=n)
    noise = g.standard_normal((n, K))
    return (centres[comp] + sigma * noise).astype(np.float32)


def weights(n: int, R: int, kind: str, seed: int) -> np.ndarray:
    g = rng(seed)
    if kind == "pos":
        w = g.random((n, R))
    elif kind == "signed":
        w = 2.0 * g.random((n, R)) - 1.0
    else:
        raise ValueError(kind)
    return w.astype(np.float32)


def make(cfg: Config | int, *, M: int | None = None, N: int | None = None,
         wkind: str = "pos", sigma: float | None = None, same_points: bool | None = None,
         seed_offset: int = 0):
    """Return (alpha [M,K], W [M,R], beta [N,K], h) as float32 arrays.

    M / N override the config's sizes (parity tests run reduced sizes of the
    same distribution); sigma overrides the GM spread (tight-cluster case).
    """
    if isinstance(cfg, int):
        cfg = CONFIGS[cfg]
    M = cfg.M if M is None else M
    N = cfg.N if N is None else N
    sig = cfg.sigma if sigma is None else sigma
    same = cfg.same_points if same_points is None else same_points
    s = SEED_BASE + cfg.cfg + seed_offset
    if cfg.dist == "uniform":
        alpha = uniform_points(M, cfg.K, s)
        beta = alpha[:N].copy() if same else uniform_points(N, cfg.K, s + 1)
    elif cfg.dist == "gm":
        cen = mixture_centres(cfg.K, 16, s + 3)
        alpha = gm_points(M, cfg.K, cen, sig, s)
        beta = alpha[:N].copy() if same else gm_points(N, cfg.K, cen, sig, s + 1)
    else:
        raise ValueError(cfg.dist)
    if same and N > M:
        raise ValueError("same_points needs N <= M")
    W = weights(M, cfg.R, wkind, s + 2)
    return alpha, W, beta, np.float32(cfg.h)


def custom(M: int, N: int, K: int, R: int, h: float, *, dist: str = "uniform",
           sigma: float = 0.1, wkind: str = "pos", seed: int = 1, same_points: bool = False):
    """Ad-hoc shapes (edge cases) with the same recipe and an explicit seed."""
    if dist == "uniform":
        alpha = uniform_points(M, K, seed)
        beta = alpha[:N].copy() if same_points else uniform_points(N, K, seed + 1)
    elif dist == "gm":
        cen = mixture_centres(K, 16, seed + 3)
        alpha = gm_points(M, K, cen, sigma, seed)
        beta = alpha[:N].copy() if same_points else gm_points(N, K, cen, sigma, seed + 1)
    else:
        raise ValueError(dist)
    W = weights(M, R, wkind, seed + 2)
    return alpha, W, beta, np.float32(h)


def separable_grid(K: int, G: int, seed: int):
    """Sources on a product grid {g[d,0], g[d,1]}^G x fixed constants c[d] (d >= G).

    Source i (0 <= i < 2^G) takes coordinate g[d, bit_d(i)] in dim d < G and
    c[d] in dims d >= G; its weight is prod_d w[d, bit_d(i)].  Returns
    (alpha [2^G, K] f32, W [2^G, 1] f32, g [G,2] f32, c [K-G] f32, w [G,2] f32).
    Coordinates/weights are FP32 values; the factors are powers of two, so W
    is exact (the closed form in the tests sees the exact same weights).
    """
    gen = rng(seed)
    g = gen.random((G, 2)).astype(np.float32)
    c = gen.random(K - G).astype(np.float32)
    # powers of two: every product weight is exact in FP32, so the FP64
    # closed form and the FP32 W the GPU/oracle receive describe the same sum.
    w = np.exp2(gen.integers(-2, 3, size=(G, 2))).astype(np.float32)
    M = 1 << G
    idx = np.arange(M, dtype=np.int64)
    bits = (idx[:, None] >> np.arange(G)[None, :]) & 1          # [M, G]
    alpha = np.empty((M, K), dtype=np.float32)
    alpha[:, :G] = g[np.arange(G)[None, :], bits]
    alpha[:, G:] = c[None, :]
    Wf = np.ones(M, dtype=np.float64)
    for d in range(G):
        Wf *= w[d, bits[:, d]].astype(np.float64)
    return alpha, Wf.astype(np.float32)[:, None], g, c, w, bits


def sample_targets(N: int, n: int, seed: int, tile: int = 128, extra=()):
    """Seeded target subset for sampled parity: n distinct uniform indices (drawn
    without replacement, so n = N covers every target) plus the first/last target
    of the range and of tile boundaries, plus `extra`."""
    g = rng(seed)
    pick = set(int(x) for x in g.choice(N, size=min(n, N), replace=False)) if N > 0 else set()
    for b in (0, N - 1, tile - 1, tile, N - tile, N - tile - 1):
        if 0 <= b < N:
            pick.add(b)
    for e in extra:
        if 0 <= e < N:
            pick.add(int(e))
    return np.array(sorted(pick), dtype=np.int64)
