"""Multi-GPU kernel summation by target sharding (scope row e).

Each V_j depends on all sources but on one target only, so the work splits
into independent target blocks -- the paper's "individual tasks with few
dependencies" (SS I).  One process per GPU:

  1. ``broadcast`` alpha [M,K] and W [M,R] from ``src`` (NCCL over NVLink /
     NVSwitch);
  2. every rank runs ``ks_set_sources`` (a1) locally -- redundant but
     microseconds -- and ``ks_eval`` on its own contiguous target block;
  3. ``all_gather`` of the V blocks (equal-sized, padded to 128) so every rank
     holds V [N,R].

There is no cross-rank sum: per-target arithmetic is the single-GPU one.
torch.distributed is plumbing only; the arithmetic runs in libks.so.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

TILE = 128


def shard_size(N: int, world: int, tile: int = TILE) -> int:
    """Per-rank block: ceil(N / world) rounded up to a multiple of `tile`."""
    if world <= 0:
        raise ValueError("world must be positive")
    per = -(-N // world)
    return -(-per // tile) * tile if per else 0


def shard_bounds(N: int, world: int, rank: int, tile: int = TILE):
    """[lo, hi) target range owned by `rank` (may be empty for trailing ranks)."""
    s = shard_size(N, world, tile)
    lo = min(N, rank * s)
    return lo, min(N, lo + s)


def _all_gather(out_list, local, group):
    backend = dist.get_backend(group)
    if backend == "nccl":
        big = torch.empty((len(out_list) * local.shape[0],) + tuple(local.shape[1:]),
                          dtype=local.dtype, device=local.device)
        dist.all_gather_into_tensor(big, local, group=group)
        return big
    dist.all_gather(out_list, local, group=group)
    return torch.cat(out_list, 0)


def eval_sharded(alpha: torch.Tensor, W: torch.Tensor, beta_local: torch.Tensor, N: int, *,
                 eval_fn, src: int = 0, group=None, broadcast_sources: bool = True) -> torch.Tensor:
    """Target-sharded evaluation; every rank calls it.

    alpha [M,K], W [M,R]: valid on ``src``; same-shaped receive buffers on the
    other ranks (overwritten by the broadcast).  beta_local: this rank's
    target block ``shard_bounds(N, world, rank)``.  ``eval_fn(alpha, W,
    beta_block) -> V_block [n, R]`` is the local evaluation (``KernelSum``
    based in production; tests inject others).  Returns V [N, R] on every rank.
    """
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    if broadcast_sources and world > 1:
        dist.broadcast(alpha, src=src, group=group)
        dist.broadcast(W, src=src, group=group)
    lo, hi = shard_bounds(N, world, rank)
    if beta_local.shape[0] != hi - lo:
        raise ValueError(f"rank {rank}: beta_local has {beta_local.shape[0]} rows, shard is {hi - lo}")
    R = W.shape[1]
    S = shard_size(N, world)
    Vb = torch.zeros((S, R), dtype=torch.float32, device=beta_local.device)
    if hi > lo:
        Vb[: hi - lo] = eval_fn(alpha, W, beta_local)
    if world == 1:
        return Vb[:N]
    parts = [torch.empty_like(Vb) for _ in range(world)]
    return _all_gather(parts, Vb, group)[:N]


class ShardedKernelSum:
    """``KernelSum`` + target sharding over the default process group."""

    def __init__(self, K: int, h: float, precision: str = "auto", group=None):
        from . import KernelSum
        self.plan = KernelSum(K, h, precision)
        self.group = group

    def _local(self, alpha, W, beta_block):
        self.plan.set_sources(alpha, W)
        return self.plan.eval(beta_block)

    def __call__(self, alpha, W, beta_local, N, src=0):
        return eval_sharded(alpha, W, beta_local, N, eval_fn=self._local, src=src, group=self.group)

    def close(self):
        self.plan.close()
