"""Target sharding (scope row e) through libks.so on one GPU (the run has one B200):
world-size-2 gloo process groups with both ranks on cuda:0 calling ShardedKernelSum (the
production class: broadcast alpha/W, ks_set_sources + ks_eval on the local target block,
all-gather V), and the same shards evaluated one after the other in one process.  Each
result is compared with the unsharded evaluation and the FP64 oracle.

Not bitwise: a shard has fewer target tiles, so the persistent schedule (which CTA and which
epilogue group sums which source tiles, and where stream-K splits a tile) differs from the
unsharded launch and FP32 partial sums round differently; the difference stays far inside
the 1e-5 bar (SS8)."""
import os
import socket

import numpy as np
import pytest

import workloads
from tests.parity import TOL_3XTF32, e_norm

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402

import paper_conf_icppw_wangkbgj16_b200 as ks  # noqa: E402
from paper_conf_icppw_wangkbgj16_b200.dist import ShardedKernelSum, shard_bounds  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


CASES = [(3, 6000, 3000, "pos", 1), (4, 1500, 700, "signed", 16)]  # (cfg, M, N, W kind, R)


def _inputs(cfg, M, N, wkind):
    return workloads.make(cfg, M=M, N=N, wkind=wkind)


def _worker(rank, world, port, case, outdir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    cfg, M, N, wkind, _ = case
    a, W, b, h = _inputs(cfg, M, N, wkind)
    if rank == 0:
        ta, tw = torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda()
    else:  # receive buffers, garbage contents
        ta, tw = torch.full((M, a.shape[1]), 7.0, device="cuda"), torch.full((M, W.shape[1]), -3.0, device="cuda")
    lo, hi = shard_bounds(N, world, rank)
    tb = torch.from_numpy(b[lo:hi].copy()).cuda()
    sk = ShardedKernelSum(a.shape[1], float(h))
    V = sk(ta, tw, tb, N)
    torch.cuda.synchronize()
    np.save(os.path.join(outdir, f"V{rank}.npy"), V.cpu().numpy())
    sk.close()
    dist.destroy_process_group()


def _unsharded(a, W, b, h):
    with ks.KernelSum(a.shape[1], float(h)) as plan:
        plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
        V = plan.eval(torch.from_numpy(b).cuda())
        torch.cuda.synchronize()
        return V.cpu().numpy().astype(np.float64)


@pytest.mark.parametrize("case", CASES)
def test_two_gloo_ranks_on_one_gpu(tmp_path, oracle_mod, case):
    mp.spawn(_worker, args=(2, _free_port(), case, str(tmp_path)), nprocs=2, join=True)
    cfg, M, N, wkind, R = case
    a, W, b, h = _inputs(cfg, M, N, wkind)
    ref = oracle_mod.oracle_eval(a, W, b, float(h))
    V1 = _unsharded(a, W, b, h)
    for r in range(2):
        V = np.load(tmp_path / f"V{r}.npy").astype(np.float64)
        assert V.shape == (N, R)
        assert e_norm(V, ref, W) <= TOL_3XTF32
        assert np.max(np.abs(V - V1)) / np.abs(W).sum() <= 1e-6


@pytest.mark.parametrize("world", [2, 3, 8])
def test_sequential_shards_through_libks(oracle_mod, world):
    """Each rank's block evaluated in turn (what rank r computes), concatenated."""
    a, W, b, h = workloads.make(3, M=5000, N=2100, wkind="pos")
    N = b.shape[0]
    parts = []
    with ks.KernelSum(a.shape[1], float(h)) as plan:
        plan.set_sources(torch.from_numpy(a).cuda(), torch.from_numpy(W).cuda())
        for r in range(world):
            lo, hi = shard_bounds(N, world, r)
            if hi > lo:
                parts.append(plan.eval(torch.from_numpy(b[lo:hi].copy()).cuda()).cpu().numpy())
    V = np.concatenate(parts).astype(np.float64)
    ref = oracle_mod.oracle_eval(a, W, b, float(h))
    assert e_norm(V, ref, W) <= TOL_3XTF32
    assert np.max(np.abs(V - _unsharded(a, W, b, h))) / np.abs(W).sum() <= 1e-6
