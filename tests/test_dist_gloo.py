"""Multi-process (world_size 2, gloo, CPU) tests of the target-sharding host
logic in paper_conf_icppw_wangkbgj16_b200/dist.py.  The local evaluation is
injected (the FP64 oracle here, test infrastructure), so these run without a
GPU; on a GPU box the same code path calls libks.so."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icppw_wangkbgj16_b200.dist import eval_sharded, shard_bounds, shard_size


def test_shard_bounds_cover_exactly():
    for N in (0, 1, 127, 128, 129, 1000, 65536, 65537):
        for P in (1, 2, 3, 4, 8):
            covered = []
            for r in range(P):
                lo, hi = shard_bounds(N, P, r)
                assert 0 <= lo <= hi <= N
                assert (hi - lo) <= shard_size(N, P)
                if hi > lo:
                    assert lo % 128 == 0
                covered.extend(range(lo, hi))
            assert covered == list(range(N))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, N, M, K, R, h, outdir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import workloads
    a, W, b, _ = workloads.custom(M, N, K, R, h, seed=5, wkind="signed")
    if rank == 0:
        ta, tw = torch.from_numpy(a), torch.from_numpy(W)
    else:  # receive buffers, garbage contents
        ta, tw = torch.full((M, K), 7.0), torch.full((M, R), -3.0)
    lo, hi = shard_bounds(N, world, rank)
    tb = torch.from_numpy(b[lo:hi].copy())

    def local(alpha, Wt, beta_blk):
        return torch.from_numpy(oracle.oracle_eval(alpha.numpy(), Wt.numpy(), beta_blk.numpy(), h)).float()

    V = eval_sharded(ta, tw, tb, N, eval_fn=local)
    np.save(os.path.join(outdir, f"V{rank}.npy"), V.numpy())
    dist.destroy_process_group()


@pytest.mark.parametrize("N", [300, 129, 1])
def test_two_rank_sharded_matches_single(tmp_path, N, oracle_mod):
    import workloads
    M, K, R, h = 257, 5, 2, 0.6
    mp.spawn(_worker, args=(2, _free_port(), N, M, K, R, h, str(tmp_path)), nprocs=2, join=True)
    a, W, b, _ = workloads.custom(M, N, K, R, h, seed=5, wkind="signed")
    ref = oracle_mod.oracle_eval(a, W, b, h).astype(np.float32)
    for r in range(2):
        V = np.load(tmp_path / f"V{r}.npy")
        assert V.shape == (N, R)
        assert np.array_equal(V, ref), r   # no cross-rank arithmetic: bitwise
