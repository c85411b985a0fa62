"""Row-sharded mode host logic with torch.distributed gloo on CPU, world_size 2 and 3 (no GPU).

The per-rank SpMM is a CPU stand-in built on the oracle (test-only injection); everything else --
partition by nnz, shard slicing, B broadcast, C all-gather and reassembly in original row order --
is the product code of paper_conf_ispass_mehrabilcslo21_b200.sharded.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synthetic as syn


class OracleLocal:
    """CPU stand-in for the per-rank CUDA SpMM (tests only)."""

    def __init__(self, shard):
        self.csr = syn.CSR(shard.M, shard.N, shard.rowidx, shard.colidx, shard.value)
        self.policy = "identity"

    def permute(self, policy, **kw):
        self.policy = policy
        self.perm = oracle.permute(self.csr, policy, **kw)

    def run(self, B, C=None):
        out, _ = oracle.spmm(self.csr, B.numpy())
        return torch.from_numpy(out.astype(np.float32))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, K, results):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ispass_mehrabilcslo21_b200.sharded import ShardedSpMM
        a = syn.rmat(10, 8, 99, "natural", int_values=True)
        sh = ShardedSpMM(a.M, a.N, a.rowidx, a.colidx, a.value, local_factory=OracleLocal)
        sh.permute("nnz_sort")
        B = torch.from_numpy(syn.dense(a.N, K, 5, int_values=True)) if rank == 0 else torch.zeros((a.N, K))
        sh.broadcast_B(B, src=0)
        C_local = sh.run(B)
        C = sh.allgather_C(C_local)
        ref, _ = oracle.spmm(a, syn.dense(a.N, K, 5, int_values=True))
        nnz_local = sh.shard.nnz
        results[rank] = (bool(np.array_equal(C.numpy().astype(np.float64), ref)), nnz_local, a.nnz,
                         int(np.diff(a.rowidx).max()), sh.shard.lo, sh.shard.hi)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_gloo(world):
    mgr = mp.Manager()
    results = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(world, port, 8, results), nprocs=world, join=True)
    assert len(results) == world
    lo_hi = sorted((results[r][4], results[r][5]) for r in range(world))
    assert lo_hi[0][0] == 0 and all(lo_hi[i][1] == lo_hi[i + 1][0] for i in range(world - 1))
    for r in range(world):
        ok, nnz_local, nnz, maxrow, _, _ = results[r]
        assert ok, f"rank {r}: reassembled C differs from the oracle"
        assert nnz_local <= -(-nnz // world) + maxrow
