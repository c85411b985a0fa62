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
        self.csr = syn.CSR(shard.M, shard.N, np.asarray(shard.rowidx), np.asarray(shard.colidx),
                           np.asarray(shard.value))
        self.policy = "identity"

    def permute(self, policy, **kw):
        self.policy = policy
        self.perm = oracle.permute(self.csr, policy, **kw)

    def run(self, B, C=None):
        out, _ = oracle.spmm(self.csr, B.numpy())
        return torch.from_numpy(out.astype(np.float32))

    def run_ld(self, B, C, col_offset=0):
        """spmm_run_ld semantics: C[:, col_offset:col_offset + K] = A.B, other columns untouched."""
        C[:, col_offset:col_offset + B.shape[1]] = self.run(B)
        return C

    def run_to(self, B, dsts, row_offset=0, stream=None):
        """spmm_run_to semantics: this shard's rows stored into every destination at row_offset + r."""
        out = self.run(B)
        for d in dsts:
            d[row_offset:row_offset + out.shape[0]] = out
        return dsts


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _worker(rank, world, port, K, results, compact, how):
    _init(rank, world, port)
    try:
        from paper_conf_ispass_mehrabilcslo21_b200.sharded import ShardedSpMM
        a = syn.rmat(10, 8, 99, "natural", int_values=True)
        if how == "scatter":      # rank 0 alone holds the matrix
            sh = ShardedSpMM.scatter(a if rank == 0 else None, src=0, compact_B=compact, local_factory=OracleLocal)
        else:
            sh = ShardedSpMM.from_full(a.M, a.N, a.rowidx, a.colidx, a.value, local_factory=OracleLocal,
                                       compact_B=compact)
        assert (sh.M, sh.N) == (a.M, a.N)
        sh.permute("nnz_sort")
        Bfull = syn.dense(a.N, K, 5, int_values=True)
        B = torch.from_numpy(Bfull) if rank == 0 else torch.zeros((a.N, K))
        ref, _ = oracle.spmm(a, Bfull)
        lo, hi = sh.shard.lo, sh.shard.hi
        # the shard is exactly this rank's rows (columns through cols_p when compact)
        r0 = a.rowidx[lo]
        cc = np.asarray(sh.shard.colidx)
        ok_shard = (np.array_equal(np.asarray(sh.shard.rowidx), a.rowidx[lo:hi + 1] - r0)
                    and np.array_equal(np.asarray(sh.cols)[cc] if compact else cc, a.colidx[r0:r0 + len(cc)]))
        if compact:
            Bl = sh.distribute_B(B if rank == 0 else None, K=K, src=0)
            assert Bl.shape == (sh.shard.N, K) and sh.shard.N < a.N
            assert np.array_equal(Bl.numpy(), Bfull[np.asarray(sh.cols)])
            assert int(cc.max()) < sh.shard.N
            C_local = sh.run(Bl)
            # B arriving row-sharded (rank q owns B[bo[q]:bo[q+1]]): one all-to-allv delivers exactly B[cols_p]
            bo = sh.b_owner_bounds()
            Ba = sh.exchange_B_alltoall(torch.from_numpy(Bfull[bo[rank]:bo[rank + 1]]))
            assert torch.equal(Ba, Bl)
            Ba2 = sh.exchange_B_alltoall(torch.from_numpy(Bfull[bo[rank]:bo[rank + 1]]) * 2)   # reuses the setup
            assert torch.equal(Ba2, Bl * 2)
            # f2 (iii): B in column chunks, each chunk's SpMM into its C columns as it arrives
            for chunks in (1, 3, 4):
                Cp = torch.full((sh.shard.M, K), float("nan"))
                sh.run_pipelined(B if rank == 0 else None, K=K, chunks=chunks, C_local=Cp, src=0)
                assert torch.equal(Cp, C_local), chunks
        else:
            sh.broadcast_B(B, src=0)
            C_local = sh.run(B)
        C = sh.allgather_C(C_local)
        if not compact:
            # fused all-gather (f2 ii): each rank stores its rows into "every rank's" full-C buffer at its row
            # offset; here the peers' buffers are local stand-ins, so the disjoint writes are summed over ranks
            bufs = [torch.zeros((a.M, K)) for _ in range(world)]
            sh.run_allgather_fused(B, bufs)
            for b in bufs:
                dist.all_reduce(b)
                assert np.array_equal(b.numpy().astype(np.float64), ref)
        results[rank] = (bool(np.array_equal(C.numpy().astype(np.float64), ref)) and ok_shard, sh.shard.nnz, a.nnz,
                         int(np.diff(a.rowidx).max()), lo, hi)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("how", ["scatter", "full"])
@pytest.mark.parametrize("compact", [False, True])
@pytest.mark.parametrize("world", [2, 3, 4])
def test_sharded_gloo(world, compact, how):
    """Partition, shard scatter from rank 0 (or local slicing when every rank holds A), B exchange (broadcast, or
    per-rank compact B rows: SURVEY.md §8(f) f2(i)), the column-chunk pipeline (f2 iii), local SpMM and the C
    all-gather reassemble the oracle's C exactly (integer-valued inputs)."""
    mgr = mp.Manager()
    results = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(world, port, 24, results, compact, how), nprocs=world, join=True)
    assert len(results) == world
    lo_hi = sorted((results[r][4], results[r][5]) for r in range(world))
    assert lo_hi[0][0] == 0 and all(lo_hi[i][1] == lo_hi[i + 1][0] for i in range(world - 1))
    for r in range(world):
        ok, nnz_local, nnz, maxrow, _, _ = results[r]
        assert ok, f"rank {r}: shard or reassembled C differs from the oracle"
        assert nnz_local <= -(-nnz // world) + maxrow


def test_chunk_bounds():
    from paper_conf_ispass_mehrabilcslo21_b200.sharded import chunk_bounds
    assert chunk_bounds(128, 4) == [(0, 32), (32, 64), (64, 96), (96, 128)]
    assert chunk_bounds(24, 3) == [(0, 8), (8, 16), (16, 24)]
    assert chunk_bounds(64, 1) == [(0, 64)]
    for K in (8, 24, 64, 72, 128, 256):
        for c in (1, 2, 3, 4, 5, 16):
            cb = chunk_bounds(K, c)
            assert cb[0][0] == 0 and cb[-1][1] == K and all(x[1] == y[0] for x, y in zip(cb, cb[1:]))
            assert all(c0 % 8 == 0 for c0, _ in cb) and len(cb) <= c


def test_bench_reference_arm_torchrun():
    """bench.py --impl reference under torchrun N=2 (CPU): rank 0 alone times the oracle and prints ONE JSON
    line with impl/cpu_baseline/e2e; the other rank exits 0 without work."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(root, "bench.py"), "--impl", "reference", "--config", "c1",
           "--gpus", "2", "--steps", "2", "--warmup", "3"]
    out = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2 and d["steps"] == 2 and d["warmup"] == 3
    assert d["value"] > 0 and d["unit"] == "GFLOP/s" and d["higher_is_better"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": d["unit"], "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    # torchrun exports OMP_NUM_THREADS=1; the oracle must still run on every core of the affinity set
    assert d["cpu_baseline"]["cores"] == len(os.sched_getaffinity(0))
