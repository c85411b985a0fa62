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


def _worker(rank, world, port, K, results, compact=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ispass_mehrabilcslo21_b200.sharded import ShardedSpMM
        a = syn.rmat(10, 8, 99, "natural", int_values=True)
        sh = ShardedSpMM(a.M, a.N, a.rowidx, a.colidx, a.value, local_factory=OracleLocal, compact_B=compact)
        sh.permute("nnz_sort")
        B = torch.from_numpy(syn.dense(a.N, K, 5, int_values=True)) if rank == 0 else torch.zeros((a.N, K))
        if compact:
            Bl = sh.distribute_B(B if rank == 0 else None, K=K, src=0)
            assert Bl.shape == (sh.shard.N, K) and sh.shard.N < a.N
            # the compact rows are exactly B[cols_p] and the shard's columns index them
            assert np.array_equal(Bl.numpy(), syn.dense(a.N, K, 5, int_values=True)[sh.cols])
            assert int(sh.shard.colidx.max()) < sh.shard.N
            C_local = sh.run(Bl)
        else:
            sh.broadcast_B(B, src=0)
            C_local = sh.run(B)
        C = sh.allgather_C(C_local)
        ref, _ = oracle.spmm(a, syn.dense(a.N, K, 5, int_values=True))
        if not compact:
            # fused all-gather (f2 ii): each rank stores its rows into "every rank's" full-C buffer at its row
            # offset; here the peers' buffers are local stand-ins, so the disjoint writes are summed over ranks
            bufs = [torch.zeros((a.M, K)) for _ in range(world)]
            sh.run_allgather_fused(B, bufs)
            for b in bufs:
                dist.all_reduce(b)
                assert np.array_equal(b.numpy().astype(np.float64), ref)
        nnz_local = sh.shard.nnz
        results[rank] = (bool(np.array_equal(C.numpy().astype(np.float64), ref)), nnz_local, a.nnz,
                         int(np.diff(a.rowidx).max()), sh.shard.lo, sh.shard.hi)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("compact", [False, True])
@pytest.mark.parametrize("world", [2, 3])
def test_sharded_gloo(world, compact):
    """Partition, shard slicing, B exchange (broadcast, or per-rank compact B rows: SURVEY.md §8(f) f2(i)),
    local SpMM and the C all-gather reassemble the oracle's C exactly (integer-valued inputs)."""
    mgr = mp.Manager()
    results = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(world, port, 8, results, compact), nprocs=world, join=True)
    assert len(results) == world
    lo_hi = sorted((results[r][4], results[r][5]) for r in range(world))
    assert lo_hi[0][0] == 0 and all(lo_hi[i][1] == lo_hi[i + 1][0] for i in range(world - 1))
    for r in range(world):
        ok, nnz_local, nnz, maxrow, _, _ = results[r]
        assert ok, f"rank {r}: reassembled C differs from the oracle"
        assert nnz_local <= -(-nnz // world) + maxrow


def _bench_worker(rank, world, port, compact, results):
    """bench.py's own N>1 input path (rank 0 generates, shards by nnz, optionally compacts the columns) on gloo/CPU."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import bench
        import paper_conf_ispass_mehrabilcslo21_b200 as pkg
        a = syn.rmat(10, 8, 98, "local", int_values=True)
        Mr, lo, (r, c, v), meta, cols, _ = bench.shard_inputs(torch, dist, a if rank == 0 else None, world, rank,
                                                               torch.device("cpu"), pkg, compact=compact)
        r, c, v = r.numpy(), c.numpy(), v.numpy()
        orig_c = cols.numpy()[c] if compact else c
        r0 = a.rowidx[lo]
        ok = (np.array_equal(r, a.rowidx[lo:lo + Mr + 1] - r0) and np.array_equal(orig_c, a.colidx[r0:r0 + len(c)])
              and np.array_equal(v, a.value[r0:r0 + len(v)]))
        if compact:
            ok = ok and np.array_equal(cols.numpy(), np.unique(a.colidx[r0:r0 + len(c)])) and int(meta[rank, 3]) == len(cols)
        results[rank] = (bool(ok), int(Mr), int(a.M))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("compact", [False, True])
def test_bench_shard_inputs_gloo(compact):
    """bench.py --gpus 2 input distribution: shards cover the rows exactly; compact shards index B[cols]."""
    mgr = mp.Manager()
    results = mgr.dict()
    mp.spawn(_bench_worker, args=(2, _free_port(), compact, results), nprocs=2, join=True)
    assert all(results[r][0] for r in range(2)), dict(results)
    assert results[0][1] + results[1][1] == results[0][2]


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
