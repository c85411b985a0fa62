"""Row-sharded multi-GPU mode (BASELINE.json north star (4)).

One process per GPU (torchrun), torch.distributed for the plumbing:
  1. A is split into contiguous original-order row ranges of about nnz/P non-zeros each
     (spmm_partition_by_nnz, computed identically on every rank -- no communication);
  2. each rank creates and permutes its own shard (spmm_create / spmm_permute run locally);
  3. B is broadcast from `src` (NCCL over NVLink/NVSwitch on GPUs; gloo in the CPU tests);
  4. each rank runs spmm_run on its shard -- C stays row-sharded in original row order;
  5. optionally C is all-gathered (shards padded to the largest shard, gathered, trimmed).

With compact_B=True a rank holds only the B rows its shard touches: the shard's
columns are renumbered to their rank in the sorted list cols_p of distinct columns it references (a
monotone map, so every row keeps its ascending column order and C is bit-identical), and `distribute_B`
sends each rank B[cols_p] from the source (NCCL point-to-point) instead of broadcasting all N rows --
|cols_p| / N of the volume, and a B working set that shrinks with P.

The only data-path collectives are the B broadcast (or the per-rank B-row sends) and the optional C
all-gather: the SpMM itself has no exchange step.  `local_factory` builds the per-rank SpMM object; it defaults to the CUDA
library (paper_conf_ispass_mehrabilcslo21_b200.SpMM).  Tests inject a CPU stand-in so the host logic
(partition, shard slicing, broadcast, reassembly) is checked with gloo on CPU.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class Shard:
    lo: int              # first original row of this shard
    hi: int              # one past the last
    M: int
    N: int
    rowidx: np.ndarray   # int64[M+1], rebased to 0
    colidx: np.ndarray
    value: np.ndarray

    @property
    def nnz(self) -> int:
        return int(self.rowidx[-1]) if self.M else 0


def partition(rowidx: np.ndarray, P: int) -> np.ndarray:
    from . import spmm_partition_by_nnz
    return spmm_partition_by_nnz(rowidx, P)


def make_shard(M: int, N: int, rowidx, colidx, value, bounds, rank: int) -> Shard:
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    r0, r1 = int(rowidx[lo]), int(rowidx[hi])
    return Shard(lo, hi, hi - lo, N, np.asarray(rowidx[lo:hi + 1], dtype=np.int64) - r0,
                 np.asarray(colidx[r0:r1], dtype=np.int32), np.asarray(value[r0:r1], dtype=np.float32))


def shard_columns(rowidx, colidx, bounds, rank: int) -> np.ndarray:
    """Sorted distinct columns referenced by shard `rank` (int64)."""
    lo, hi = int(bounds[rank]), int(bounds[rank + 1])
    r0, r1 = int(rowidx[lo]), int(rowidx[hi])
    return np.unique(np.asarray(colidx[r0:r1], dtype=np.int64))


def compact_shard(sh: Shard, cols: np.ndarray) -> Shard:
    """Renumber the shard's columns to their index in `cols` (monotone: row order of columns preserved)."""
    cc = np.searchsorted(cols, sh.colidx).astype(np.int32)
    return Shard(sh.lo, sh.hi, sh.M, int(len(cols)), sh.rowidx, cc, sh.value)


class ShardedSpMM:
    """C = A.B with A row-sharded across the ranks of `group` (default: the world)."""

    def __init__(self, M, N, rowidx, colidx, value, group=None, local_factory=None, device=None, compact_B=False):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.M, self.N = int(M), int(N)
        self.bounds = partition(np.asarray(rowidx, dtype=np.int64), self.world)
        self.compact_B = bool(compact_B)
        self.cols = None
        if self.compact_B:
            # every rank holds the full CSR here, so every rank can derive every shard's column list
            self.cols_all = [shard_columns(rowidx, colidx, self.bounds, p) for p in range(self.world)]
            self.cols = self.cols_all[self.rank]
            self.shard = compact_shard(make_shard(M, N, rowidx, colidx, value, self.bounds, self.rank), self.cols)
        else:
            self.shard = make_shard(M, N, rowidx, colidx, value, self.bounds, self.rank)
        self.device = device
        if local_factory is None:
            from . import SpMM
            local_factory = lambda s: SpMM(s.M, s.N, s.rowidx, s.colidx, s.value)  # noqa: E731
        self.local = local_factory(self.shard)

    def permute(self, policy, **params):
        self.local.permute(policy, **params)
        return self

    def broadcast_B(self, B, src: int = 0):
        """B must be allocated (N x K) on every rank; rank `src` holds the values."""
        self.dist.broadcast(B, src=src, group=self.group)
        return B

    def distribute_B(self, B, K=None, src: int = 0, dtype=None, device=None):
        """compact_B: rank `src` passes the full B (N x K); every rank returns its compact B_p = B[cols_p]
        (|cols_p| x K), sent point-to-point from `src`.  Other ranks may pass B=None (give K)."""
        import torch
        assert self.compact_B, "distribute_B needs compact_B=True (else use broadcast_B)"
        if self.rank == src:
            K = B.shape[1]
            reqs = []
            for p in range(self.world):
                if p == src:
                    continue
                idx = torch.from_numpy(self.cols_all[p]).to(B.device)
                reqs.append(self.dist.isend(B.index_select(0, idx).contiguous(),
                                            dst=self.dist.get_global_rank(self.group, p) if self.group else p,
                                            group=self.group))
            mine = B.index_select(0, torch.from_numpy(self.cols).to(B.device)).contiguous()
            for r in reqs:
                r.wait()
            return mine
        mine = torch.empty((len(self.cols), int(K)), dtype=dtype or torch.float32, device=device)
        self.dist.recv(mine, src=self.dist.get_global_rank(self.group, src) if self.group else src, group=self.group)
        return mine

    def run(self, B, C_local=None):
        """Local SpMM on this rank's row shard (B resident on every rank). Returns the C shard."""
        return self.local.run(B, C_local)

    def symmetric_C(self, K, dtype=None):
        """A full-C buffer [M, K] in torch symmetric memory on this rank, plus every rank's view of it as device
        pointers (the destinations for run_allgather_fused; peer addresses are NVLink-mapped on an NVSwitch
        node).  Needs an NCCL process group."""
        import torch
        import torch.distributed._symmetric_memory as symm_mem
        buf = symm_mem.empty((self.M, int(K)), dtype=dtype or torch.float32, device=torch.device("cuda"))
        grp = self.group if self.group is not None else self.dist.group.WORLD
        hdl = symm_mem.rendezvous(buf, grp.group_name)
        return buf, [int(p) for p in hdl.buffer_ptrs], hdl

    def run_allgather_fused(self, B, C_bufs, stream=None):
        """the C all-gather fused into the SpMM epilogue.  This rank's SpMM stores its C rows
        straight into every rank's full-C buffer (C_bufs[p]: cuda tensors [M, K] or device pointers addressable
        from this GPU -- on an NVLink/NVSwitch node the peer views of a torch symmetric-memory allocation), at its
        shard's row offset (spmm_run_to); no separate collective.  Every rank calls it; each buffer holds the
        full C once all ranks' kernels are done (the caller's barrier)."""
        self.local.run_to(B, C_bufs, row_offset=int(self.bounds[self.rank]), stream=stream)
        return C_bufs

    def allgather_C(self, C_local):
        """Reassemble the full C (original row order) on every rank."""
        import torch
        counts = [int(self.bounds[p + 1] - self.bounds[p]) for p in range(self.world)]
        mx = max(counts) if counts else 0
        K = C_local.shape[1]
        pad = torch.zeros((mx, K), dtype=C_local.dtype, device=C_local.device)
        pad[: C_local.shape[0]] = C_local
        parts = [torch.empty_like(pad) for _ in range(self.world)]
        self.dist.all_gather(parts, pad, group=self.group)
        return torch.cat([parts[p][: counts[p]] for p in range(self.world)], dim=0)

    def close(self):
        close = getattr(self.local, "close", None)
        if close:
            close()
