"""Row-sharded multi-GPU mode (BASELINE.json north star (4)).

One process per GPU (torchrun), torch.distributed for the plumbing:
  1. A is split into contiguous original-order row ranges of about nnz/P non-zeros each
     (spmm_partition_by_nnz, computed identically on every rank -- no communication);
  2. each rank creates and permutes its own shard (spmm_create / spmm_permute run locally);
  3. B is broadcast from `src` (NCCL over NVLink/NVSwitch on GPUs; gloo in the CPU tests);
  4. each rank runs spmm_run on its shard -- C stays row-sharded in original row order;
  5. optionally C is all-gathered (shards padded to the largest shard, gathered, trimmed).

The only data-path collectives are the B broadcast and the optional C all-gather: the SpMM itself
has no exchange step.  `local_factory` builds the per-rank SpMM object; it defaults to the CUDA
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


class ShardedSpMM:
    """C = A.B with A row-sharded across the ranks of `group` (default: the world)."""

    def __init__(self, M, N, rowidx, colidx, value, group=None, local_factory=None, device=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.M, self.N = int(M), int(N)
        self.bounds = partition(np.asarray(rowidx, dtype=np.int64), self.world)
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

    def run(self, B, C_local=None):
        """Local SpMM on this rank's row shard (B resident on every rank). Returns the C shard."""
        return self.local.run(B, C_local)

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
