"""Row-sharded multi-GPU mode (BASELINE.json north star (4)).

One process per GPU (torchrun), torch.distributed for the plumbing:
  1. rank `src` holds the matrix; it splits A into contiguous original-order row ranges of about nnz/P
     non-zeros each (spmm_partition_by_nnz) and sends every rank ITS shard only (ShardedSpMM.scatter: NCCL
     point-to-point of device tensors over NVLink / NVSwitch; host tensors under gloo) -- no rank ever holds
     another rank's rows;
  2. each rank creates and permutes its own shard (spmm_create / spmm_permute run locally);
  3. B exchange (compact_B, f2 i): a rank holds only the B rows its shard references -- the shard's columns are
     renumbered to their index in its sorted distinct-column list cols_p (a monotone map: every row keeps its
     ascending column order, so C is bit-identical) and `src` sends each rank B[cols_p] (|cols_p| / N of a
     broadcast); when B arrives row-sharded (each rank owns N/P rows), exchange_B_alltoall moves exactly those rows
     in ONE all-to-allv in which every rank sends and receives at once; compact_B=False keeps the plain NCCL
     broadcast of all N rows;
  4. each rank runs spmm_run on its shard -- C stays row-sharded in original row order;
  5. optionally C is all-gathered: NCCL all_gather (allgather_C), or fused into the SpMM epilogue -- per-peer
     stores into every rank's symmetric-memory buffer (run_allgather_fused, spmm_run_to) or one NVLS multicast
     store per element (run_allgather_multicast, spmm_run_multicast, multimem.st).
f2 iii, B chunks pipelined with compute (run_pipelined): B[cols_p] is sent in column chunks; each rank runs the
SpMM of chunk c (spmm_run_ld into C's columns of that chunk) as soon as chunk c has arrived, while chunk c + 1 is
still in flight.

The only data-path communication is the B exchange and the optional C all-gather: the SpMM itself has no
exchange step.  `local_factory` builds the per-rank SpMM object; it defaults to the CUDA library
(paper_conf_ispass_mehrabilcslo21_b200.SpMM).  Tests inject a CPU stand-in so the host logic (partition, shard
scatter, B exchange, chunk pipeline, reassembly) is checked with gloo on CPU.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class Shard:
    lo: int              # first original row of this shard
    hi: int              # one past the last
    M: int
    N: int               # columns of the shard's matrix (= |cols_p| when compacted)
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


def chunk_bounds(K: int, chunks: int, align: int = 8):
    """Column chunks [c0, c1) of K for the pipelined B exchange: `chunks` nearly equal pieces, each a multiple of
    `align` columns (256-bit lane loads and 32-byte aligned C column blocks), the last one taking the rest."""
    chunks = max(1, min(int(chunks), K // align if K >= align else 1))
    step = max(align, (K // chunks) // align * align)
    cuts = [min(K, c * step) for c in range(chunks)] + [K]
    return [(cuts[c], cuts[c + 1]) for c in range(chunks) if cuts[c + 1] > cuts[c]]


class _Comm:
    """Point-to-point / collective plumbing: device tensors under NCCL, host tensors under gloo."""

    def __init__(self, dist, group):
        self.dist, self.group = dist, group
        self.nccl = dist.get_backend(group) == "nccl"

    def g(self, p):   # group rank -> global rank
        return self.dist.get_global_rank(self.group, p) if self.group is not None else p

    def wire(self, t):
        return t if self.nccl else t.cpu()

    def send(self, t, dst):
        self.dist.send(self.wire(t).contiguous(), dst=self.g(dst), group=self.group)

    def isend(self, t, dst):
        w = self.wire(t).contiguous()
        return self.dist.isend(w, dst=self.g(dst), group=self.group), w

    def recv(self, t, src):
        if self.nccl:
            self.dist.recv(t, src=self.g(src), group=self.group)
        else:
            import torch
            h = torch.empty(t.shape, dtype=t.dtype)
            self.dist.recv(h, src=self.g(src), group=self.group)
            t.copy_(h)

    def broadcast(self, t, src):
        if self.nccl:
            self.dist.broadcast(t, src=self.g(src), group=self.group)
        else:
            h = t.cpu()
            self.dist.broadcast(h, src=self.g(src), group=self.group)
            t.copy_(h)


class ShardedSpMM:
    """C = A.B with A row-sharded across the ranks of `group` (default: the world).  Build with scatter() (one
    rank holds the matrix) or from_full() (every rank holds it: shards derived locally, no communication)."""

    def __init__(self, shard: Shard, bounds, M: int, N: int, cols=None, cols_all=None, group=None, local_factory=None,
                 device=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.comm = _Comm(dist, group)
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.M, self.N = int(M), int(N)
        self.bounds = np.asarray(bounds, dtype=np.int64)
        self.shard = shard
        self.cols = cols                  # this rank's distinct columns (compact_B), else None
        self.cols_all = cols_all          # every rank's columns -- on the source rank only
        self.compact_B = cols is not None
        self.device = device
        if local_factory is None:
            from . import SpMM
            local_factory = lambda s: SpMM(s.M, s.N, s.rowidx, s.colidx, s.value)  # noqa: E731
        self.local = local_factory(self.shard)

    # ---- construction ----------------------------------------------------------------------------------------
    @classmethod
    def scatter(cls, csr=None, src: int = 0, group=None, compact_B: bool = True, device=None, local_factory=None):
        """Rank `src` passes the full CSR (host arrays; M, N, rowidx, colidx, value attributes), the others None.
        `src` partitions by nnz and sends every rank its own shard (rowidx, colidx, value and, with compact_B, its
        column list); nothing else crosses ranks."""
        import torch
        import torch.distributed as dist
        comm = _Comm(dist, group)
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                                 if comm.nccl else torch.device("cpu"))
        if rank == src:
            bounds = partition(np.asarray(csr.rowidx, dtype=np.int64), world)
            cols_all = [shard_columns(csr.rowidx, csr.colidx, bounds, p) for p in range(world)] if compact_B else None
            shards = []
            for p in range(world):
                sh = make_shard(csr.M, csr.N, csr.rowidx, csr.colidx, csr.value, bounds, p)
                shards.append(compact_shard(sh, cols_all[p]) if compact_B else sh)
            meta = torch.tensor([[csr.M, csr.N, world, 0]] + [[s.M, s.nnz, s.N, 0] for s in shards],
                                dtype=torch.int64, device=dev)
            bt = torch.from_numpy(np.asarray(bounds, dtype=np.int64)).to(dev)
        else:
            meta = torch.empty((world + 1, 4), dtype=torch.int64, device=dev)
            bt = torch.empty(world + 1, dtype=torch.int64, device=dev)
        if world > 1:
            comm.broadcast(meta, src)
            comm.broadcast(bt, src)
        M, N = int(meta[0, 0]), int(meta[0, 1])
        bounds = bt.cpu().numpy()
        if rank == src:
            for p in range(world):
                if p == src:
                    continue
                parts = [shards[p].rowidx, shards[p].colidx, shards[p].value] + ([cols_all[p]] if compact_B else [])
                for a in parts:
                    comm.send(torch.from_numpy(np.ascontiguousarray(a)).to(dev), p)
            mine, cols = shards[src], (cols_all[src] if compact_B else None)
        else:
            Mr, nnzr, Nr = int(meta[rank + 1, 0]), int(meta[rank + 1, 1]), int(meta[rank + 1, 2])
            bufs = [torch.empty(Mr + 1, dtype=torch.int64, device=dev), torch.empty(nnzr, dtype=torch.int32, device=dev),
                    torch.empty(nnzr, dtype=torch.float32, device=dev)]
            if compact_B:
                bufs.append(torch.empty(Nr, dtype=torch.int64, device=dev))
            for b in bufs:
                comm.recv(b, src)
            # NCCL: the shard stays on the device (spmm_create copies device arrays, no host round trip)
            arrs = bufs if (comm.nccl or dev.type == "cuda") else [b.numpy() for b in bufs]
            lo, hi = int(bounds[rank]), int(bounds[rank + 1])
            mine = Shard(lo, hi, Mr, Nr if compact_B else N, arrs[0], arrs[1], arrs[2])
            cols, cols_all = (arrs[3] if compact_B else None), None
        return cls(mine, bounds, M, N, cols=cols, cols_all=cols_all if rank == src else None, group=group,
                   local_factory=local_factory, device=device)

    @classmethod
    def from_full(cls, M, N, rowidx, colidx, value, group=None, compact_B=False, local_factory=None, device=None):
        """Every rank holds the full CSR: each derives its own shard (and, with compact_B, every rank's column list,
        so any rank can serve distribute_B) without communication."""
        import torch.distributed as dist
        world, rank = dist.get_world_size(group), dist.get_rank(group)
        bounds = partition(np.asarray(rowidx, dtype=np.int64), world)
        sh = make_shard(M, N, rowidx, colidx, value, bounds, rank)
        cols_all = [shard_columns(rowidx, colidx, bounds, p) for p in range(world)] if compact_B else None
        if compact_B:
            sh = compact_shard(sh, cols_all[rank])
        return cls(sh, bounds, M, N, cols=cols_all[rank] if compact_B else None, cols_all=cols_all, group=group,
                   local_factory=local_factory, device=device)

    # ---- per-rank work ---------------------------------------------------------------------------------------
    def permute(self, policy, **params):
        self.local.permute(policy, **params)
        return self

    @property
    def row_offset(self) -> int:
        return int(self.bounds[self.rank])

    def broadcast_B(self, B, src: int = 0):
        """B must be allocated (N x K) on every rank; rank `src` holds the values."""
        self.comm.broadcast(B, src)
        return B

    def _my_rows(self, B, p):
        import torch
        return B.index_select(0, torch.from_numpy(self.cols_all[p]).to(B.device))

    def distribute_B(self, B, K=None, src: int = 0, dtype=None, device=None):
        """compact_B: rank `src` passes the full B (N x K); every rank returns its compact B_p = B[cols_p]
        (|cols_p| x K), sent point-to-point from `src`.  Other ranks may pass B=None (give K)."""
        import torch
        assert self.compact_B, "distribute_B needs compact_B=True (else use broadcast_B)"
        if self.rank == src:
            assert self.cols_all is not None, "the source rank needs every shard's column list (scatter / from_full)"
            reqs = [self.comm.isend(self._my_rows(B, p), p) for p in range(self.world) if p != src]
            mine = self._my_rows(B, src).contiguous()
            for r, _keep in reqs:
                r.wait()
            return mine
        mine = torch.empty((len(self.cols), int(K)), dtype=dtype or torch.float32, device=device)
        self.comm.recv(mine, src)
        return mine

    # ---- B arriving row-sharded: all-to-allv of exactly the rows each shard references ----------------------------
    def b_owner_bounds(self):
        """Row ranges of B owned by the ranks when B arrives row-sharded: rank q holds B[b_lo[q]:b_lo[q + 1]]
        (equal splits of N)."""
        return np.array([(q * self.N) // self.world for q in range(self.world + 1)], dtype=np.int64)

    def setup_alltoall(self, device=None):
        """Once per sharding (structure only): every rank tells every owner which of its B rows it needs (its sorted
        columns cols_p cut at the owner boundaries), so that exchange_B_alltoall moves exactly B[cols_p]."""
        import torch
        assert self.compact_B, "the all-to-all exchange needs compact_B=True"
        dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                                 if self.comm.nccl else torch.device("cpu"))
        bo = self.b_owner_bounds()
        cols = torch.as_tensor(self.cols).to(dev).long()
        cuts = torch.searchsorted(cols, torch.from_numpy(bo).to(dev))
        need = (cuts[1:] - cuts[:-1]).to(torch.int64)           # rows I need from each owner q
        give = torch.empty_like(need)                              # rows each rank p needs from me
        self.dist.all_to_all_single(give, need, group=self.group)
        self._a2a_need = [int(x) for x in need.cpu().tolist()]
        self._a2a_give = [int(x) for x in give.cpu().tolist()]
        req = torch.empty(sum(self._a2a_give), dtype=torch.int64, device=dev)
        self.dist.all_to_all_single(req, cols, output_split_sizes=self._a2a_give, input_split_sizes=self._a2a_need,
                                    group=self.group)
        self._a2a_rows = req - int(bo[self.rank])                  # local row ids of my B slice, per requester
        self._a2a_dev = dev
        return self

    def exchange_B_alltoall(self, B_slice, K=None):
        """f2 (i) when B arrives row-sharded (rank q holds B_slice = B[b_lo[q]:b_lo[q + 1]], [n_q, K]): one
        all-to-allv in which every owner sends each rank exactly the rows of its slice that the rank's shard
        references.  Every rank sends and receives at once (aggregate NVLink bandwidth instead of one source's
        link); the result is this rank's compact B_p = B[cols_p] (|cols_p| x K, sorted by column: owners are
        ordered by row range).  setup_alltoall() first."""
        import torch
        if not hasattr(self, "_a2a_rows"):
            self.setup_alltoall(B_slice.device)
        K = int(B_slice.shape[1]) if K is None else int(K)
        send = B_slice.index_select(0, self._a2a_rows.to(B_slice.device)) if len(self._a2a_rows) else \
            torch.empty((0, K), dtype=B_slice.dtype, device=B_slice.device)
        out = torch.empty((sum(self._a2a_need), K), dtype=B_slice.dtype, device=B_slice.device)
        self.dist.all_to_all_single(out, send, output_split_sizes=self._a2a_need, input_split_sizes=self._a2a_give,
                                    group=self.group)
        return out

    def run(self, B, C_local=None):
        """Local SpMM on this rank's row shard (B resident on every rank). Returns the C shard."""
        return self.local.run(B, C_local)

    def run_pipelined(self, B=None, K=None, chunks=None, C_local=None, src: int = 0, device=None):
        """f2 (iii): the compact B exchange and the SpMM pipelined over column chunks of B.  `src` sends each rank
        B[cols_p][:, c0:c1] chunk by chunk (all sends posted at once); a rank runs the SpMM of chunk c (spmm_run_ld
        into C_local[:, c0:c1]) as soon as chunk c has arrived -- under NCCL the wait is a stream dependency, so the
        SpMM of chunk c overlaps the transfer of chunk c + 1.  Returns this rank's C shard [M_p, K].
        chunks=None: K // 64 chunks of 64 columns -- the lane geometry of K = 64 has the rows per warp task of
        K = 128 / 256, so split rows are cut into the same chunks and C is bit-identical to spmm_run's; other chunk
        widths change the split-row summation order (C within the north-star tolerance)."""
        import torch
        assert self.compact_B, "run_pipelined needs compact_B=True"
        if self.rank == src:
            K = int(B.shape[1])
        K = int(K)
        cb = chunk_bounds(K, chunks if chunks is not None else max(1, K // 64))
        if C_local is None:
            if device is None:
                device = B.device if B is not None else (torch.device("cuda", torch.cuda.current_device())
                                                         if self.comm.nccl else torch.device("cpu"))
            C_local = torch.empty((self.shard.M, K), dtype=torch.float32, device=device)
        if self.rank == src:
            keep = []
            for p in range(self.world):
                if p == src:
                    continue
                rows = self._my_rows(B, p)
                for c0, c1 in cb:
                    keep.append(self.comm.isend(rows[:, c0:c1], p))
            mine = self._my_rows(B, src)
            for c0, c1 in cb:
                self.local.run_ld(mine[:, c0:c1].contiguous(), C_local, col_offset=c0)
            for r, _k in keep:
                r.wait()
            return C_local
        bufs = [torch.empty((len(self.cols), c1 - c0), dtype=torch.float32, device=C_local.device) for c0, c1 in cb]
        if self.comm.nccl:
            reqs = [self.dist.irecv(b, src=self.comm.g(src), group=self.group) for b in bufs]
            for (c0, _c1), b, r in zip(cb, bufs, reqs):
                r.wait()                       # NCCL: the current stream waits for chunk c, the host does not
                self.local.run_ld(b, C_local, col_offset=c0)
        else:
            for (c0, _c1), b in zip(cb, bufs):
                self.comm.recv(b, src)
                self.local.run_ld(b, C_local, col_offset=c0)
        return C_local

    # ---- C all-gather ----------------------------------------------------------------------------------------
    def symmetric_C(self, K, dtype=None):
        """A full-C buffer [M, K] in torch symmetric memory on this rank, plus every rank's view of it as device
        pointers (the destinations for run_allgather_fused; peer addresses are NVLink-mapped on an NVSwitch node)
        and the rendezvous handle (handle.multicast_ptr: the NVLS multicast address, 0 where unsupported).  Needs an
        NCCL process group."""
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
        self.local.run_to(B, C_bufs, row_offset=self.row_offset, stream=stream)
        return C_bufs

    def run_allgather_multicast(self, B, mc_ptr: int, stream=None):
        """f2 (ii) with NVLS: one multimem.st per C element to the multicast address of the group's symmetric
        full-C buffer (symmetric_C()[2].multicast_ptr); the NVSwitch delivers it to every rank's buffer."""
        self.local.run_multicast(B, int(mc_ptr), row_offset=self.row_offset, stream=stream)

    def allgather_C(self, C_local):
        """Reassemble the full C (original row order) on every rank (NCCL all_gather of padded shards)."""
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
