"""spmm_run_to (SURVEY §8(f) f2 ii): the C all-gather fused into the SpMM epilogue -- every C row a handle computes is
stored to n destination buffers at a row offset.  On one GPU the destinations are local buffers standing in for
the peers' (the kernel's stores do not depend on where the pointers map).  Checks: every destination equals the
plain spmm_run result bit for bit (whole rows, row-fusion records, long-row combine and empty-row zero fill all
write every destination); two nnz-balanced shards writing into shared full-size buffers at their row offsets
reassemble the unsharded C bit for bit and match the oracle; rows outside the shard are untouched; argument
errors."""
import numpy as np
import pytest

import oracle
import synthetic as syn

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402
from paper_conf_ispass_mehrabilcslo21_b200.sharded import make_shard  # noqa: E402


def _with_long_and_empty_rows(a):
    rows = [a.colidx[a.rowidx[i]:a.rowidx[i + 1]].tolist() for i in range(a.M)]
    rows[3] = list(range(0, a.N, 2))          # a long row (split into chunk groups + k_combine)
    rows[5] = []                              # empty rows (k_zero_rows)
    rows[6] = []
    return syn.from_lists(a.M, a.N, rows)


CASES = {
    "rmat_long_empty_k128": (lambda: _with_long_and_empty_rows(syn.rmat(12, 10, 3100, "local")), 128, "cta_aware"),
    "stencil_fused_k64": (lambda: syn.stencil27(18, 3101), 64, "identity"),      # row fusion R = 4
    "uniform_k36": (lambda: syn.uniform(3000, 4000, 7, 3102, poisson=True), 36, "nnz_sort"),   # W = 4 path
}


@pytest.mark.parametrize("name", list(CASES))
@pytest.mark.parametrize("n_dsts", [1, 3, 8])
def test_run_to_every_destination(name, n_dsts):
    gen, K, pol = CASES[name]
    a = gen()
    h = pkg.SpMM.from_csr(a)
    h.permute(pol)
    B = torch.from_numpy(syn.dense(a.N, K, 3103)).cuda()
    ref = h.run(B).clone()
    dsts = [torch.full((a.M, K), float("nan"), device="cuda") for _ in range(n_dsts)]
    h.run_to(B, dsts)
    torch.cuda.synchronize()
    for d in dsts:
        assert torch.equal(d.view(torch.int32), ref.view(torch.int32))
    h.close()


def test_run_to_shards_reassemble():
    a = _with_long_and_empty_rows(syn.rmat(13, 8, 3104, "natural"))
    K = 64
    Bn = syn.dense(a.N, K, 3105)
    B = torch.from_numpy(Bn).cuda()
    whole = pkg.SpMM.from_csr(a)
    whole.permute("hybrid_2_1")
    ref = whole.run(B).clone()
    whole.close()
    bounds = pkg.spmm_partition_by_nnz(a.rowidx, 2)
    bufs = [torch.full((a.M, K), float("nan"), device="cuda") for _ in range(2)]
    for r in range(2):
        sh = make_shard(a.M, a.N, a.rowidx, a.colidx, a.value, bounds, r)
        hs = pkg.SpMM(sh.M, sh.N, sh.rowidx, sh.colidx, sh.value)
        hs.permute("cta_aware")
        hs.run_to(B, bufs, row_offset=int(bounds[r]))
        torch.cuda.synchronize()
        if r == 0:   # rows of the other shard untouched so far
            assert torch.isnan(bufs[0][int(bounds[1]):]).all()
        hs.close()
    for d in bufs:
        assert torch.equal(d.view(torch.int32), ref.view(torch.int32))
    C_ref, bound = oracle.spmm(a, Bn)
    err = np.abs(bufs[0].cpu().numpy().astype(np.float64) - C_ref)
    assert np.all(err <= 1e-5 * bound + 1e-6)


def test_run_to_errors():
    a = syn.rmat(10, 6, 3106, "natural")
    h = pkg.SpMM.from_csr(a)
    B = torch.zeros((a.N, 32), device="cuda")
    C = torch.zeros((a.M + 8, 32), device="cuda")
    lib = pkg.load_library()
    import ctypes
    for n in (0, 9):
        arr = (ctypes.c_void_p * max(n, 1))(*([C.data_ptr()] * max(n, 1)))
        assert lib.spmm_run_to(h._h, B.data_ptr(), 32, arr, n, 0, None) == 1
    with pytest.raises(pkg.SpmmError) as ex:
        h.run_to(B, [C.data_ptr() + 4])                 # destination rows not 16-byte aligned
    assert ex.value.status == 3
    with pytest.raises(pkg.SpmmError) as ex:
        h.run_to(B, [C], row_offset=-1)
    assert ex.value.status == 1
    h.run_to(B, [C], row_offset=8)                      # in bounds: rows 8 .. 8 + M
    h.close()


def test_run_allgather_fused_symmetric_memory():
    """ShardedSpMM.run_allgather_fused into a torch symmetric-memory full-C buffer (world 1 NCCL group on one GPU:
    the destination is the symmetric allocation's own device pointer, the same address kind a peer would use)."""
    import os
    import socket
    import torch.distributed as dist
    from paper_conf_ispass_mehrabilcslo21_b200.sharded import ShardedSpMM

    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        a = syn.rmat(12, 8, 3110, "local")
        K = 64
        Bn = syn.dense(a.N, K, 3111)
        B = torch.from_numpy(Bn).cuda()
        sh = ShardedSpMM.scatter(a, src=0, compact_B=False)     # NCCL group of one: the shard is all of A
        sh.permute("cta_aware")
        buf, ptrs, hdl = sh.symmetric_C(K)
        assert len(ptrs) == 1
        buf.fill_(float("nan"))
        sh.run_allgather_fused(B, ptrs)
        torch.cuda.synchronize()
        ref = sh.run(B)
        assert torch.equal(buf.view(torch.int32), ref.view(torch.int32))
        C_ref, bound = oracle.spmm(a, Bn)
        err = np.abs(buf.cpu().numpy().astype(np.float64) - C_ref)
        assert np.all(err <= 1e-5 * bound + 1e-6)
        mc = int(getattr(hdl, "multicast_ptr", 0) or 0)
        if mc:    # NVLS multicast store path, where the rendezvous provides one
            buf.fill_(float("nan"))
            torch.cuda.synchronize()
            sh.run_allgather_multicast(B, mc)
            torch.cuda.synchronize()
            assert torch.equal(buf.view(torch.int32), ref.view(torch.int32))
        sh.close()
        # the compact exchange + column-chunk pipeline on an NCCL group of one (the source's own chunks)
        shc = ShardedSpMM.scatter(a, src=0, compact_B=True)
        shc.permute("cta_aware")
        Bl = shc.distribute_B(B, src=0)
        refc = shc.run(Bl)
        assert torch.equal(refc.view(torch.int32), ref.view(torch.int32))
        Cp = shc.run_pipelined(B, src=0)              # default: 64-column chunks (here one)
        torch.cuda.synchronize()
        assert torch.equal(Cp.view(torch.int32), ref.view(torch.int32))
        Cp = shc.run_pipelined(B, chunks=4, src=0)    # 16-column chunks: another lane geometry, same tolerance
        torch.cuda.synchronize()
        assert np.all(np.abs(Cp.cpu().numpy().astype(np.float64) - C_ref) <= 1e-5 * bound + 1e-6)
        shc.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", list(CASES))
def test_run_ld_column_blocks(name):
    """spmm_run_ld (f2 iii's building block): column chunks of B computed into the matching columns of a wider C
    reassemble the full-width spmm_run result bit for bit; columns outside a block stay untouched."""
    gen, K, pol = CASES[name]
    a = gen()
    h = pkg.SpMM.from_csr(a)
    h.permute(pol)
    B = torch.from_numpy(syn.dense(a.N, K, 3300)).cuda()
    ref = h.run(B)
    from paper_conf_ispass_mehrabilcslo21_b200.sharded import chunk_bounds
    C_ref, bound = oracle.spmm(a, B.cpu().numpy())
    for chunks in (2, 3):
        C = torch.full((a.M, K), float("nan"), device="cuda")
        cb = chunk_bounds(K, chunks, align=4 if K % 8 else 8)
        for c0, c1 in cb:
            h.run_ld(B[:, c0:c1].contiguous(), C, col_offset=c0)
            torch.cuda.synchronize()
            assert torch.isnan(C[:, c1:]).all()            # later columns not written yet
        assert np.all(np.abs(C.cpu().numpy().astype(np.float64) - C_ref) <= 1e-5 * bound + 1e-6), (name, chunks)
        # bit-identical whenever the split rows are cut the same way: no split rows, or 64-column chunks of K = 128
        if h.info()["split_rows"] == 0 or all(c1 - c0 == 64 for c0, c1 in cb):
            assert torch.equal(C.view(torch.int32), ref.view(torch.int32)), (name, chunks)
    h.close()


def test_run_multicast_arguments():
    """spmm_run_multicast needs a multicast address, K % 8 == 0 and 32-byte aligned rows (the NVLS store path itself
    needs a multi-GPU multicast group: unmeasured on one GPU)."""
    a = syn.rmat(10, 8, 3400, "natural")
    h = pkg.SpMM.from_csr(a)
    B = torch.from_numpy(syn.dense(a.N, 64, 3401)).cuda()
    with pytest.raises(ValueError):
        h.run_multicast(B, 0)
    lib = pkg.load_library()
    C = torch.empty((a.M, 64), device="cuda")
    assert lib.spmm_run_multicast(h._h, B.data_ptr(), 64, None, 0, None) == 1            # NULL -> INVALID_ARG
    assert lib.spmm_run_multicast(h._h, B.data_ptr(), 64, C.data_ptr(), -1, None) == 1   # negative row offset
    B36 = torch.from_numpy(syn.dense(a.N, 36, 3402)).cuda()
    assert lib.spmm_run_multicast(h._h, B36.data_ptr(), 36, C.data_ptr(), 0, None) == 3  # K % 8 -> UNSUPPORTED
    assert lib.spmm_run_multicast(h._h, B.data_ptr(), 64, C.data_ptr() + 16, 0, None) == 3   # misaligned rows
    h.close()
