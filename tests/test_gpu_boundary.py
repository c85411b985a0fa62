"""GPU tests of the C-ABI boundary semantics (include/spmm.h): spmm_prepare makes spmm_run
asynchronous, concurrent runs on one handle from several streams, atomic spmm_permute under allocation failure
(fault injection through the allocator hook), and the binding's argument checks.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import synthetic as syn

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _matrix():
    """Power-law rows with split rows (> 128 nnz), empty rows and short rows: every run class."""
    return syn.rmat(13, 12, 4100, "local")


def test_prepare_then_run():
    a = _matrix()
    h = pkg.SpMM.from_csr(a)
    h.permute("cta_aware")
    assert h.schedule_info()["rows_per_task"] == 0           # dropped by the permute
    for K in (64, 128):
        h.prepare(K)
        B = syn.dense(a.N, K, 4101)
        ref, bound = oracle.spmm(a, B)
        C = h.run(torch.from_numpy(B).cuda())
        assert h.schedule_info()["rows_per_task"] == 4       # G = 8 lanes per row at K = 64 / 128
        err = np.abs(C.cpu().numpy().astype(np.float64) - ref)
        assert np.all(err <= 1e-5 * bound + 1e-6), K
    h.close()


def test_concurrent_runs_on_streams():
    """Runs on one handle issued back to back on 4 streams (more runs than scratch slots), each with its own B
    and C: every C is bit-identical to the same run issued alone."""
    a = _matrix()
    h = pkg.SpMM.from_csr(a)
    h.permute("hybrid_2_1")
    K = 128
    h.prepare(K)
    Bs = [torch.from_numpy(syn.dense(a.N, K, 4200 + i)).cuda() for i in range(10)]
    solo = []
    for B in Bs:
        solo.append(h.run(B).clone())
    torch.cuda.synchronize()
    streams = [torch.cuda.Stream() for _ in range(4)]
    Cs = [torch.full((a.M, K), float("nan"), device="cuda") for _ in Bs]
    torch.cuda.synchronize()
    for i, (B, C) in enumerate(zip(Bs, Cs)):
        s = streams[i % 4]
        with torch.cuda.stream(s):
            h.run(B, C, stream=s)
    torch.cuda.synchronize()
    for i in range(len(Bs)):
        assert torch.equal(Cs[i].view(torch.int32), solo[i].view(torch.int32)), i
    ref, bound = oracle.spmm(a, Bs[3].cpu().numpy())
    assert np.all(np.abs(Cs[3].cpu().numpy() - ref) <= 1e-5 * bound + 1e-6)
    h.close()


_OOM = r"""
import ctypes, sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle, synthetic as syn, paper_conf_ispass_mehrabilcslo21_b200 as pkg
lib = pkg.load_library()
budget = [10 ** 9]
fails = [0]
def _a(n, stream, ctx):
    if budget[0] <= 0:
        fails[0] += 1
        return None
    budget[0] -= 1
    return torch.cuda.caching_allocator_alloc(int(n), 0, stream or 0)
def _f(p, stream, ctx):
    torch.cuda.caching_allocator_delete(p)
cbs = (pkg._ALLOC_T(_a), pkg._FREE_T(_f))
assert lib.spmm_set_allocator(cbs[0], cbs[1], None) == 0
a = syn.rmat(12, 12, 4300, "local")
B = syn.dense(a.N, 64, 4301)
ref, bound = oracle.spmm(a, B)
Bd = torch.from_numpy(B).cuda()
h = pkg.SpMM.from_csr(a)
h.permute("nnz_sort")
good = h.perm().copy()
n_oom = 0
for k in range(0, 40, 3):                 # fail the (k+1)-th allocation of the permute
    budget[0] = k
    try:
        h.permute("hybrid_2_1", window=1024)
        ok = True
    except pkg.SpmmError as e:
        ok = False
        assert e.status == 5, e           # SPMM_ERR_OOM
        n_oom += 1
    budget[0] = 10 ** 9
    if ok:
        assert np.array_equal(h.perm(), oracle.permute(a, "hybrid_2_1", window=1024))
        h.permute("nnz_sort")
    else:                                  # the handle kept its previous permutation and still runs
        assert np.array_equal(h.perm(), good)
    C = h.run(Bd)
    torch.cuda.synchronize()
    assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-5 * bound + 1e-6), k
    # a run whose schedule build fails reports OOM too and leaves the handle usable
    h.permute("cta_aware")
    budget[0] = 0
    try:
        h.run(Bd)
        raise SystemExit("run with no memory for its schedule did not fail")
    except pkg.SpmmError as e:
        assert e.status == 5, e
    budget[0] = 10 ** 9
    C = h.run(Bd)
    torch.cuda.synchronize()
    assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-5 * bound + 1e-6), k
    h.permute("nnz_sort")
assert n_oom >= 3 and fails[0] >= n_oom
h.close()
print("OK", n_oom)
"""


def test_oom_fault_injection():
    """Fault injection through the allocator hook: an allocator that returns NULL after k
    allocations makes spmm_permute / spmm_run fail with SPMM_ERR_OOM; the handle keeps its previous permutation
    and computes correct C afterwards (a failed permute used to leave freed buffers in the handle).
    In a subprocess: the allocator hook is process-wide."""
    r = subprocess.run([sys.executable, "-c", _OOM.format(root=ROOT)], capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "OK" in r.stdout, r.stdout[-2000:] + r.stderr[-3000:]


def test_binding_argument_checks():
    a = syn.rmat(10, 8, 4400, "natural")
    h = pkg.SpMM.from_csr(a)
    K = 64
    B = torch.from_numpy(syn.dense(a.N, K, 4401)).cuda()
    with pytest.raises(ValueError):
        h.run(B.t().contiguous().t())                      # column-major (non-contiguous) B
    with pytest.raises(ValueError):
        h.run(B.double())                                   # wrong dtype
    with pytest.raises(ValueError):
        h.run(B[: a.N - 1])                                 # too few rows
    with pytest.raises(ValueError):
        h.run(B.cpu())                                      # host tensor
    with pytest.raises(ValueError):
        h.run(B, torch.empty((a.M - 1, K), device="cuda"))  # C too small
    with pytest.raises(ValueError):
        h.run_to(B, [torch.empty((a.M, K), device="cuda")], row_offset=1)   # destination too short for the offset
    with pytest.raises(ValueError):
        pkg.SpMM(a.M, a.N, torch.from_numpy(a.rowidx).cuda().int(), torch.from_numpy(a.colidx).cuda(),
                 torch.from_numpy(a.value).cuda())           # int32 rowidx
    C = h.run(B)
    ref, bound = oracle.spmm(a, B.cpu().numpy())
    assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-5 * bound + 1e-6)
    h.close()


def test_set_perm_and_cache(tmp_path):
    """spmm_set_perm installs a caller-supplied permutation (C bit-identical to the built one; a non-bijection is
    rejected and leaves the handle unchanged); permcache stores a build and reinstalls it on the next call."""
    from paper_conf_ispass_mehrabilcslo21_b200 import permcache
    a = _matrix()
    B = torch.from_numpy(syn.dense(a.N, 64, 4500)).cuda()
    h = pkg.SpMM.from_csr(a)
    h.permute("hybrid_2_1", window=2048)
    built = h.perm()
    C1 = h.run(B).clone()
    h.permute("identity")
    h.set_perm(built)
    assert np.array_equal(h.perm(), built)
    assert torch.equal(h.run(B).view(torch.int32), C1.view(torch.int32))
    bad = built.copy()
    bad[1] = bad[0]                                        # a duplicate: not a bijection
    with pytest.raises(pkg.SpmmError):
        h.set_perm(bad)
    assert np.array_equal(h.perm(), built)                 # unchanged
    bad[1] = a.M                                           # out of range
    with pytest.raises(pkg.SpmmError):
        h.set_perm(bad)
    h2 = pkg.SpMM.from_csr(a)
    p1, hit1 = permcache.permute_cached(h2, a, "cta_aware+md", str(tmp_path), window=1024)
    p2, hit2 = permcache.permute_cached(h2, a, "cta_aware+md", str(tmp_path), window=1024)
    assert (hit1, hit2) == (False, True) and np.array_equal(p1, p2) and np.array_equal(h2.perm(), p1)
    assert np.array_equal(p1, oracle.permute(a, "cta_aware", window=1024, preorder=2))
    _, hit3 = permcache.permute_cached(h2, a, "cta_aware+md", str(tmp_path), window=2048)   # other params: miss
    assert not hit3
    h.close()
    h2.close()


def test_cuda_graph_capture():
    """spmm_run captured into a CUDA graph (torch.cuda.graph) after spmm_prepare: replays with new B values give
    C bit-identical to eager runs (split rows, empty rows and the side-stream zero fill included); capturing an
    unprepared K fails cleanly with SPMM_ERR_STATE."""
    a = _matrix()
    h = pkg.SpMM.from_csr(a)
    h.permute("cta_aware")
    K = 64
    Bs = [torch.from_numpy(syn.dense(a.N, K, 4600 + i)).cuda() for i in range(3)]
    eager = [h.run(B).clone() for B in Bs]
    B_static = torch.empty_like(Bs[0])
    C_static = torch.full((a.M, K), float("nan"), device="cuda")
    h.prepare(K, B_static, C_static)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            h.run(B_static, C_static, stream=s)
    for B, ref in zip(Bs, eager):
        B_static.copy_(B)
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(C_static.view(torch.int32), ref.view(torch.int32))
    g.reset()
    h.permute("identity")                                   # drops the schedules: K = 64 is unprepared now
    g2 = torch.cuda.CUDAGraph()
    with pytest.raises(pkg.SpmmError) as e:
        with torch.cuda.stream(s):
            with torch.cuda.graph(g2, stream=s):
                h.run(B_static, C_static, stream=s)
    assert e.value.status == 6                                # SPMM_ERR_STATE
    torch.cuda.synchronize()
    C = h.run(Bs[0])                                          # the handle is fine afterwards
    ref, bound = oracle.spmm(a, Bs[0].cpu().numpy())
    assert np.all(np.abs(C.cpu().numpy() - ref) <= 1e-5 * bound + 1e-6)
    h.close()
