"""GPU parity of the inverted-index chain builders (k_chain_xl for windows of <= 4096 rows, k_chain_x above, up to
the whole matrix): paper-exact greedy chains (W = 0).

Small sizes: forced onto the inverted-index builder (SPMM_CHAIN_EXACT=1) and compared bit-exact with the
oracle (oracle.c, O(W^2) brute force of the definition) for CTA_AWARE and HYBRID_2_1, whole-matrix and
multi-window, original and MinHash pre-orders.  Full size (C2 stencil, M = 1M, W = 0): a bijection whose
sampled steps are locally optimal under the policy key, checked with scipy sparse products (independent of
both the oracle and the kernel: DESIGN.md §3).
"""
import os

import numpy as np
import pytest

import oracle
import synthetic as syn

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

GENS = {
    "rmat12_natural": lambda: syn.rmat(12, 12, 2100, "natural"),
    "rmat13_local": lambda: syn.rmat(13, 8, 2101, "local"),
    "stencil14": lambda: syn.stencil27(14, 2102),
    "block_planted": lambda: syn.blockcluster(3000, 6000, 30, 3, 12, 2103, planted=True),
    "uniform_poisson": lambda: syn.uniform(3500, 5000, 3, 2104, poisson=True),   # many empty rows
    "banded": lambda: syn.banded(4000, 9, 40, 2105),
}


@pytest.fixture
def exact_builder(monkeypatch):
    monkeypatch.setenv("SPMM_CHAIN_EXACT", "1")
    yield


@pytest.mark.parametrize("name", list(GENS))
@pytest.mark.parametrize("policy", ["cta_aware", "hybrid_2_1", "warp_aware", "hybrid_2_3", "hybrid_1", "hybrid_2_2"])
@pytest.mark.parametrize("window,preorder", [(0, 0), (1024, 0), (1024, 1)])
def test_exact_builder_matches_oracle(exact_builder, name, policy, window, preorder):
    a = GENS[name]()
    h = pkg.SpMM.from_csr(a)
    h.permute(policy, window=window, preorder=preorder, seed=7)
    got = h.perm()
    h.close()
    ref = oracle.permute(a, policy, window=window, preorder=preorder, seed=7)
    assert np.array_equal(got, ref), (name, policy, window, int(np.argmax(got != ref)))


@pytest.mark.parametrize("policy", ["cta_aware", "hybrid_2_2", "hybrid_1"])
def test_exact_builder_wide_prefix(monkeypatch, policy):
    """The 64-bit posting-list prefix variant (taken when 1024 x the longest list could overflow int32)."""
    monkeypatch.setenv("SPMM_CHAIN_EXACT", "1")
    monkeypatch.setenv("SPMM_CHAIN_WIDE", "1")
    a = GENS["rmat13_local"]()
    h = pkg.SpMM.from_csr(a)
    for window in (0, 1024):
        h.permute(policy, window=window)
        assert np.array_equal(h.perm(), oracle.permute(a, policy, window=window)), (policy, window)
    h.close()


@pytest.mark.parametrize("policy", ["warp_aware", "hybrid_2_3", "hybrid_2_2"])
@pytest.mark.parametrize("nw", [1, 2])
def test_exact_builder_small_nw(exact_builder, policy, nw):
    """nw = 1: the reference row out[q - nw] is the previous position, written by thread 0 after the previous
    step's last barrier -- the builder must take it from its register copy (a read of out[q - 1] raced
    that write).  Bit-exact against the oracle at nw = 1 and 2, whole matrix and windows."""
    a = GENS["rmat12_natural"]()
    h = pkg.SpMM.from_csr(a)
    for window in (0, 512):
        h.permute(policy, window=window, nw=nw)
        ref = oracle.permute(a, policy, nw=nw, window=window)
        assert np.array_equal(h.perm(), ref), (policy, nw, window)
    h.close()


def test_exact_builder_matches_k_chain():
    """Same answer as the shared-memory bitmap builder k_chain on a window it can also take (32768 rows)."""
    a = syn.rmat(15, 6, 2110, "local")
    h = pkg.SpMM.from_csr(a)
    outs = []
    for force in ("0", "1"):
        os.environ["SPMM_CHAIN_EXACT"] = force
        try:
            h.permute("hybrid_2_1", window=32768)
            outs.append(h.perm())
        finally:
            os.environ.pop("SPMM_CHAIN_EXACT", None)
    h.close()
    assert np.array_equal(outs[0], outs[1])


def _block_matrix(a, bw=32):
    import scipy.sparse as sp
    rows = np.repeat(np.arange(a.M), np.diff(a.rowidx))
    m = sp.csr_matrix((np.ones(a.nnz, dtype=np.int32), (rows, np.asarray(a.colidx) // bw)),
                      shape=(a.M, (a.N + bw - 1) // bw))
    m = m.tocsr()
    m.sum_duplicates()
    m.data[:] = 1                                     # duplicate (row, block) pairs summed -> back to 1
    return m


def check_sampled_steps(a, perm, policy, samples, seed=0, nt=32, nw=32):
    """At sampled positions q the row placed at q minimises (ham(r, ref), [|wl_r - wl_prev|,] r) over the rows not
    placed before q; ref = perm[q-1] (CTA_AWARE, HYBRID_2_1: P:L122, L134) or perm[q-nw] for q >= nw (WARP_AWARE,
    HYBRID_2_3: P:L118-120, L146); wl_prev = wl of perm[q-1]; HYBRID_2_2's second key is ham(r, perm[q-nw]) for
    q >= nw.  W = 0: one window."""
    Bm = _block_matrix(a)
    nb = np.diff(Bm.indptr).astype(np.int64)
    wl = (np.diff(np.asarray(a.rowidx)).astype(np.int64) + nt - 1) // nt
    pos = np.empty(a.M, dtype=np.int64)
    pos[perm] = np.arange(a.M)
    rng = np.random.default_rng(seed)
    back = nw if policy in ("warp_aware", "hybrid_2_3") else 1
    qs = np.unique(np.concatenate([[back, a.M - 1], rng.integers(back, a.M, samples)]))
    for q in qs:
        p = int(perm[q - back])
        inter = np.asarray((Bm @ Bm[p].T).todense()).ravel().astype(np.int64)
        ham = nb + nb[p] - 2 * inter
        cand = np.nonzero(pos >= q)[0]
        wprev = wl[int(perm[q - 1])]
        if policy in ("hybrid_2_1", "hybrid_2_3"):
            k2 = np.abs(wl[cand] - wprev)
        elif policy == "hybrid_2_2" and q >= nw:      # second key: Hamming to perm[q - nw]
            p2 = int(perm[q - nw])
            inter2 = np.asarray((Bm @ Bm[p2].T).todense()).ravel().astype(np.int64)
            k2 = (nb + nb[p2] - 2 * inter2)[cand]
        else:
            k2 = np.zeros(len(cand), dtype=np.int64)
        order = np.lexsort((cand, k2, ham[cand]))
        assert int(cand[order[0]]) == int(perm[q]), (policy, int(q))


@pytest.mark.parametrize("policy", ["cta_aware", "hybrid_2_1", "warp_aware", "hybrid_2_3", "hybrid_2_2"])
def test_exact_whole_matrix_c2(policy):
    """C2 (27-point stencil 100^3, M = 1M): the paper's whole-matrix chain (W = 0)."""
    a = syn.stencil27(100, 2000)
    h = pkg.SpMM.from_csr(a)
    h.permute(policy, window=0)
    perm = h.perm()
    h.close()
    assert np.array_equal(np.sort(perm), np.arange(a.M))
    check_sampled_steps(a, perm, policy, samples=40)


def _hub_matrix(M, N, seed):
    """2-3 random columns per row plus one column (0) shared by every row: every greedy step touches every
    unplaced row of its window through block 0's posting list."""
    rng = np.random.default_rng(seed)
    rows = [sorted({0, *rng.choice(np.arange(1, N), size=int(rng.integers(2, 4)), replace=False).tolist()})
            for _ in range(M)]
    return syn.from_lists(M, N, rows)


@pytest.mark.parametrize("window,M,policies", [
    (8192, 2 * 8192 + 1000, ("cta_aware", "hybrid_2_1")),        # k_chain_x, multi-window, ragged last window
    (16384, 16384 + 3000, ("cta_aware", "hybrid_2_2")),          # > 8192 touched rows per step: list overflow path
])
def test_exact_builder_large_windows(exact_builder, window, M, policies):
    """Windows above k_chain_xl's 4096 rows go to k_chain_x, whose per-step touched-row list (8192 rows) falls back
    to re-walking the posting lists when a step touches more rows: both paths against the oracle."""
    a = _hub_matrix(M, 30000, 2107)
    h = pkg.SpMM.from_csr(a)
    for policy in policies:
        h.permute(policy, window=window)
        got = h.perm()
        ref = oracle.permute(a, policy, window=window)
        assert np.array_equal(got, ref), (policy, window, int(np.argmax(got != ref)))
    h.close()
