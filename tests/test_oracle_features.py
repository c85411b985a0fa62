"""Pins for the oracle's 24 Table II features (oracle.c c3; §V.A) -- CPU only.

Pins: E1 (hand-worked), the paper's own arithmetic (P:L88 warp load, P:L92 cache
lines, P:L114 mask length), 27-point-stencil closed forms, invariants
(sum of requests = sum of T_w, T >= D, mean nnz = nnz/M, sum of warp loads
invariant under permutation), a brute-force Python recount, and consistency of
the permuted-order features with features of the permuted CSR.
"""
import math

import numpy as np
import pytest

import oracle
import synthetic as syn
import checkers as ck


def test_e1_features(e1):
    a = syn.from_lists(e1["M"], e1["N"], e1["rows"])
    f = oracle.features(a, nw=2, nt=2, bw=2)
    np.testing.assert_array_equal(f, np.array(e1["features_identity"], dtype=np.float64))


def one_row(cols, N):
    return syn.from_lists(1, N, [list(cols)])


def test_paper_warp_load(paper_arith):
    for nnz, wl in paper_arith["warp_load"]["cases"]:
        f = oracle.features(one_row(range(nnz), 128), nw=1, nt=32, bw=32)
        assert f[9] == f[10] == f[11] == wl


def test_paper_cache_lines(paper_arith):
    pc = paper_arith["cache_lines"]
    for case in ("consecutive_32", "stride_32"):
        d = pc[case]
        cols = [d["cols_start"] + d["cols_step"] * t for t in range(d["count"])]
        f = oracle.features(one_row(cols, cols[-1] + 1), nw=1, nt=pc["nt"], bw=pc["bw"])
        assert f[18] == d["lines"]          # total-cache-lines-per-warp
        assert f[15] == d["lines"]          # distinct lines
        assert f[6] == d["lines"]           # nnz-blocks-per-row


def test_paper_mask_bits(paper_arith):
    for N, bits in paper_arith["mask_bits"]["cases"]:
        f = oracle.features(one_row(range(N), N), nw=1, nt=32, bw=32)
        assert f[6] == bits


def test_stencil_closed_form():
    n = 12
    a = syn.stencil27(n, 3)
    f = oracle.features(a)
    M = n ** 3
    nnz = (3 * n - 2) ** 3
    assert a.nnz == nnz == (n - 2) ** 3 * 27 + 6 * (n - 2) ** 2 * 18 + 12 * (n - 2) * 12 + 8 * 8
    assert f[0] == M and f[1] == M
    assert f[2] == nnz / (M * M)
    assert (f[3], f[4], f[5]) == (8, nnz / M, 27)
    # every wl = 1 (nnz <= 27 <= 32): WL_w = number of rows congruent to w mod 32
    counts = [len(range(w, M, 32)) for w in range(32)]
    assert (f[9], f[10], f[11]) == (min(counts), M / 32, max(counts))


def brute_features(a, perm=None, nw=32, nt=32, bw=32):
    """Straight recount from the Table II wording with Python sets."""
    order = list(range(a.M)) if perm is None else [int(x) for x in perm]
    rows = [a.colidx[a.rowidx[i]:a.rowidx[i + 1]].tolist() for i in order]
    blocks = [sorted({c // bw for c in r}) for r in rows]
    req = {}
    T = [0] * nw
    D = [set() for _ in range(nw)]
    WL = [0] * nw
    for p, r in enumerate(rows):
        WL[p % nw] += math.ceil(len(r) / nt)
        D[p % nw] |= set(blocks[p])
        for c0 in range(0, len(r), nt):
            lines = {c // bw for c in r[c0:c0 + nt]}
            T[p % nw] += len(lines)
            for b in lines:
                req[b] = req.get(b, 0) + 1
    def st(v):
        return [min(v), sum(v) / len(v), max(v)] if v else [0, 0, 0]
    adj = [len(set(blocks[p]) ^ set(blocks[p + 1])) for p in range(len(rows) - 1)]
    return np.array([a.M, a.N, a.nnz / (a.M * a.N)] + st([len(r) for r in rows]) + st([len(b) for b in blocks])
                    + st(WL) + st(list(req.values())) + st([len(s) for s in D]) + st(T) + st(adj),
                    dtype=np.float64)


@pytest.mark.parametrize("gen", ["rmat", "block", "uniform"])
def test_features_brute_force(gen):
    a = {"rmat": lambda: syn.rmat(9, 8, 5, "natural"),
         "block": lambda: syn.blockcluster(500, 5000, 32, 4, 40, 6),
         "uniform": lambda: syn.uniform(400, 3000, 50, 7, poisson=True)}[gen]()
    np.testing.assert_array_equal(oracle.features(a), brute_features(a))
    perm = oracle.permute(a, "nnz_sort")
    np.testing.assert_array_equal(oracle.features(a, perm), brute_features(a, perm))


def test_invariants():
    a = syn.rmat(10, 10, 9, "random-label")
    f = oracle.features(a)
    nreq = len(np.unique(a.colidx // 32))
    # sum over lines of requests == sum over warps of T_w
    assert math.isclose(f[13] * nreq, f[19] * 32, rel_tol=1e-12)
    assert f[4] == a.nnz / a.M
    f1 = oracle.features(a, nw=1)
    assert f1[18] >= f1[15]                  # T >= D for the single warp
    # sum of warp loads (hence the mean) is invariant under any permutation (Fig. 7)
    for pol in ("plain_sort", "lpt", "cta_aware"):
        fp = oracle.features(a, oracle.permute(a, pol, window=256))
        assert fp[10] == f[10]
        assert fp[3:9].tolist() == f[3:9].tolist()


def test_permuted_features_consistency():
    a = syn.rmat(9, 6, 13, "natural")
    perm = oracle.permute(a, "cta_aware", window=64)
    r2, c2, v2 = oracle.permuted_csr(a, perm)
    b = syn.CSR(a.M, a.N, r2, c2, v2)
    np.testing.assert_array_equal(oracle.features(a, perm), oracle.features(b))


def test_degenerate():
    z = syn.from_lists(1, 10, [[]])
    f = oracle.features(z)
    assert f[0] == 1 and f[2] == 0 and np.all(f[3:] == 0)
