"""Pins for the oracle SpMM (oracle.c c1, Alg.1) -- CPU only.

The oracle is checked against things other than itself: numpy dense float64
matmul (a library routine), scipy.sparse CSR @ dense (an independent library
implementation with the same sequential per-row order, so bit-identical),
integer-valued inputs (exact), the worked example E1, and the invariance of C
under every row permutation (permutations "preserve the CSR representation").
"""
import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import synthetic as syn
from checkers import is_bijection


def dense_of(csr):
    A = np.zeros((csr.M, csr.N), dtype=np.float64)
    for i in range(csr.M):
        for j in range(csr.rowidx[i], csr.rowidx[i + 1]):
            A[i, csr.colidx[j]] = csr.value[j]
    return A


@pytest.mark.parametrize("seed", [1, 2, 3])
@pytest.mark.parametrize("K", [4, 32, 36])
def test_spmm_vs_dense_numpy(seed, K):
    a = syn.uniform(50, 70, 6, seed, poisson=True)
    B = syn.dense(a.N, K, seed + 1)
    C, bound = oracle.spmm(a, B)
    A = dense_of(a)
    np.testing.assert_allclose(C, A @ B.astype(np.float64), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(bound, np.abs(A) @ np.abs(B.astype(np.float64)), rtol=1e-12, atol=1e-12)
    assert np.all(bound >= np.abs(C) - 1e-12)


@pytest.mark.parametrize("gen", ["rmat", "stencil", "block"])
def test_spmm_vs_scipy_bit_identical(gen):
    if gen == "rmat":
        a = syn.rmat(10, 8, 11, "natural")
    elif gen == "stencil":
        a = syn.stencil27(8, 12)
    else:
        a = syn.blockcluster(600, 2000, 32, 4, 10, 13)
    B = syn.dense(a.N, 32, 99)
    C, _ = oracle.spmm(a, B)
    S = sp.csr_matrix((a.value.astype(np.float64), a.colidx, a.rowidx), shape=(a.M, a.N))
    ref = S @ B.astype(np.float64)
    assert np.array_equal(C, ref)


def test_spmm_integer_exact():
    a = syn.rmat(9, 6, 5, "random-label", int_values=True)
    B = syn.dense(a.N, 16, 6, int_values=True)
    C, _ = oracle.spmm(a, B)
    ref = dense_of(a).astype(np.int64) @ B.astype(np.int64)
    assert np.array_equal(C, ref.astype(np.float64))


def test_spmm_e1(e1):
    a = syn.from_lists(e1["M"], e1["N"], e1["rows"])
    K = e1["spmm"]["K"]
    B = np.array([[j + 1 + 10 * k for k in range(K)] for j in range(e1["N"])], dtype=np.float32)
    C, _ = oracle.spmm(a, B)
    assert C.tolist() == e1["spmm"]["C"]


def test_spmm_row_subset_and_empty():
    a = syn.from_lists(4, 5, [[], [0, 4], [], [1, 2, 3]], [[], [2.0, -1.0], [], [1.0, 1.0, 1.0]])
    B = syn.dense(5, 8, 3)
    C, _ = oracle.spmm(a, B)
    assert np.all(C[0] == 0) and np.all(C[2] == 0)
    Cs, _ = oracle.spmm(a, B, rows=[3, 1])
    assert np.array_equal(Cs, C[[3, 1]])
    z = syn.from_lists(0, 5, [])
    Cz, _ = oracle.spmm(z, B)
    assert Cz.shape == (0, 8)


@pytest.mark.parametrize("policy", list(oracle.POLICIES))
def test_spmm_permutation_invariance(policy):
    """C computed through the permuted CSR and scattered to C[perm[p]] is bit-identical (c1)."""
    a = syn.rmat(10, 6, 21, "natural")
    B = syn.dense(a.N, 8, 22)
    C, _ = oracle.spmm(a, B)
    perm = oracle.permute(a, policy, window=64)
    assert is_bijection(perm, a.M)
    r2, c2, v2 = oracle.permuted_csr(a, perm)
    b = syn.CSR(a.M, a.N, r2, c2, v2)
    Cp, _ = oracle.spmm(b, B)
    out = np.empty_like(Cp)
    out[perm] = Cp
    assert np.array_equal(out, C)


def test_validate_csr():
    ok = syn.from_lists(3, 4, [[0, 2], [], [1, 3]])
    assert oracle.validate_csr(3, 4, ok.rowidx, ok.colidx) == 0
    assert oracle.validate_csr(3, 4, ok.rowidx, np.array([0, 2, 3, 1], np.int32)) != 0   # unsorted row
    assert oracle.validate_csr(3, 4, ok.rowidx, np.array([0, 2, 1, 4], np.int32)) != 0   # out of range
    assert oracle.validate_csr(3, 4, np.array([0, 2, 1, 4]), ok.colidx) != 0             # non-monotone
    assert oracle.validate_csr(3, 4, ok.rowidx, ok.colidx, nnz=4) == 0
    assert oracle.validate_csr(3, 4, np.array([1, 2, 2, 4]), ok.colidx, nnz=4) != 0      # rowidx[0] != 0
    assert oracle.validate_csr(3, 4, np.array([0, 2, 2, 3]), ok.colidx, nnz=4) != 0      # rowidx[M] != nnz
    assert oracle.validate_csr(3, 4, ok.rowidx, ok.colidx, nnz=5) != 0                   # rowidx[M] != nnz
    assert oracle.validate_csr(3, 4, ok.rowidx, np.array([0, 2, -1, 3], np.int32)) != 0  # negative column
    assert oracle.validate_csr(3, 4, ok.rowidx, np.array([0, 0, 1, 3], np.int32)) != 0   # duplicate column
