"""CPU oracle for the row-permuted CSR SpMM hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline``
/ ``--impl reference`` legs may import this package.  The product package
(``paper_conf_ispass_mehrabilcslo21_b200``) never imports it and shares no code
with it.  Arithmetic lives in ``oracle.c`` (plain C, float64); every function
there cites the PAPER.md passage it follows.  This wrapper only marshals
arguments.

Parity unpinned: none (see oracle.c header and DESIGN.md §"Oracle pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
# ORACLE_LIB: a prebuilt variant of the same source (tests/test_oracle_sanitizers.py: ASan + UBSan build)
_LIB_PATH = os.environ.get("ORACLE_LIB") or os.path.join(_HERE, "liboracle.so")
_lib = None

POLICIES = {
    "identity": 0, "nnz_sort": 1, "plain_sort": 2, "cta_aware": 3, "hybrid_1": 4, "hybrid_2_1": 5,
    "flipped": 6, "lpt": 7, "warp_aware": 8, "hybrid_2_2": 9, "hybrid_2_3": 10, "dcsr": 11,
}


def build(force: bool = False) -> str:
    if os.environ.get("ORACLE_LIB"):
        return _LIB_PATH
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=gnu11", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, i32, i64, u64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
        lib.oracle_validate_csr.restype = ctypes.c_int
        lib.oracle_validate_csr.argtypes = [i64, i64, i64, vp, vp]
        lib.oracle_spmm_rows.restype = None
        lib.oracle_spmm_rows.argtypes = [i64, vp, vp, vp, vp, i64, vp, i64, vp, vp]
        lib.oracle_permute.restype = ctypes.c_int
        lib.oracle_permute.argtypes = [i32, i64, vp, vp, i32, i32, i32, i64, i32, u64, vp]
        lib.oracle_permuted_csr.restype = None
        lib.oracle_permuted_csr.argtypes = [i64, vp, vp, vp, vp, vp, vp, vp]
        lib.oracle_features.restype = None
        lib.oracle_features.argtypes = [i64, i64, vp, vp, vp, i32, i32, i32, vp]
        lib.oracle_partition_by_nnz.restype = None
        lib.oracle_partition_by_nnz.argtypes = [vp, i64, i32, vp]
        lib.oracle_minhash_keys.restype = None
        lib.oracle_minhash_keys.argtypes = [i64, vp, vp, i32, u64, vp]
        lib.oracle_features_b200.restype = None
        lib.oracle_features_b200.argtypes = [i64, i64, vp, vp, vp, i64, vp]
        lib.oracle_mlp_forward_n.restype = i32
        lib.oracle_mlp_forward_n.argtypes = [vp, i32, vp, i32, vp]
        lib.oracle_median_block_keys.restype = None
        lib.oracle_median_block_keys.argtypes = [i64, vp, vp, i32, vp]
        lib.oracle_threads.restype = ctypes.c_int
        lib.oracle_threads.argtypes = [ctypes.c_int]
        lib.oracle_mlp_forward.restype = i32
        lib.oracle_mlp_forward.argtypes = [vp, vp, i32, vp]
        _lib = lib
    return _lib


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def set_threads(n: int = 0) -> int:
    """OpenMP threads of the oracle's parallel loops: n > 0 sets them (overriding an inherited OMP_NUM_THREADS,
    e.g. torchrun's 1); returns the count actually in effect."""
    return int(_load().oracle_threads(int(n)))


def validate_csr(M, N, rowidx, colidx, nnz=None) -> int:
    """0 if valid (nnz defaults to rowidx[M], i.e. only the other checks apply)."""
    r, c = _c(rowidx, np.int64), _c(colidx, np.int32)
    if nnz is None:
        nnz = int(r[-1]) if M >= 0 else 0
    return int(_load().oracle_validate_csr(M, N, nnz, r.ctypes.data, c.ctypes.data))


def spmm(csr, B: np.ndarray, rows=None):
    """(C, bound) float64 for all rows (rows=None) or the listed original rows (c1)."""
    B = _c(B, np.float32)
    K = B.shape[1]
    r, c, v = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32), _c(csr.value, np.float32)
    if rows is None:
        n, rp = csr.M, None
    else:
        rows = _c(rows, np.int64)
        n, rp = len(rows), rows.ctypes.data
    C = np.empty((n, K), dtype=np.float64)
    bound = np.empty((n, K), dtype=np.float64)
    _load().oracle_spmm_rows(csr.M, r.ctypes.data, c.ctypes.data, v.ctypes.data, B.ctypes.data, K, rp, n,
                             C.ctypes.data, bound.ctypes.data)
    return C, bound


def permute(csr, policy, nw=32, nt=32, bw=32, window=0, preorder=0, seed=0) -> np.ndarray:
    pid = POLICIES[policy] if isinstance(policy, str) else int(policy)
    r, c = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32)
    perm = np.empty(csr.M, dtype=np.int32)
    rc = _load().oracle_permute(pid, csr.M, r.ctypes.data, c.ctypes.data, nw, nt, bw, window, preorder, seed,
                                perm.ctypes.data)
    if rc != 0:
        raise ValueError(f"oracle_permute: invalid arguments (policy={policy}, window={window}, nw={nw})")
    return perm


def permuted_csr(csr, perm):
    r, c, v = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32), _c(csr.value, np.float32)
    perm = _c(perm, np.int32)
    r2 = np.empty(csr.M + 1, dtype=np.int64)
    c2 = np.empty(csr.nnz, dtype=np.int32)
    v2 = np.empty(csr.nnz, dtype=np.float32)
    _load().oracle_permuted_csr(csr.M, r.ctypes.data, c.ctypes.data, v.ctypes.data, perm.ctypes.data,
                                r2.ctypes.data, c2.ctypes.data, v2.ctypes.data)
    return r2, c2, v2


def features(csr, perm=None, nw=32, nt=32, bw=32) -> np.ndarray:
    r, c = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32)
    pp = None
    if perm is not None:
        perm = _c(perm, np.int32)
        pp = perm.ctypes.data
    f = np.empty(24, dtype=np.float64)
    _load().oracle_features(csr.M, csr.N, r.ctypes.data, c.ctypes.data, pp, nw, nt, bw, f.ctypes.data)
    return f


B200_FEATURES = ["fusion_union_r2", "fusion_union_r4", "window1024_distinct_cols", "b_row_byte_share",
                 "empty_row_fraction", "split_row_nnz_fraction", "lane_slot_efficiency"]


def features_b200(csr, K, perm=None) -> np.ndarray:
    """The 7 B200 platform features g0..g6 (oracle.c c3b) of the matrix in its order (or perm's)."""
    r, c = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32)
    pp = None
    if perm is not None:
        perm = _c(perm, np.int32)
        pp = perm.ctypes.data
    g = np.empty(7, dtype=np.float64)
    _load().oracle_features_b200(csr.M, csr.N, r.ctypes.data, c.ctypes.data, pp, int(K), g.ctypes.data)
    return g


def partition_by_nnz(rowidx, P: int) -> np.ndarray:
    r = _c(rowidx, np.int64)
    b = np.empty(P + 1, dtype=np.int64)
    _load().oracle_partition_by_nnz(r.ctypes.data, len(r) - 1, P, b.ctypes.data)
    return b


def minhash_keys(csr, bw=32, seed=0) -> np.ndarray:
    r, c = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32)
    h = np.empty(csr.M, dtype=np.uint64)
    _load().oracle_minhash_keys(csr.M, r.ctypes.data, c.ctypes.data, bw, seed, h.ctypes.data)
    return h


def median_block_keys(csr, bw=32) -> np.ndarray:
    r, c = _c(csr.rowidx, np.int64), _c(csr.colidx, np.int32)
    h = np.empty(csr.M, dtype=np.uint64)
    _load().oracle_median_block_keys(csr.M, r.ctypes.data, c.ctypes.data, bw, h.ctypes.data)
    return h


def mlp_forward(feat, weights, P):
    f = _c(feat, np.float64)
    w = _c(weights, np.float32)
    out = np.empty(P, dtype=np.float64)
    best = _load().oracle_mlp_forward(f.ctypes.data, w.ctypes.data, P, out.ctypes.data)
    return int(best), out


def mlp_forward_n(feat, weights, P):
    f = _c(feat, np.float64)
    w = _c(weights, np.float32)
    out = np.empty(P, dtype=np.float64)
    best = _load().oracle_mlp_forward_n(f.ctypes.data, len(f), w.ctypes.data, P, out.ctypes.data)
    return int(best), out
