"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no SpMM, permutation or
feature): it only draws CSR matrices and dense operands shaped like the paper's
workloads -- SuiteSparse-like power-law graphs, banded FEM stencils, uniform
random and block-clustered matrices (§IV "Dataset";
SURVEY.md §8(d) "Synthetic inputs"; recipe in DESIGN.md §"Input recipe").

All draws are counter-based (splitmix64 of (seed, stream, counter)) in
``gen.c``, so a matrix depends only on its parameters and seed.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB_PATH = os.path.join(_HERE, "libsynth.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gen.c into libsynth.so (gcc -O3 -fopenmp)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-march=x86-64-v2", "-fopenmp", "-shared", "-fPIC",
                               "-std=gnu11", _SRC, "-o", tmp, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        vp, i32, i64, u64, f64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double
        lib.synth_rmat.restype = vp
        lib.synth_rmat.argtypes = [i32, f64, u64, i32, f64, i32]
        lib.synth_stencil27.restype = vp
        lib.synth_stencil27.argtypes = [i32, u64, i32]
        lib.synth_uniform.restype = vp
        lib.synth_uniform.argtypes = [i64, i64, f64, i32, u64, i32]
        lib.synth_blockcluster.restype = vp
        lib.synth_blockcluster.argtypes = [i64, i64, i64, i64, i64, i32, i32, u64, i32]
        lib.synth_banded.restype = vp
        lib.synth_banded.argtypes = [i64, i64, i64, i64, u64, i32]
        lib.synth_from_degrees.restype = vp
        lib.synth_from_degrees.argtypes = [i64, i64, vp, u64, i32]
        lib.synth_sizes.restype = None
        lib.synth_sizes.argtypes = [vp, vp, vp, vp]
        lib.synth_take.restype = None
        lib.synth_take.argtypes = [vp, vp, vp, vp]
        lib.synth_dense.restype = None
        lib.synth_dense.argtypes = [i64, i64, i64, u64, i32, vp]
        lib.synth_num_threads.restype = i32
        _lib = lib
    return _lib


@dataclass
class CSR:
    """Host CSR: rowidx int64[M+1], colidx int32[nnz] (strictly increasing per row), value float32[nnz]."""
    M: int
    N: int
    rowidx: np.ndarray
    colidx: np.ndarray
    value: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.rowidx[-1]) if self.M > 0 else 0


def _take(h, name: str) -> CSR:
    lib = _load()
    M, N, nnz = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
    lib.synth_sizes(h, ctypes.byref(M), ctypes.byref(N), ctypes.byref(nnz))
    rowidx = np.empty(M.value + 1, dtype=np.int64)
    colidx = np.empty(max(nnz.value, 0), dtype=np.int32)
    value = np.empty(max(nnz.value, 0), dtype=np.float32)
    lib.synth_take(h, rowidx.ctypes.data, colidx.ctypes.data, value.ctypes.data)
    return CSR(M.value, N.value, rowidx, colidx, value, name)


RMAT_VARIANTS = {"natural": 0, "random-label": 1, "local": 2}


def rmat(S: int, edge_factor: float, seed: int, variant: str = "natural", p_local: float = 0.8,
         int_values: bool = False) -> CSR:
    """R-MAT power-law graph, 2^S x 2^S, (a,b,c,d) = (.57,.19,.19,.05), deduplicated."""
    h = _load().synth_rmat(S, float(edge_factor), seed, RMAT_VARIANTS[variant], float(p_local), int(int_values))
    return _take(h, f"rmat{S}-{variant}-ef{edge_factor:g}-s{seed}")


def stencil27(n: int, seed: int, int_values: bool = False) -> CSR:
    """3-D 27-point stencil on an n^3 grid in lexicographic order (banded FEM-like)."""
    return _take(_load().synth_stencil27(n, seed, int(int_values)), f"stencil27-{n}-s{seed}")


def uniform(M: int, N: int, d: float, seed: int, poisson: bool = False, int_values: bool = False) -> CSR:
    """d distinct uniform columns per row (fixed d, or Poisson(d))."""
    return _take(_load().synth_uniform(M, N, float(d), int(poisson), seed, int(int_values)),
                 f"uniform-{M}x{N}-d{d:g}-s{seed}")


def blockcluster(M: int, N: int, g: int, c: int, d: int, seed: int, planted: bool = False, bw: int = 32,
                 int_values: bool = False) -> CSR:
    """Groups of g rows share c column blocks of bw columns; d columns per row; rows shuffled."""
    return _take(_load().synth_blockcluster(M, N, g, c, d, bw, int(planted), seed, int(int_values)),
                 f"blockcluster-{M}-g{g}-c{c}-d{d}{'-planted' if planted else ''}-s{seed}")


def banded(M: int, d: int, halfwidth: int, seed: int, int_values: bool = False) -> CSR:
    """Banded random (FEM-like bandwidth): d distinct uniform columns within [i - w, i + w]."""
    return _take(_load().synth_banded(M, M, d, halfwidth, seed, int(int_values)), f"banded-{M}-d{d}-w{halfwidth}-s{seed}")


def from_degrees(M: int, N: int, degrees: np.ndarray, seed: int, int_values: bool = False) -> CSR:
    """Uniform random columns with an explicit per-row degree list."""
    deg = np.ascontiguousarray(degrees, dtype=np.int64)
    assert deg.shape == (M,)
    return _take(_load().synth_from_degrees(M, N, deg.ctypes.data, seed, int(int_values)), f"degrees-{M}-s{seed}")


def dense(rows: int, K: int, seed: int, int_values: bool = False, row0: int = 0) -> np.ndarray:
    """Rows [row0, row0+rows) of a row-major float32 [*, K] operand, U[-1,1) (or integers in [-8,8])."""
    out = np.empty((rows, K), dtype=np.float32)
    if rows and K:
        _load().synth_dense(row0, rows, K, seed, int(int_values), out.ctypes.data)
    return out


def from_lists(M: int, N: int, rows: list[list[int]], values: list[list[float]] | None = None,
               name: str = "explicit") -> CSR:
    """CSR from explicit per-row column lists (tests / worked examples)."""
    lens = [len(r) for r in rows]
    assert len(rows) == M
    rowidx = np.zeros(M + 1, dtype=np.int64)
    rowidx[1:] = np.cumsum(lens)
    colidx = np.array([c for r in rows for c in r], dtype=np.int32)
    if values is None:
        value = np.ones(len(colidx), dtype=np.float32)
    else:
        value = np.array([v for r in values for v in r], dtype=np.float32)
    return CSR(M, N, rowidx, colidx, value, name)


def host_threads() -> int:
    return int(_load().synth_num_threads())
