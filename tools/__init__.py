"""Measurement helpers (not the method, not the oracle): an L2-capacity LRU model of B-row reuse."""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liblru.so")
_lib = None


def build():
    src = os.path.join(_HERE, "lru_model.c")
    if not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", src, "-o", _LIB])
    return _LIB


def lru_misses(csr, order, cap_rows):
    """B-row misses of a fully-associative LRU cache of cap_rows rows, rows processed in `order`."""
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_LIB)
        _lib.lru_misses.restype = ctypes.c_int64
        _lib.lru_misses.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p,
                                    ctypes.c_void_p, ctypes.c_int64]
    r = np.ascontiguousarray(csr.rowidx, dtype=np.int64)
    c = np.ascontiguousarray(csr.colidx, dtype=np.int32)
    o = None if order is None else np.ascontiguousarray(order, dtype=np.int32)
    return int(_lib.lru_misses(csr.M, csr.N, r.ctypes.data, c.ctypes.data, None if o is None else o.ctypes.data,
                               int(cap_rows)))
