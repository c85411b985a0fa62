"""Measurement helpers (not the method, not the oracle): an L2-capacity LRU model of B-row reuse, an L2->SM
bandwidth probe and the cuSPARSE SpMM baseline (tools/cusparse_ref.cu)."""
import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liblru.so")
_lib = None


_PROBE = os.path.join(_HERE, "libl2probe.so")
_LDPATH = os.path.join(_HERE, "libldpath.so")


def build():
    src = os.path.join(_HERE, "lru_model.c")
    if not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-shared", "-fPIC", src, "-o", _LIB])
    psrc = os.path.join(_HERE, "l2probe.cu")
    if not os.path.exists(_PROBE) or os.path.getmtime(_PROBE) < os.path.getmtime(psrc):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-shared", "-Xcompiler", "-fPIC", psrc, "-o", _PROBE])
    lsrc = os.path.join(_HERE, "ldpathprobe.cu")
    if not os.path.exists(_LDPATH) or os.path.getmtime(_LDPATH) < os.path.getmtime(lsrc):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3",
                               "-DLDPATH_NO_MAIN", "-shared", "-Xcompiler", "-fPIC", lsrc, "-o", _LDPATH])
    csrc = os.path.join(_HERE, "cusparse_ref.cu")
    if not os.path.exists(_CUSP) or os.path.getmtime(_CUSP) < os.path.getmtime(csrc):
        subprocess.check_call(["/usr/local/cuda/bin/nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2",
                               "-shared", "-Xcompiler", "-fPIC", csrc, "-o", _CUSP, "-lcusparse"])
    return _LIB


_CUSP = os.path.join(_HERE, "libcusparse_ref.so")


def cusparse_spmm_times(M, N, nnz, rowptr, colidx, value, B, K, C, alg, reps, flush, stream):
    """cuSPARSE SpMM (CSR ALG1/2/3 or default, row-major B/C) per-rep CUDA-event times in ms, L2 flushed before
    each rep.  Device pointers as ints (int32 rowptr/colidx).  Raises RuntimeError with the status on failure."""
    build()
    lib = ctypes.CDLL(_CUSP)
    f = lib.cusparse_ref_spmm
    f.restype = ctypes.c_int
    f.argtypes = [ctypes.c_int64] * 3 + [ctypes.c_void_p] * 4 + [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int,
                                                                 ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t,
                                                                 ctypes.c_void_p, ctypes.c_void_p]
    out = np.zeros(reps, dtype=np.float32)
    fptr, fbytes = flush if flush else (None, 0)
    rc = f(M, N, nnz, rowptr, colidx, value, B, K, C, int(alg), int(reps), fptr, fbytes, stream, out.ctypes.data)
    if rc != 0:
        raise RuntimeError(f"cusparse_ref_spmm alg {alg}: status {rc}")
    return out.tolist()


def l2_read_bandwidth(bytes_=64 << 20, reps=50):
    """Achievable L2->SM read bandwidth (bytes/s) measured on the current GPU (buffer < L2)."""
    build()
    lib = ctypes.CDLL(_PROBE)
    lib.l2probe_read_bw.restype = ctypes.c_double
    lib.l2probe_read_bw.argtypes = [ctypes.c_int64, ctypes.c_int]
    return float(lib.l2probe_read_bw(int(bytes_), int(reps)))


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


def l2_read_bandwidth_sms(limit, bytes_=64 << 20, reps=20):
    """L2->SM read bandwidth (bytes/s) of the SMs with smid < limit (the others idle)."""
    build()
    lib = ctypes.CDLL(_PROBE)
    lib.l2probe_read_bw_sms.restype = ctypes.c_double
    lib.l2probe_read_bw_sms.argtypes = [ctypes.c_int64, ctypes.c_int, ctypes.c_int]
    return float(lib.l2probe_read_bw_sms(int(bytes_), int(reps), int(limit)))


def ldpath_gather(shape=0, window=16 << 20, row_bytes=512, reps=5):
    """SM load-path gather ceiling (tools/ldpathprobe.cu): random rows of row_bytes gathered from a window of
    `window` bytes with k_spmm's load shape (shape 0: 8-lane groups x one 256-bit load per lane).  16 MiB window =
    L2-resident, 32 KiB = L1-resident.  Returns (GB/s, bytes per SM clock)."""
    build()
    lib = ctypes.CDLL(_LDPATH)
    lib.ldpath_gather.restype = ctypes.c_double
    lib.ldpath_gather.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
    bpc = ctypes.c_double(0.0)
    gbs = float(lib.ldpath_gather(int(shape), int(window), int(row_bytes), int(reps), ctypes.byref(bpc)))
    return gbs, float(bpc.value)
