"""Thin Python binding of libspmm_b200.so (include/spmm.h) -- argument marshalling only.

Every step of the hot path runs in the CUDA library; this module only converts
numpy arrays / torch tensors to pointers, passes torch's current CUDA stream,
and (optionally) routes the library's device allocations through PyTorch's
caching allocator.  There is NO CPU fallback: if the extension cannot be loaded
every entry point raises.

Names follow the C ABI (``spmm_create``, ``spmm_permute``, ``spmm_run`` ...);
``SpMM`` is a convenience object wrapping one handle.
Paper: Mehrabi et al., ISPASS 2021; see include/spmm.h for the
passage each entry point implements.
"""
from __future__ import annotations

import atexit
import ctypes
import os
import weakref

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libspmm_b200.so")

POLICIES = {
    "identity": 0, "nnz_sort": 1, "plain_sort": 2, "cta_aware": 3, "hybrid_1": 4, "hybrid_2_1": 5,
    "flipped": 6, "lpt": 7, "warp_aware": 8, "hybrid_2_2": 9, "hybrid_2_3": 10, "dcsr": 11,
}
POLICY_NAMES = {v: k for k, v in POLICIES.items()}
HOT_PATH_POLICIES = ["identity", "nnz_sort", "plain_sort", "cta_aware", "hybrid_1", "hybrid_2_1"]

STATUS = {0: "SPMM_OK", 1: "SPMM_ERR_INVALID_ARG", 2: "SPMM_ERR_INVALID_CSR", 3: "SPMM_ERR_UNSUPPORTED",
          4: "SPMM_ERR_CUDA", 5: "SPMM_ERR_OOM", 6: "SPMM_ERR_STATE"}

FEATURE_NAMES = (["n_row", "n_col", "density"]
                 + [f"{n}_{s}" for n in ("nnz_per_row", "nnz_blocks_per_row", "warp_load", "same_cache_lines",
                                         "distinct_cache_lines_per_warp", "total_cache_lines_per_warp",
                                         "adjacent_vector_distance") for s in ("min", "mean", "max")])


class SpmmError(RuntimeError):
    def __init__(self, status: int, detail: str):
        self.status = status
        super().__init__(f"{STATUS.get(status, status)}: {detail}")


class _Params(ctypes.Structure):
    _fields_ = [("nw", ctypes.c_int32), ("nt", ctypes.c_int32), ("bw", ctypes.c_int32), ("split_nnz", ctypes.c_int32),
                ("window", ctypes.c_int64), ("preorder", ctypes.c_int32), ("fuse_rows", ctypes.c_int32),
                ("seed", ctypes.c_uint64)]


_lib = None
_ALLOC_T = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
_FREE_T = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p)
_alloc_cbs = None
EXPORTS = ["spmm_default_params", "spmm_set_allocator", "spmm_create", "spmm_permute", "spmm_prepare", "spmm_set_perm", "spmm_get_perm",
           "spmm_get_permuted_csr", "spmm_get_info", "spmm_get_schedule_info", "spmm_features", "spmm_features_b200", "spmm_run", "spmm_run_to", "spmm_run_ld", "spmm_run_multicast", "spmm_run_host", "spmm_run_host_batch", "spmm_predict", "spmm_predict_n",
           "spmm_partition_by_nnz", "spmm_destroy", "spmm_status_string", "spmm_last_error",
           "spmm_last_run_launches", "spmm_set_kernel_timing", "spmm_last_kernel_ms"]


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libspmm_b200.so (raises if missing -- there is no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise ImportError(f"{path} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(path)
    vp, i32, i64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    st = ctypes.c_int
    sig = {
        "spmm_default_params": (st, [vp]),
        "spmm_set_allocator": (st, [_ALLOC_T, _FREE_T, vp]),
        "spmm_create": (st, [vp, i64, i64, i64, vp, vp, vp, ctypes.c_int, vp]),
        "spmm_permute": (st, [vp, ctypes.c_int, vp, vp]),
        "spmm_prepare": (st, [vp, i64, vp, vp, vp]),
        "spmm_set_perm": (st, [vp, vp, vp, vp]),
        "spmm_get_perm": (st, [vp, vp]),
        "spmm_get_permuted_csr": (st, [vp, vp, vp, vp]),
        "spmm_get_info": (st, [vp, vp]),
        "spmm_get_schedule_info": (st, [vp, vp]),
        "spmm_features": (st, [vp, ctypes.c_int, vp, vp, vp]),
        "spmm_features_b200": (st, [vp, ctypes.c_int, i64, vp, vp]),
        "spmm_run": (st, [vp, vp, i64, vp, vp]),
        "spmm_run_to": (st, [vp, vp, i64, vp, i32, i64, vp]),
        "spmm_run_ld": (st, [vp, vp, i64, vp, i64, vp]),
        "spmm_run_multicast": (st, [vp, vp, i64, vp, i64, vp]),
        "spmm_run_host": (st, [vp, vp, i64, vp, vp]),
        "spmm_run_host_batch": (st, [vp, i64, vp, i64, vp, vp]),
        "spmm_predict": (st, [vp, vp, i64, i32, vp, vp]),
        "spmm_predict_n": (st, [vp, i32, vp, i64, i32, vp, vp]),
        "spmm_partition_by_nnz": (st, [vp, i64, i32, vp]),
        "spmm_destroy": (st, [vp]),
        "spmm_status_string": (ctypes.c_char_p, [st]),
        "spmm_last_error": (ctypes.c_char_p, []),
        "spmm_last_run_launches": (i32, []),
        "spmm_set_kernel_timing": (st, [vp, ctypes.c_int]),
        "spmm_last_kernel_ms": (st, [vp, vp]),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


def _check(status: int):
    if status != 0:
        raise SpmmError(status, load_library().spmm_last_error().decode(errors="replace"))


def use_torch_allocator(enable: bool = True):
    """Route the library's device allocations through torch's caching allocator (stream-ordered)."""
    global _alloc_cbs
    lib = load_library()
    if not enable:
        _check(lib.spmm_set_allocator(_ALLOC_T(), _FREE_T(), None))
        _alloc_cbs = None
        return
    import torch

    def _a(nbytes, stream, ctx):
        try:
            return torch.cuda.caching_allocator_alloc(int(nbytes), torch.cuda.current_device(), stream or 0)
        except Exception:   # noqa: BLE001 -- report as NULL -> SPMM_ERR_OOM
            return None

    def _f(ptr, stream, ctx):
        try:
            torch.cuda.caching_allocator_delete(ptr)
        except Exception:   # noqa: BLE001
            pass

    _alloc_cbs = (_ALLOC_T(_a), _FREE_T(_f))
    _check(lib.spmm_set_allocator(_alloc_cbs[0], _alloc_cbs[1], None))


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def make_params(nw=32, nt=32, bw=32, split_nnz=128, window=1024, preorder=0, seed=0, fuse_rows=0) -> _Params:
    p = _Params()
    _check(load_library().spmm_default_params(ctypes.byref(p)))
    p.nw, p.nt, p.bw, p.split_nnz, p.window, p.preorder, p.seed = nw, nt, bw, split_nnz, window, preorder, seed
    p.fuse_rows = fuse_rows
    return p


def _ptr(a):
    """(pointer, on_device, keepalive) of a numpy array or torch tensor."""
    if isinstance(a, np.ndarray):
        return a.ctypes.data, False, a
    return a.data_ptr(), bool(a.is_cuda), a


def _need(cond, msg):
    if not cond:
        raise ValueError(msg)


def _check_dense(t, name, rows, K=None, device=True, min_rows=None):
    """The C ABI takes raw pointers and cannot check buffer sizes or layouts: this is the one place they are
    checked (a transposed / non-contiguous / too small tensor would otherwise give a wrong C or write out of
    bounds).  rows: exact row count, or min_rows: at least that many."""
    import torch
    _need(isinstance(t, torch.Tensor), f"{name} must be a torch tensor")
    _need(t.is_cuda == device, f"{name} must be a {'CUDA' if device else 'host (CPU)'} tensor")
    _need(t.dtype == torch.float32, f"{name} must be float32, got {t.dtype}")
    _need(t.dim() == 2 and t.is_contiguous(), f"{name} must be a contiguous (row-major) 2-D tensor")
    if rows is not None:
        _need(t.shape[0] == rows, f"{name} must have {rows} rows, got {t.shape[0]}")
    if min_rows is not None:
        _need(t.shape[0] >= min_rows, f"{name} must have at least {min_rows} rows, got {t.shape[0]}")
    if K is not None:
        _need(t.shape[1] == K, f"{name} must have {K} columns, got {t.shape[1]}")


def _check_host(a, name, rows, K):
    """Host buffers of the end-to-end calls: numpy arrays or CPU tensors, float32, C-contiguous [rows, K]."""
    if isinstance(a, np.ndarray):
        _need(a.dtype == np.float32 and a.ndim == 2 and a.flags.c_contiguous, f"{name} must be C-contiguous float32 2-D")
        _need(a.shape == (rows, K), f"{name} must be [{rows}, {K}], got {list(a.shape)}")
    else:
        _check_dense(a, name, rows, K, device=False)


_live = weakref.WeakSet()


class SpMM:
    """One spmm_handle: create (a1) -> permute (a2-a7) -> run (a8) / features (a9)."""

    def __init__(self, M, N, rowidx, colidx, value, stream=None):
        import torch  # noqa: F401  (device / stream plumbing)
        lib = load_library()
        if isinstance(rowidx, np.ndarray):
            rowidx = np.ascontiguousarray(rowidx, dtype=np.int64)
            colidx = np.ascontiguousarray(colidx, dtype=np.int32)
            value = np.ascontiguousarray(value, dtype=np.float32)
        else:   # torch tensors: the library reads raw int64 / int32 / float32 arrays of these lengths
            import torch
            _need(rowidx.dtype == torch.int64 and colidx.dtype == torch.int32 and value.dtype == torch.float32,
                  "rowidx / colidx / value must be int64 / int32 / float32")
            _need(all(t.is_contiguous() and t.dim() == 1 for t in (rowidx, colidx, value)),
                  "rowidx / colidx / value must be contiguous 1-D tensors")
            _need(rowidx.is_cuda == colidx.is_cuda == value.is_cuda, "CSR arrays must all be on the same side")
        _need(len(rowidx) == int(M) + 1, f"rowidx must have M + 1 = {int(M) + 1} entries")
        _need(len(colidx) >= (int(rowidx[-1]) if M > 0 else 0) and len(value) == len(colidx),
              "colidx / value must hold rowidx[M] entries")
        r, on_dev, _k1 = _ptr(rowidx)
        c, _, _k2 = _ptr(colidx)
        v, _, _k3 = _ptr(value)
        nnz = int(rowidx[-1]) if M > 0 else 0
        self._h = ctypes.c_void_p()
        self.M, self.N, self.nnz = int(M), int(N), nnz
        _check(lib.spmm_create(ctypes.byref(self._h), self.M, self.N, nnz, r, c, v, int(on_dev), _stream_ptr(stream)))
        self.policy = "identity"
        _live.add(self)

    @classmethod
    def from_csr(cls, csr, stream=None):
        return cls(csr.M, csr.N, csr.rowidx, csr.colidx, csr.value, stream=stream)

    def permute(self, policy, stream=None, **params):
        """spmm_permute.  policy: a name of POLICIES, optionally with a pre-order suffix for the chain policies --
        "+md" (median-block pre-order, preorder = 2) or "+mh" (MinHash pre-order, preorder = 1, seed 1 unless given)."""
        if isinstance(policy, str) and policy.endswith(("+md", "+mh")):
            params.setdefault("preorder", 2 if policy.endswith("+md") else 1)
            if policy.endswith("+mh"):
                params.setdefault("seed", 1)
            policy = policy[:-3]
        pid = POLICIES[policy] if isinstance(policy, str) else int(policy)
        p = make_params(**params)
        _check(load_library().spmm_permute(self._h, pid, ctypes.byref(p), _stream_ptr(stream)))
        self.policy = POLICY_NAMES[pid]
        return self

    def prepare(self, K, B=None, C=None, stream=None):
        """spmm_prepare: build the run schedule of K's lane geometry now, so spmm_run with this K is asynchronous
        (B / C: the buffers the runs will use -- only their alignment matters; None = aligned)."""
        _check(load_library().spmm_prepare(self._h, int(K), None if B is None else B.data_ptr(),
                                           None if C is None else C.data_ptr(), _stream_ptr(stream)))
        return self

    def set_perm(self, perm, stream=None, **params):
        """spmm_set_perm: install a caller-supplied permutation (perm[p] = original row at position p), e.g. one
        cached from an earlier spmm_permute (permcache.py)."""
        pm = np.ascontiguousarray(perm, dtype=np.int32)
        _need(pm.shape == (self.M,), f"perm must have M = {self.M} entries")
        p = make_params(**params)
        _check(load_library().spmm_set_perm(self._h, pm.ctypes.data, ctypes.byref(p), _stream_ptr(stream)))
        self.policy = "custom"
        return self

    def perm(self) -> np.ndarray:
        out = np.empty(self.M, dtype=np.int32)
        _check(load_library().spmm_get_perm(self._h, out.ctypes.data))
        return out

    def permuted_csr(self):
        r = np.empty(self.M + 1, dtype=np.int64)
        c = np.empty(self.nnz, dtype=np.int32)
        v = np.empty(self.nnz, dtype=np.float32)
        _check(load_library().spmm_get_permuted_csr(self._h, r.ctypes.data, c.ctypes.data, v.ctypes.data))
        return r, c, v

    def info(self) -> dict:
        out = np.empty(5, dtype=np.int64)
        _check(load_library().spmm_get_info(self._h, out.ctypes.data))
        return dict(empty_rows=int(out[0]), whole_rows=int(out[1]), split_rows=int(out[2]), chunks=int(out[3]),
                    max_row_nnz=int(out[4]))

    def schedule_info(self) -> dict:
        """The a7 run schedule of the most recent run (spmm_get_schedule_info)."""
        out = np.empty(6, dtype=np.int64)
        _check(load_library().spmm_get_schedule_info(self._h, out.ctypes.data))
        return dict(rows_per_task=int(out[0]), fuse=int(out[1]), tasks=int(out[2]), groups=int(out[3]),
                    records=int(out[4]), fused_nnz=int(out[5]))

    def features(self, current_order=False, nw=32, nt=32, bw=32, stream=None) -> np.ndarray:
        out = np.empty(24, dtype=np.float64)
        p = make_params(nw=nw, nt=nt, bw=bw, window=0)
        _check(load_library().spmm_features(self._h, int(bool(current_order)), ctypes.byref(p), out.ctypes.data,
                                            _stream_ptr(stream)))
        return out

    def features_b200(self, K, current_order=False, stream=None) -> np.ndarray:
        """The 7 B200 platform features g0..g6 (spmm_features_b200) for right-hand-side width K."""
        out = np.empty(7, dtype=np.float64)
        _check(load_library().spmm_features_b200(self._h, int(bool(current_order)), int(K), out.ctypes.data,
                                                 _stream_ptr(stream)))
        return out

    def run(self, B, C=None, stream=None):
        """C = A.B on the device (B: cuda float32 [N, K] row-major). Returns C (cuda float32 [M, K])."""
        import torch
        _check_dense(B, "B", self.N)
        K = int(B.shape[1])
        if C is None:
            C = torch.empty((self.M, K), dtype=torch.float32, device=B.device)
        _check_dense(C, "C", self.M, K)
        _need(C.device == B.device, "B and C must be on the same device")
        _check(load_library().spmm_run(self._h, B.data_ptr(), K, C.data_ptr(), _stream_ptr(stream)))
        return C

    def run_to(self, B, dsts, row_offset=0, stream=None):
        """spmm_run_to: this handle's C rows stored to every destination buffer (cuda float32 [>= row_offset + M, K]
        tensors, or raw device / peer-mapped pointers as ints) at rows row_offset + r -- the C all-gather fused
        into the SpMM epilogue."""
        _check_dense(B, "B", self.N)
        K = int(B.shape[1])
        for d in dsts:
            if not isinstance(d, int):   # raw (peer) pointers are the caller's responsibility
                _check_dense(d, "destination", None, K, min_rows=int(row_offset) + self.M)
        ptrs = [d if isinstance(d, int) else d.data_ptr() for d in dsts]
        arr = (ctypes.c_void_p * len(ptrs))(*ptrs)
        _check(load_library().spmm_run_to(self._h, B.data_ptr(), K, arr, len(ptrs), int(row_offset),
                                          _stream_ptr(stream)))
        return dsts

    def run_ld(self, B, C, col_offset=0, stream=None):
        """spmm_run_ld: C[:, col_offset:col_offset + K] = A.B for a wider row-major C (cuda float32 [M, ldc]); the
        other columns are untouched (column blocks of C, e.g. chunks of a B that arrives in pieces)."""
        _check_dense(B, "B", self.N)
        K = int(B.shape[1])
        _check_dense(C, "C", self.M)
        ldc = int(C.shape[1])
        _need(0 <= int(col_offset) and int(col_offset) + K <= ldc, "column block outside C")
        _check(load_library().spmm_run_ld(self._h, B.data_ptr(), K, C.data_ptr() + 4 * int(col_offset), ldc,
                                          _stream_ptr(stream)))
        return C

    def run_multicast(self, B, C_mc, row_offset=0, stream=None):
        """spmm_run_multicast: this handle's C rows stored once through an NVLS multicast address (int: e.g. torch
        symmetric memory's multicast_ptr) at rows row_offset + r of the group-wide buffer."""
        _check_dense(B, "B", self.N)
        _need(isinstance(C_mc, int) and C_mc != 0, "C_mc must be a (nonzero) multicast device address")
        _check(load_library().spmm_run_multicast(self._h, B.data_ptr(), int(B.shape[1]), C_mc, int(row_offset),
                                                 _stream_ptr(stream)))

    def run_host(self, B_host, C_host, stream=None):
        """End-to-end: host B -> device, SpMM, device -> host C (host buffers, ideally pinned)."""
        K = int(B_host.shape[1])
        _check_host(B_host, "B_host", self.N, K)
        _check_host(C_host, "C_host", self.M, K)
        b, _, _ = _ptr(B_host)
        c, _, _ = _ptr(C_host)
        _check(load_library().spmm_run_host(self._h, b, K, c, _stream_ptr(stream)))
        return C_host

    def run_host_batch(self, Bs, Cs, stream=None):
        """Pipelined end-to-end over a list of host B's (pinned) into a list of host C's (spmm_run_host_batch):
        the H2D of the next B and the D2H of the previous C overlap the current SpMM."""
        assert len(Bs) == len(Cs)
        n = len(Bs)
        if n == 0:
            return Cs
        K = int(Bs[0].shape[1])
        for b, c in zip(Bs, Cs):
            _check_host(b, "B_host", self.N, K)
            _check_host(c, "C_host", self.M, K)
        bp = (ctypes.c_void_p * n)(*[_ptr(b)[0] for b in Bs])
        cp = (ctypes.c_void_p * n)(*[_ptr(c)[0] for c in Cs])
        _check(load_library().spmm_run_host_batch(self._h, n, bp, K, cp, _stream_ptr(stream)))
        return Cs

    @staticmethod
    def last_run_launches() -> int:
        return int(load_library().spmm_last_run_launches())

    def set_kernel_timing(self, enable: bool = True):
        """CUDA events around the main SpMM kernel of every run (spmm_set_kernel_timing)."""
        _check(load_library().spmm_set_kernel_timing(self._h, int(bool(enable))))

    def last_kernel_ms(self) -> float:
        """Duration of the main SpMM kernel of the most recent run (synchronises its end event)."""
        ms = ctypes.c_float(0.0)
        _check(load_library().spmm_last_kernel_ms(self._h, ctypes.byref(ms)))
        return float(ms.value)

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            load_library().spmm_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:   # noqa: BLE001 -- interpreter shutdown
            pass


@atexit.register
def _close_all():
    for h in list(_live):
        try:
            h.close()
        except Exception:   # noqa: BLE001
            pass


def spmm_predict(features, weights, n_policies):
    """Predictor inference in the library: returns (policy id, predicted times)."""
    f = np.ascontiguousarray(features, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float32)
    pol = ctypes.c_int32()
    times = np.empty(n_policies, dtype=np.float64)
    _check(load_library().spmm_predict(f.ctypes.data, w.ctypes.data, len(w), n_policies, ctypes.byref(pol),
                                       times.ctypes.data))
    return int(pol.value), times


def spmm_predict_n(features, weights, n_policies):
    """spmm_predict for any number of input features (e.g. 24 Table II + 7 B200 features)."""
    f = np.ascontiguousarray(features, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float32)
    pol = ctypes.c_int32()
    times = np.empty(n_policies, dtype=np.float64)
    _check(load_library().spmm_predict_n(f.ctypes.data, len(f), w.ctypes.data, len(w), n_policies, ctypes.byref(pol),
                                         times.ctypes.data))
    return int(pol.value), times


# classes of the bundled predictor (reading A20): the hot-path policies plus CTA-aware over the median-block
# pre-order (round 2: the corpus' shuffled matrices make the pre-order the most frequent winner)
PREDICTOR_POLICIES = HOT_PATH_POLICIES + ["cta_aware+md"]
PAPER4_POLICIES = ["identity", "dcsr", "lpt", "warp_aware"]   # the paper's four classes


def predictor_weights(K: int, paper_classes: bool = False, b200: bool = False) -> np.ndarray:
    """Bundled MLP weights (spmm_predict layout) trained on the C4 corpus for the nearest trained K
    (b200: the 31-feature model with the B200 platform features, f4)."""
    d = os.path.join(_HERE, "predictor4" if paper_classes else ("predictor_b200" if b200 else "predictor"))
    ks = sorted(int(f[5:-4]) for f in os.listdir(d) if f.startswith("mlp_K") and f.endswith(".npy"))
    k = min(ks, key=lambda x: (abs(np.log2(x) - np.log2(K)), x))
    return np.load(os.path.join(d, f"mlp_K{k}.npy"))


def select_policy(h: "SpMM", K: int, paper_classes: bool = False, b200: bool = False) -> str:
    """a10 predicted selection: features of the original order on the GPU (spmm_features), MLP inference
    in the library (spmm_predict), argmin of the predicted times.  b200: the 24 features plus
    the 7 B200 platform features (spmm_features_b200, f4) through spmm_predict_n."""
    classes = PAPER4_POLICIES if paper_classes else PREDICTOR_POLICIES
    if b200 and not paper_classes:
        f = np.concatenate([h.features(current_order=False), h.features_b200(K, current_order=False)])
        pol, _ = spmm_predict_n(f, predictor_weights(K, b200=True), len(classes))
        return classes[pol]
    pol, _ = spmm_predict(h.features(current_order=False), predictor_weights(K, paper_classes), len(classes))
    return classes[pol]


def spmm_partition_by_nnz(rowidx, P: int) -> np.ndarray:
    r = np.ascontiguousarray(rowidx, dtype=np.int64)
    b = np.empty(P + 1, dtype=np.int64)
    _check(load_library().spmm_partition_by_nnz(r.ctypes.data, len(r) - 1, P, b.ctypes.data))
    return b


def spmm_create(M, N, rowidx, colidx, value, stream=None) -> SpMM:
    return SpMM(M, N, rowidx, colidx, value, stream=stream)


def spmm_permute(h: SpMM, policy, stream=None, **params) -> SpMM:
    return h.permute(policy, stream=stream, **params)


def spmm_run(h: SpMM, B, C=None, stream=None):
    return h.run(B, C, stream=stream)


def spmm_features(h: SpMM, current_order=False, **kw):
    return h.features(current_order, **kw)


def spmm_destroy(h: SpMM):
    h.close()
