"""On-disk cache of row permutations (SURVEY.md §5 checkpoint / resume; "row permutations happen offline
or the cost is amortized").  A permutation is a pure function of the CSR's structure (rowidx, colidx), the policy
and its parameters, so it is stored under a SHA-256 of exactly those bytes and reinstalled with spmm_set_perm --
an expensive build (an exact whole-matrix chain, W = 0: 7-60 s at M = 1-4M) is paid once per matrix.

  perm, hit = permcache.permute_cached(h, csr, "hybrid_2_1", cache_dir, window=0)
"""
from __future__ import annotations

import hashlib
import json
import os

import numpy as np


def cache_key(rowidx, colidx, policy: str, params: dict) -> str:
    h = hashlib.sha256()
    h.update(b"spmm-perm-v1")
    for a, dt in ((rowidx, np.int64), (colidx, np.int32)):
        h.update(np.ascontiguousarray(a, dtype=dt).tobytes())
    h.update(json.dumps({"policy": policy, **{k: int(v) for k, v in sorted(params.items())}}, sort_keys=True).encode())
    return h.hexdigest()


def permute_cached(h, csr, policy: str, cache_dir: str, **params):
    """h.permute(policy, **params) through the cache: on a hit the stored permutation is installed with
    spmm_set_perm (bit-identical to a fresh build -- the builders are deterministic); on a miss the permutation is
    built and stored.  csr: the host CSR the handle was created from (its structure is the key).  Returns
    (perm, hit)."""
    os.makedirs(cache_dir, exist_ok=True)
    key = cache_key(csr.rowidx, csr.colidx, policy, params)
    path = os.path.join(cache_dir, f"perm_{key}.npy")
    split = {k: v for k, v in params.items() if k == "split_nnz"}
    if os.path.exists(path):
        perm = np.load(path)
        h.set_perm(perm, **split)
        h.policy = policy
        return perm, True
    h.permute(policy, **params)
    perm = h.perm()
    tmp = path + f".tmp{os.getpid()}.npy"
    np.save(tmp, perm)
    os.replace(tmp, path)
    return perm, False
