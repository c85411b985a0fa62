"""Implementation-independent checkers used to pin the oracle (and, on GPU, the kernels).

These do NOT recompute the greedy orders; they verify properties the paper's
definitions fix (§III), using Python-int bit masks for the Hamming
distance ("bit mask ... ceil(N/32) bits ... Hamming distance (XOR)")
instead of the oracle's sorted-list merge.
"""
from __future__ import annotations

import numpy as np


def row_masks(csr, bw=32):
    """Python-int bit masks, bit b set iff the row has a nnz in columns [b*bw, (b+1)*bw)."""
    masks = []
    for i in range(csr.M):
        m = 0
        for c in csr.colidx[csr.rowidx[i]:csr.rowidx[i + 1]]:
            m |= 1 << (int(c) // bw)
        masks.append(m)
    return masks


def popham(a: int, b: int) -> int:
    return bin(a ^ b).count("1")


def nnz_rows(csr):
    return np.diff(csr.rowidx).astype(np.int64)


def wl_rows(csr, nt=32):
    n = nnz_rows(csr)
    return (n + nt - 1) // nt


def is_bijection(perm, M):
    return len(perm) == M and np.array_equal(np.sort(np.asarray(perm, dtype=np.int64)), np.arange(M))


def check_sorted_desc_stable(perm, key):
    """key non-increasing along perm; equal keys in ascending row id (readings A1, A2)."""
    k = np.asarray(key)[perm]
    assert np.all(k[:-1] >= k[1:]), "key not non-increasing"
    eq = k[:-1] == k[1:]
    p = np.asarray(perm)
    assert np.all(p[:-1][eq] < p[1:][eq]), "ties not in ascending row id"


def windows_of(M, W, pre=None):
    W = M if (W == 0 or W > M) else W
    pre = np.arange(M) if pre is None else np.asarray(pre)
    return [pre[s:s + W] for s in range(0, M, W)] if M else []


def check_chain_local_optimality(perm, csr, mode, nw=32, nt=32, bw=32, W=0, pre=None, segments=None):
    """At every greedy step the chosen row minimises the policy key over the still-unplaced rows of
    its window / segment (P:L118-134 definitions, readings A6-A11).  Brute force, O(W^2) per window.

    mode: 'cta' | 'h21' | 'h22' | 'h1' | 'warp' | 'h23'
    segments: list of (start, end) position ranges (h1); else windows of W over `pre`.
    """
    masks = row_masks(csr, bw)
    wl = wl_rows(csr, nt)
    perm = np.asarray(perm)
    if segments is None:
        segs = []
        s = 0
        for w in windows_of(csr.M, W, pre):
            segs.append((s, s + len(w), set(int(x) for x in w)))
            s += len(w)
    else:
        segs = [(a, b, set(int(x) for x in perm[a:b])) for a, b in segments]
    for a, b, members in segs:
        out = [int(x) for x in perm[a:b]]
        assert set(out) == members, "window content changed"
        n = len(out)
        if n == 0:
            continue
        if mode in ("warp", "h23"):
            nf = min(nw, n)
            first = sorted(members, key=lambda r: (wl[r], r))[:nf]
            assert out[:nf] == first, "warp-aware initial rows must be the lowest (wl, id)"
            q0 = nf
        elif mode == "h1":
            q0 = 1
        else:
            assert out[0] == min(members, key=lambda r: (wl[r], r)), "chain must start at lowest (wl, id)"
            q0 = 1
        unplaced = set(members) - set(out[:q0])
        for q in range(q0, n):
            def key(r):
                if mode in ("cta", "h1"):
                    return (popham(masks[r], masks[out[q - 1]]), 0, r)
                if mode == "h21":
                    return (popham(masks[r], masks[out[q - 1]]), abs(int(wl[r]) - int(wl[out[q - 1]])), r)
                if mode == "h22":
                    return (popham(masks[r], masks[out[q - 1]]),
                            popham(masks[r], masks[out[q - nw]]) if q >= nw else 0, r)
                if mode == "warp":
                    return (popham(masks[r], masks[out[q - nw]]), 0, r)
                return (popham(masks[r], masks[out[q - nw]]), abs(int(wl[r]) - int(wl[out[q - 1]])), r)
            best = min(unplaced, key=key)
            assert out[q] == best, f"step {q}: chose {out[q]} key {key(out[q])}, best {best} key {key(best)}"
            unplaced.remove(out[q])


def hybrid1_segments(perm_plain, wl, W):
    """Maximal runs of equal wl in Plain-Sort order, cut into W-sized pieces (reading A8)."""
    M = len(perm_plain)
    W = M if (W == 0 or W > M) else W
    segs, run_start = [], 0
    starts = []
    for p in range(M):
        if p > 0 and wl[perm_plain[p]] != wl[perm_plain[p - 1]]:
            run_start = p
        if p == run_start or (p - run_start) % W == 0:
            starts.append(p)
    starts.append(M)
    for t in range(len(starts) - 1):
        segs.append((starts[t], starts[t + 1]))
    return segs


def warp_loads(perm, wl, nw):
    loads = np.zeros(nw, dtype=np.int64)
    for p, r in enumerate(perm):
        loads[p % nw] += wl[r]
    return loads


def check_lpt(perm, wl, nw):
    """Replay the assignment implied by perm (row at position p is on warp p mod nw, list order
    p div nw) in Plain-Sort order and verify every row went to a least-loaded non-full warp."""
    M = len(perm)
    order = sorted(range(M), key=lambda r: (-wl[r], r))
    warp_of = {int(r): p % nw for p, r in enumerate(perm)}
    slot_of = {int(r): p // nw for p, r in enumerate(perm)}
    cap = [len(range(w, M, nw)) for w in range(nw)]
    load = [0] * nw
    cnt = [0] * nw
    for r in order:
        w = warp_of[r]
        assert slot_of[r] == cnt[w], "rows must fill a warp's slots in assignment order"
        cands = [x for x in range(nw) if cnt[x] < cap[x]]
        mn = min(load[x] for x in cands)
        assert load[w] == mn and w == min(x for x in cands if load[x] == mn), "not the least-loaded warp"
        load[w] += wl[r]
        cnt[w] += 1
