"""Pins for the oracle's row permutations (oracle.c, §III) -- CPU only.

Pins: worked examples E1/E2 (tests/golden), bijection, sort-order properties
(readings A1-A3), the 27-point-stencil closed form, brute-force local optimality
of every greedy step with Python-int bit-mask Hamming distances (independent of
the oracle's sorted-list merge), the planted block-cluster structure, LPT's
least-loaded-warp property and the Fig. 7 warp-load example.
"""
import numpy as np
import pytest

import oracle
import synthetic as syn
import checkers as ck


def e1_csr(e1):
    return syn.from_lists(e1["M"], e1["N"], e1["rows"])


def test_e1_row_quantities(e1):
    a = e1_csr(e1)
    assert ck.nnz_rows(a).tolist() == e1["nnz"]
    assert ck.wl_rows(a, e1["nt"]).tolist() == e1["wl"]
    masks = ck.row_masks(a, e1["bw"])
    assert [[b for b in range(8) if m >> b & 1] for m in masks] == e1["blocks"]


@pytest.mark.parametrize("name", ["identity", "plain_sort", "nnz_sort", "flipped", "lpt", "cta_aware",
                                  "cta_aware_w4", "hybrid_2_1", "hybrid_2_2", "warp_aware", "hybrid_2_3",
                                  "hybrid_1", "dcsr"])
def test_e1_perms(e1, name):
    a = e1_csr(e1)
    spec = e1["perm"][name]
    policy = spec.get("policy", name)
    perm = oracle.permute(a, policy, nw=e1["nw"], nt=e1["nt"], bw=e1["bw"], window=spec["window"])
    assert perm.tolist() == spec["perm"]
    assert ck.warp_loads(perm, e1["wl"], e1["nw"]).tolist() == spec["warp_loads"]


def test_e1_permuted_csr(e1):
    a = e1_csr(e1)
    perm = oracle.permute(a, "plain_sort", nw=2, nt=2, bw=2)
    r2, c2, _ = oracle.permuted_csr(a, perm)
    assert r2.tolist() == e1["plain_sort_permuted_csr"]["rowidx"]
    assert c2.tolist() == e1["plain_sort_permuted_csr"]["colidx"]


def test_e2_lpt_capacity(e2):
    a = syn.from_lists(len(e2["rows"]), e2["N"], e2["rows"])
    perm = oracle.permute(a, "lpt", nw=e2["nw"], nt=e2["nt"], bw=e2["bw"])
    assert perm.tolist() == e2["lpt_perm"]
    assert ck.warp_loads(perm, e2["wl"], e2["nw"]).tolist() == e2["lpt_warp_loads"]


def test_fig7_lpt_balances(paper_arith):
    """warp loads 12,13,10,10 -> 12,11,11,11 under LPT (sum 45 invariant; max = ceil(45/4))."""
    before = paper_arith["fig7_warp_loads"]["before"]
    after = paper_arith["fig7_warp_loads"]["after"]
    nw = 4
    # a 48-row matrix with nt = 32 whose row-wise warp loads give the Fig. 7 "before" per-warp loads
    wl_rows = []
    per_warp = [[1] * 12, [1] * 11 + [2], [1] * 10 + [0, 0], [1] * 10 + [0, 0]]
    for k in range(12):
        for w in range(nw):
            wl_rows.append(per_warp[w][k])
    rows = [list(range(32 * (w - 1) + 1)) if w > 0 else [] for w in wl_rows]
    a = syn.from_lists(48, 64, rows)
    wl = ck.wl_rows(a, 32)
    assert ck.warp_loads(np.arange(48), wl, nw).tolist() == before
    perm = oracle.permute(a, "lpt", nw=nw, nt=32, bw=32)
    loads = ck.warp_loads(perm, wl, nw)
    assert loads.sum() == sum(before) == sum(after) == 45
    assert sorted(loads.tolist(), reverse=True) == sorted(after, reverse=True)
    ck.check_lpt(perm, wl.tolist(), nw)


GENS = {
    "rmat": lambda: syn.rmat(9, 6, 31, "natural"),
    "rmat_rl": lambda: syn.rmat(9, 6, 32, "random-label"),
    "block": lambda: syn.blockcluster(400, 3000, 16, 3, 6, 33),
    "uniform": lambda: syn.uniform(300, 1000, 5, 34, poisson=True),
    "stencil": lambda: syn.stencil27(6, 35),
}


@pytest.mark.parametrize("gen", list(GENS))
@pytest.mark.parametrize("policy", list(oracle.POLICIES))
def test_bijection(gen, policy):
    a = GENS[gen]()
    perm = oracle.permute(a, policy, window=64)
    assert ck.is_bijection(perm, a.M)


@pytest.mark.parametrize("gen", list(GENS))
def test_sort_properties(gen):
    a = GENS[gen]()
    ck.check_sorted_desc_stable(oracle.permute(a, "nnz_sort"), ck.nnz_rows(a))
    ck.check_sorted_desc_stable(oracle.permute(a, "plain_sort"), ck.wl_rows(a))


def test_stencil_sorts_closed_form():
    """27-point stencil: every wl = 1 so Plain Sort is the identity (A3); nnz sort = interior (27),
    faces (18), edges (12), corners (8), each class in original order."""
    n = 7
    a = syn.stencil27(n, 1)
    assert np.array_equal(oracle.permute(a, "plain_sort"), np.arange(a.M))
    perm = oracle.permute(a, "nnz_sort")
    nz = ck.nnz_rows(a)
    counts = [(n - 2) ** 3, 6 * (n - 2) ** 2, 12 * (n - 2), 8]
    off = 0
    for val, cnt in zip([27, 18, 12, 8], counts):
        seg = perm[off:off + cnt]
        assert np.all(nz[seg] == val) and np.all(np.diff(seg) > 0)
        off += cnt
    assert off == a.M


@pytest.mark.parametrize("gen", ["rmat", "block", "uniform"])
@pytest.mark.parametrize("W", [0, 32, 64])
@pytest.mark.parametrize("policy,mode", [("cta_aware", "cta"), ("hybrid_2_1", "h21"), ("hybrid_2_2", "h22"),
                                         ("warp_aware", "warp"), ("hybrid_2_3", "h23")])
def test_chain_local_optimality(gen, W, policy, mode):
    a = GENS[gen]()
    if W == 0:   # keep the brute-force checker small
        a = syn.CSR(min(a.M, 96), a.N, a.rowidx[:min(a.M, 96) + 1].copy(), a.colidx, a.value)
        a.colidx = a.colidx[:a.rowidx[-1]]
        a.value = a.value[:a.rowidx[-1]]
    nw = 8
    perm = oracle.permute(a, policy, nw=nw, window=W)
    ck.check_chain_local_optimality(perm, a, mode, nw=nw, W=W)


@pytest.mark.parametrize("W", [0, 32, 96])
def test_hybrid1_local_optimality(W):
    a = syn.rmat(9, 6, 41, "natural")
    wl = ck.wl_rows(a).tolist()
    plain = oracle.permute(a, "plain_sort")
    perm = oracle.permute(a, "hybrid_1", nw=32, window=W)
    segs = ck.hybrid1_segments(plain.tolist(), wl, W)
    # each segment holds exactly Plain Sort's rows for that range, starting with its first row
    for s, e in segs:
        assert set(perm[s:e].tolist()) == set(plain[s:e].tolist())
        assert perm[s] == plain[s]
    ck.check_chain_local_optimality(perm, a, "h1", nw=32, segments=segs)


def test_minhash_preorder_chain():
    a = syn.blockcluster(256, 4096, 16, 3, 6, 45)
    h = oracle.minhash_keys(a, bw=32, seed=7)
    pre = np.lexsort((np.arange(a.M), h))
    perm = oracle.permute(a, "cta_aware", nw=8, window=64, preorder=1, seed=7)
    ck.check_chain_local_optimality(perm, a, "cta", nw=8, W=64, pre=pre)


def test_median_block_keys_by_hand(e1):
    # E1 with bw = 2: blocks r0 {0,1,2} -> 1, r1 {3} -> 3, r2 {} -> 2^64-1, r3 {0,1} -> 0, r4 {2,3} -> 2,
    # r5 {0} -> 0, r6 {2,3} -> 2, r7 {0,1,3} -> 1 (lower median of the sorted distinct blocks)
    a = e1_csr(e1)
    assert oracle.median_block_keys(a, bw=2).tolist() == [1, 3, 2 ** 64 - 1, 0, 2, 0, 2, 1]


def test_median_block_keys_bruteforce():
    a = syn.rmat(10, 9, 46, "local")
    ref = []
    for i in range(a.M):
        b = sorted(set((a.colidx[a.rowidx[i]:a.rowidx[i + 1]] // 32).tolist()))
        ref.append(b[(len(b) - 1) // 2] if b else 2 ** 64 - 1)
    assert oracle.median_block_keys(a).tolist() == ref


@pytest.mark.parametrize("policy,mode", [("cta_aware", "cta"), ("hybrid_2_1", "h21")])
def test_median_preorder_chain(policy, mode):
    """preorder = 2: windows over the stable (median block, id) order; every greedy step locally optimal."""
    a = syn.rmat(10, 9, 47, "local")
    pre = np.lexsort((np.arange(a.M), oracle.median_block_keys(a)))
    perm = oracle.permute(a, policy, nw=8, window=64, preorder=2)
    ck.check_chain_local_optimality(perm, a, mode, nw=8, W=64, pre=pre)


def test_minhash_splitmix_vector():
    """splitmix64 test vector: the first output of the splitmix64 generator seeded with 0 is
    0xE220A8397B1DCDAF (= finaliser(0) with the golden-gamma pre-add).  A one-row matrix whose
    single block id is 0 with seed 0 must therefore get that key."""
    a = syn.from_lists(2, 64, [[3], []])
    h = oracle.minhash_keys(a, bw=32, seed=0)
    assert int(h[0]) == 0xE220A8397B1DCDAF
    assert int(h[1]) == 2 ** 64 - 1


MASK64 = (1 << 64) - 1


def _splitmix64_py(z):
    """Python-int splitmix64 (z + golden gamma, then the two xor-shift-multiplies and a final xor-shift), pinned
    below by the generator's published outputs -- independent of oracle.c's uint64 arithmetic."""
    z = (z + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def test_splitmix_python_matches_published_vectors(golden):
    g = golden("splitmix64")
    gamma = int(g["golden_gamma"], 16)
    for k, v in enumerate(g["outputs_seed0"]):
        assert _splitmix64_py((k * gamma) & MASK64) == int(v, 16)


def test_minhash_published_vectors_through_seed(golden):
    """One-block rows whose block id b XOR seed is (k-1)*gamma get the generator's k-th published output: pins the
    seed XOR (a dropped seed gives finaliser(b) instead) and the hash itself against tests/golden/splitmix64.json."""
    g = golden("splitmix64")
    gamma = int(g["golden_gamma"], 16)
    a = syn.from_lists(1, 256, [[3 * 32 + 5]])          # block 3 (bw = 32)
    for k, v in enumerate(g["outputs_seed0"]):
        seed = 3 ^ ((k * gamma) & MASK64)
        assert int(oracle.minhash_keys(a, bw=32, seed=seed)[0]) == int(v, 16), k


@pytest.mark.parametrize("seed", [0, 7, 0xDEADBEEF12345, 2 ** 64 - 3])
def test_minhash_min_over_blocks_bruteforce(seed):
    """h_i = min over b in blocks_i of splitmix64(b XOR seed), recomputed with Python ints over
    multi-block rows (R-MAT rows touch up to hundreds of blocks): a max instead of the min, a dropped seed, a wrong
    block width or a per-column (not per-block) hash all fail here."""
    a = syn.rmat(10, 9, 48, "natural")
    h = oracle.minhash_keys(a, bw=32, seed=seed)
    nblk = 0
    for i in range(a.M):
        blocks = sorted(set((a.colidx[a.rowidx[i]:a.rowidx[i + 1]] // 32).tolist()))
        nblk = max(nblk, len(blocks))
        ref = min((_splitmix64_py(b ^ seed) for b in blocks), default=MASK64)
        assert int(h[i]) == ref, (i, blocks)
    assert nblk >= 3


def test_minhash_invariants():
    """Hash-value-free properties: a row's key is the min of the keys of its one-block sub-rows; the key of block b
    under seed s is the seed-0 key of block b XOR s."""
    rows = [[0, 33, 70, 100, 200], [5, 64 + 1], [230], []]
    a = syn.from_lists(4, 256, rows)
    for s in (0, 5, 6):
        h = oracle.minhash_keys(a, bw=32, seed=s)
        for i, r in enumerate(rows):
            singles = syn.from_lists(len(r), 256, [[c] for c in r]) if r else None
            hs = oracle.minhash_keys(singles, bw=32, seed=s) if r else np.array([MASK64], dtype=np.uint64)
            assert int(h[i]) == int(hs.min())
        for b in range(8):
            one = syn.from_lists(1, 256, [[32 * b]])
            x = syn.from_lists(1, 256, [[32 * (b ^ s)]])
            assert int(oracle.minhash_keys(one, bw=32, seed=s)[0]) == int(oracle.minhash_keys(x, bw=32, seed=0)[0])
    # a two-block row where the larger hash is not the min: max-instead-of-min changes the key
    two = syn.from_lists(1, 256, [[0, 32]])
    k0 = int(oracle.minhash_keys(syn.from_lists(1, 256, [[0]]), bw=32, seed=0)[0])
    k1 = int(oracle.minhash_keys(syn.from_lists(1, 256, [[32]]), bw=32, seed=0)[0])
    assert k0 != k1 and int(oracle.minhash_keys(two, bw=32, seed=0)[0]) == min(k0, k1)


def test_planted_clusters_contiguous():
    """Planted block-clustered matrix (identical masks within a group, disjoint across groups):
    CTA-aware with W=0 keeps every group contiguous, so the chain crosses groups exactly G-1 times."""
    g, c, G = 16, 3, 12
    a = syn.blockcluster(g * G, 4096, g, c, 8, 51, planted=True)
    masks = ck.row_masks(a)
    groups = {}
    for i, m in enumerate(masks):
        groups.setdefault(m, []).append(i)
    assert len(groups) == G
    perm = oracle.permute(a, "cta_aware", nw=32, window=0)
    label = [masks[r] for r in perm]
    crossings = sum(1 for p in range(1, len(label)) if label[p] != label[p - 1])
    assert crossings == G - 1


def test_flipped_structure():
    a = syn.rmat(9, 6, 61, "natural")
    nw = 32
    plain = oracle.permute(a, "plain_sort", nw=nw)
    fl = oracle.permute(a, "flipped", nw=nw)
    for cidx, s in enumerate(range(0, a.M, nw)):
        chunk = plain[s:s + nw]
        exp = chunk[::-1] if cidx % 2 else chunk
        assert np.array_equal(fl[s:s + nw], exp)


@pytest.mark.parametrize("gen", ["rmat", "uniform"])
def test_lpt_property(gen):
    a = GENS[gen]()
    nw = 8
    wl = ck.wl_rows(a).tolist()
    perm = oracle.permute(a, "lpt", nw=nw)
    ck.check_lpt(perm, wl, nw)


def test_dcsr():
    a = syn.from_lists(6, 4, [[], [1], [], [0, 2], [3], []])
    assert oracle.permute(a, "dcsr").tolist() == [1, 3, 4, 0, 2, 5]


def test_window_contract():
    a = syn.rmat(8, 4, 71)
    with pytest.raises(ValueError):
        oracle.permute(a, "cta_aware", nw=32, window=48)   # not a multiple of nw
    p0 = oracle.permute(a, "cta_aware", window=0)
    pbig = oracle.permute(a, "cta_aware", window=32 * ((a.M + 31) // 32 + 1))
    assert np.array_equal(p0, pbig)
