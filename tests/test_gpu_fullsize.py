"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times (default params,
window 1024, torch allocator): sampled outputs the oracle computes one by one, and the permutation /
features checked against the oracle (-m gpu).

* C2  27-point stencil 100^3 (configs[1]), K=64 (row fusion engaged by default: R = 4)
* C3  R-MAT S=22 "local", nnz 99.6M (configs[2]), K=128
* C5  R-MAT S=24 "local", nnz 505M (configs[4], bench.py's default workload), K=128
Sorted policies (incl. f1's LPT, Flipped Sort, DCSR) are compared in full; chain policies (incl. f1's Warp-aware,
Hybrid-2.2, Hybrid-2.3 and the median-block pre-order) on 64 sampled windows plus the first and the last (each
window's chain depends only on its own rows, so the oracle runs on the window's rows alone -- SURVEY.md §8(d)
"Permutation parity at C5 checks ... a seeded random sample of 64 windows plus the first and last").
"""
import numpy as np
import pytest

import oracle
import synthetic as syn

torch = pytest.importorskip("torch")
pytestmark = [pytest.mark.gpu, pytest.mark.slow]

import bench  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

W = 1024


def sub_rows(a, rows):
    rows = np.asarray(rows, dtype=np.int64)
    lens = a.rowidx[rows + 1] - a.rowidx[rows]
    r = np.zeros(len(rows) + 1, dtype=np.int64)
    r[1:] = np.cumsum(lens)
    idx = np.concatenate([np.arange(a.rowidx[i], a.rowidx[i + 1]) for i in rows]) if len(rows) else np.array([], int)
    return syn.CSR(len(rows), a.N, r, a.colidx[idx], a.value[idx])


@pytest.fixture(scope="module", params=["c2", "c3", "c5"])
def full(request):
    cfg = bench.CONFIGS[request.param]
    a = bench.make_matrix(cfg)
    K = cfg["K"]
    bseed = (cfg["gen"][3] if cfg["gen"][0] == "rmat" else cfg["gen"][2]) + 1
    B = syn.dense(a.N, K, bseed)
    pkg.use_torch_allocator(True)
    h = pkg.SpMM.from_csr(a)
    yield request.param, a, K, B, h
    h.close()
    pkg.use_torch_allocator(False)


def sample_rows(a, n=3000, seed=5):
    rng = np.random.default_rng(seed)
    lens = np.diff(a.rowidx)
    picks = set(rng.choice(a.M, size=min(n, a.M), replace=False).tolist())
    picks.update(np.argsort(-lens, kind="stable")[:20].tolist())        # the longest (split) rows
    picks.update(np.flatnonzero(lens == 0)[:20].tolist())               # empty rows
    picks.update([0, a.M - 1])
    return np.array(sorted(picks), dtype=np.int64)


@pytest.mark.parametrize("policy", pkg.HOT_PATH_POLICIES + ["flipped", "lpt", "warp_aware", "hybrid_2_2",
                                                           "hybrid_2_3", "dcsr", "cta_aware+md"])
def test_fullsize_spmm_sampled(full, policy):
    name, a, K, B, h = full
    bench.permute_spec(h, policy, W)
    Bd = torch.from_numpy(B).cuda()
    C = h.run(Bd)
    torch.cuda.synchronize()
    rows = sample_rows(a)
    Cg = C[torch.from_numpy(rows).cuda()].cpu().numpy().astype(np.float64)
    Cr, bound = oracle.spmm(a, B, rows=rows)
    err = np.abs(Cg - Cr)
    assert np.all(err <= 1e-5 * bound + 1e-6), (name, policy, float((err / (1e-5 * bound + 1e-6)).max()))


def test_fullsize_sorts_and_features(full):
    name, a, K, B, h = full
    for pol in ("nnz_sort", "plain_sort"):
        h.permute(pol, window=W)
        assert np.array_equal(h.perm(), oracle.permute(a, pol)), (name, pol)
    np.testing.assert_array_equal(h.features(), oracle.features(a))
    np.testing.assert_array_equal(h.features_b200(K), oracle.features_b200(a, K))


@pytest.mark.parametrize("policy", ["lpt", "flipped", "dcsr"])
def test_fullsize_f1_orders(full, policy):
    """The rest of the paper's portfolio whose permutations are whole-matrix orders -- LPT
    (reading A5: capacity-constrained over the nw warps), Flipped Sort and DCSR --
    compared in full against the oracle at full size."""
    name, a, K, B, h = full
    h.permute(policy, window=W)
    got = h.perm()
    ref = oracle.permute(a, policy)
    assert np.array_equal(got, ref), (name, policy, int(np.argmax(got != ref)))


@pytest.mark.parametrize("policy", ["cta_aware", "hybrid_2_1", "hybrid_1", "warp_aware", "hybrid_2_2", "hybrid_2_3",
                                    "cta_aware+md", "hybrid_2_1+mh"])
def test_fullsize_chain_windows_sampled(full, policy):
    """Chain policies at full size on 64 seeded random windows plus the first and the last; each
    window's chain depends only on its own rows, so the oracle runs on them alone.  '+md': windows over the
    median-block pre-order (preorder = 2), recomputed here from the oracle's keys."""
    name, a, K, B, h = full
    bench.permute_spec(h, policy, W)
    perm = h.perm()
    rng = np.random.default_rng(11)
    NS = 64
    if policy == "hybrid_1":
        plain = oracle.permute(a, "plain_sort")
        wl = (np.diff(a.rowidx) + 31) // 32
        # segment starts: run starts of equal wl in Plain-Sort order, cut every W positions
        key = wl[plain]
        run_start = np.zeros(a.M, dtype=np.int64)
        starts = np.flatnonzero(np.r_[True, key[1:] != key[:-1]])
        run_start[starts] = starts
        run_start = np.maximum.accumulate(run_start)
        seg_starts = np.flatnonzero((np.arange(a.M) - run_start) % W == 0)
        seg_ends = np.r_[seg_starts[1:], a.M]
        pick = sorted(set(rng.choice(len(seg_starts), size=min(NS, len(seg_starts)), replace=False).tolist())
                      | {0, len(seg_starts) - 1})
        for s in pick:
            lo, hi = seg_starts[s], seg_ends[s]
            rows = plain[lo:hi]                                  # ascending ids within an equal-wl run
            ref = oracle.permute(sub_rows(a, rows), "hybrid_1", window=0)
            assert np.array_equal(perm[lo:hi], rows[ref]), (name, policy, s)
    else:
        base = policy[:-3] if policy.endswith(("+md", "+mh")) else policy
        if policy.endswith("+md"):
            pre = np.lexsort((np.arange(a.M), oracle.median_block_keys(a)))
        elif policy.endswith("+mh"):                 # the binding's "+mh" = MinHash pre-order with seed 1
            pre = np.lexsort((np.arange(a.M), oracle.minhash_keys(a, seed=1)))
        else:
            pre = np.arange(a.M)
        nwin = (a.M + W - 1) // W
        pick = sorted(set(rng.choice(nwin, size=min(NS, nwin), replace=False).tolist()) | {0, nwin - 1})
        for s in pick:
            lo, hi = s * W, min((s + 1) * W, a.M)
            rows = np.sort(pre[lo:hi])      # the window's row SET; every tie-break is by original row id (A2)
            ref = oracle.permute(sub_rows(a, rows), base, window=0)
            assert np.array_equal(perm[lo:hi], rows[ref]), (name, policy, s)
