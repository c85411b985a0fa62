"""Pins for the oracle's B200 platform features g0..g6 (oracle.c c3b; DESIGN.md readings
A24-A26) -- CPU only.

Pins: the E1 matrix (SURVEY.md §8(c) worked example) with every value worked by hand below; closed forms on the
27-point stencil (pairs / quads of consecutive x-neighbours: the union along x, independent of y and z); a
brute-force recount with Python sets (an implementation independent of the oracle's mark array); order
invariants (g3 and g4 do not depend on the order; g0..g2 computed on a permuted matrix equal the oracle's
features of that matrix's permuted CSR).
"""
import numpy as np
import pytest

import oracle
import synthetic as syn


def test_e1_by_hand(e1):
    # rows: r0 {0..4}, r1 {7}, r2 {}, r3 {0,2}, r4 {5,6,7}, r5 {1}, r6 {4,5,6,7}, r7 {0,3,6}; nnz 19, N 8
    a = syn.from_lists(e1["M"], e1["N"], e1["rows"])
    g = oracle.features_b200(a, K=64)
    # g0: pairs (0,1) {0,1,2,3,4,7}=6, (2,3) {0,2}=2, (4,5) {1,5,6,7}=4, (6,7) {0,3,4,5,6,7}=6 -> 18/19
    assert g[0] == 18 / 19
    # g1: quads (0..3) {0,1,2,3,4,7}=6, (4..7) {0,1,3,4,5,6,7}=7 -> 13/19
    assert g[1] == 13 / 19
    # g2: one window, all 8 columns -> 8/19
    assert g[2] == 8 / 19
    # g3 at K=64: 4*64*8 / (4*9 + 8*19 + 4*64*8 + 4*8*64)
    assert g[3] == 2048 / (36 + 152 + 2048 + 2048)
    assert g[4] == 1 / 8 and g[5] == 0.0
    # g6 at K=64 (RPW 4): short lengths [5,1,2,3,1,4,3] -> one window sorted [5,4,3,3 | 2,1,1]: 19 / (4*5 + 4*2)
    assert g[6] == 19 / 28
    # K=32 (RPW 8): one group [5,4,3,3,2,1,1] -> 19 / (8*5)
    assert oracle.features_b200(a, K=32)[6] == 19 / 40


@pytest.mark.parametrize("n", [4, 6, 8, 10, 12])
def test_stencil_closed_forms(n):
    """Along x a row at x covers x-1..x+1 (clipped); rows of one x-line share their y/z neighbour set, so the
    union over consecutive x-neighbours factors: pair (0,1) 3 of 5, interior pair 4 of 6, last pair 3 of 5;
    quad at the boundary 5 of 11, interior quad 6 of 12 (n = 4: one quad, 4 of 10)."""
    a = syn.stencil27(n, 3)
    g = oracle.features_b200(a, K=128)
    pairs = n // 2
    assert g[0] == pytest.approx((2 * 3 + (pairs - 2) * 4) / (2 * 5 + (pairs - 2) * 6), rel=0, abs=1e-15)
    if n % 4 == 0:
        q = n // 4
        exp = 4 / 10 if q == 1 else (2 * 5 + (q - 2) * 6) / (2 * 11 + (q - 2) * 12)
        assert g[1] == pytest.approx(exp, rel=0, abs=1e-15)
    nnz = (3 * n - 2) ** 3
    assert a.nnz == nnz
    if n ** 3 <= 1024:
        assert g[2] == n ** 3 / nnz                     # one window holds every column
    assert g[4] == 0 and g[5] == 0                      # no empty rows, all rows <= 27 nnz


def brute(a, K, perm=None):
    order = np.arange(a.M) if perm is None else np.asarray(perm)
    rows = [set(a.colidx[a.rowidx[i]:a.rowidx[i + 1]].tolist()) for i in order]
    lens = [len(r) for r in rows]
    nnz = sum(lens)

    def grp(size):
        return sum(len(set().union(*rows[p:p + size])) for p in range(0, a.M, size))

    r = lambda x, y: x / y if y else 0.0   # noqa: E731
    cn = len(set().union(*rows)) if rows else 0
    g = [r(grp(2), nnz), r(grp(4), nnz), r(grp(1024), nnz),
         r(4 * K * cn, 4 * (a.M + 1) + 8 * nnz + 4 * K * cn + 4 * a.M * K),
         r(sum(1 for x in lens if x == 0), a.M), r(sum(x for x in lens if x > 128), nnz)]
    rpw = 8 if K <= 32 else 4 if K <= 256 else 2
    sl = [x for x in lens if 0 < x <= 128]
    tot = slots = 0
    for w in range(0, len(sl), 32):
        win = sorted(sl[w:w + 32], reverse=True)
        tot += sum(win)
        slots += sum(rpw * max(win[t:t + rpw]) for t in range(0, len(win), rpw))
    g.append(r(tot, slots))
    return np.array(g)


@pytest.mark.parametrize("gen", ["rmat", "uniform", "block", "banded", "empty"])
@pytest.mark.parametrize("K", [32, 128, 512])
def test_bruteforce_recount(gen, K):
    a = {"rmat": lambda: syn.rmat(11, 9, 7, "natural"),
         "uniform": lambda: syn.uniform(3000, 2000, 5, 8, poisson=True),
         "block": lambda: syn.blockcluster(2100, 3000, 16, 3, 12, 9),
         "banded": lambda: syn.banded(2500, 20, 30, 10),
         "empty": lambda: syn.from_lists(5, 7, [[]] * 5)}[gen]()
    rng = np.random.default_rng(4)
    for perm in (None, rng.permutation(a.M).astype(np.int32)):
        np.testing.assert_array_equal(oracle.features_b200(a, K, perm), brute(a, K, perm))


def test_order_invariants_and_permuted_csr():
    a = syn.rmat(10, 12, 17, "local")
    for pol in ("nnz_sort", "cta_aware"):
        perm = oracle.permute(a, pol, window=256)
        g = oracle.features_b200(a, 128, perm)
        g0 = oracle.features_b200(a, 128)
        assert g[3] == g0[3] and g[4] == g0[4] and g[5] == g0[5]
        r, c, v = oracle.permuted_csr(a, perm)
        ap = syn.CSR(a.M, a.N, r, c, v)
        np.testing.assert_array_equal(oracle.features_b200(ap, 128), g)


def test_split_boundary_by_hand():
    """The split-row threshold is strict (A24: rows with more than split_nnz = 128 nnz are split rows, g5) and the
    short rows of g6 are 0 < len <= 128: rows of 127, 128, 129, 200 and 0 nnz, every value worked by hand."""
    lens = [127, 128, 129, 200, 0]
    a = syn.from_lists(5, 256, [list(range(n)) for n in lens])
    g = oracle.features_b200(a, K=64)
    assert g[4] == 1 / 5                                  # one empty row
    assert g[5] == (129 + 200) / (127 + 128 + 129 + 200)  # 128 is not a split row
    assert g[6] == (127 + 128) / (4 * 128)                # one RPW = 4 group [128, 127], slots 4 * 128
    # union features: rows 0..4 are nested prefixes of 0..199 -> pairs {0..127}, {0..199}, {} ; quad {0..199}, {}
    assert g[0] == (128 + 200) / 584 and g[1] == 200 / 584 and g[2] == 200 / 584
