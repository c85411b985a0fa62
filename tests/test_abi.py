"""C-ABI checks that need no GPU: the library loads, exports every function include/spmm.h declares, and
its host-only entry points (partition, predictor inference, status strings) agree with the oracle."""
import os
import re

import numpy as np
import pytest

import oracle
import synthetic as syn
import paper_conf_ispass_mehrabilcslo21_b200 as pkg

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def header_functions():
    txt = open(os.path.join(ROOT, "include", "spmm.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(spmm_[a-z_0-9]+)\s*\(", txt)))


def test_exports_every_declared_symbol():
    lib = pkg.load_library()
    names = header_functions()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), n
    assert set(names) == set(pkg.EXPORTS)


def test_built_for_sm100a():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", pkg.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_status_strings():
    lib = pkg.load_library()
    for code, name in pkg.STATUS.items():
        assert lib.spmm_status_string(code).decode() == name


@pytest.mark.parametrize("P", [1, 2, 3, 8])
def test_partition_matches_oracle(P):
    a = syn.rmat(11, 8, 7, "natural")
    assert np.array_equal(pkg.spmm_partition_by_nnz(a.rowidx, P), oracle.partition_by_nnz(a.rowidx, P))


def test_partition_invalid():
    with pytest.raises(pkg.SpmmError) as e:
        pkg.spmm_partition_by_nnz(np.array([0, 1]), 0)
    assert e.value.status == 1


@pytest.mark.parametrize("P", [4, 6])
def test_predict_matches_oracle(P):
    rng = np.random.default_rng(P)
    n = 48 + 64 * 24 + 64 + 32 * 64 + 32 + 33 * P
    w = (rng.standard_normal(n) * 0.3).astype(np.float32)
    w[24:48] = np.abs(w[24:48]) + 0.5
    for t in range(5):
        f = np.abs(rng.standard_normal(24)) * 10 ** rng.integers(0, 6)
        pol, times = pkg.spmm_predict(f, w, P)
        best, ref = oracle.mlp_forward(f, w, P)
        assert pol == best
        np.testing.assert_allclose(times, ref, rtol=1e-12, atol=1e-12)


def np_forward(f, w, F, P):
    """Independent numpy float64 forward of the F-64-32-P layout (pins oracle_mlp_forward_n)."""
    w = w.astype(np.float64)
    o = 0
    mu, sg = w[o:o + F], w[o + F:o + 2 * F]; o += 2 * F
    W1 = w[o:o + 64 * F].reshape(64, F); o += 64 * F
    b1 = w[o:o + 64]; o += 64
    W2 = w[o:o + 2048].reshape(32, 64); o += 2048
    b2 = w[o:o + 32]; o += 32
    W3 = w[o:o + 32 * P].reshape(P, 32); o += 32 * P
    b3 = w[o:o + P]
    z = (np.log1p(f) - mu) / sg
    h1 = np.maximum(W1 @ z + b1, 0)
    h2 = np.maximum(W2 @ h1 + b2, 0)
    return W3 @ h2 + b3


@pytest.mark.parametrize("F,P", [(24, 6), (31, 6), (31, 4), (5, 3)])
def test_predict_n_matches_oracle_and_numpy(F, P):
    rng = np.random.default_rng(F * 10 + P)
    n = 2 * F + 64 * F + 64 + 32 * 64 + 32 + 33 * P
    w = (rng.standard_normal(n) * 0.3).astype(np.float32)
    w[F:2 * F] = np.abs(w[F:2 * F]) + 0.5
    for t in range(5):
        f = np.abs(rng.standard_normal(F)) * 10 ** rng.integers(0, 6)
        ref = np_forward(f, w, F, P)
        best, orc = oracle.mlp_forward_n(f, w, P)
        np.testing.assert_allclose(orc, ref, rtol=1e-10, atol=1e-10)
        pol, times = pkg.spmm_predict_n(f, w, P)
        assert pol == best == int(np.argmin(orc))
        np.testing.assert_allclose(times, orc, rtol=1e-12, atol=1e-12)
        if F == 24:
            assert pkg.spmm_predict(f, w, P)[0] == pol


def test_predict_rejects_bad_layout():
    with pytest.raises(pkg.SpmmError):
        pkg.spmm_predict(np.zeros(24), np.zeros(10, np.float32), 4)


def test_no_cpu_fallback_in_product():
    """The product package must not import the oracle (or any CPU fallback)."""
    pdir = os.path.join(ROOT, "paper_conf_ispass_mehrabilcslo21_b200")
    for dp, _, fs in os.walk(pdir):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dp, f)).read()
                for bad in ("import oracle", "from oracle", "liboracle", '#include "../../oracle', "oracle/"):
                    assert bad not in src, (f, bad)


def test_bundled_predictor_matches_oracle_forward():
    """The bundled weights run through the library's C inference (spmm_predict) give the same argmin and
    times as the oracle's float64 forward, on the committed corpus features (profiles/corpus_r1.jsonl)."""
    import json
    recs = [json.loads(l) for l in open(os.path.join(ROOT, "profiles", "corpus_r1.jsonl"))][:60]
    for paper in (False, True):
        P = len(pkg.PAPER4_POLICIES if paper else pkg.PREDICTOR_POLICIES)
        for K in (32, 64, 128, 256):
            w = pkg.predictor_weights(K, paper)
            assert len(w) == 48 + 64 * 24 + 64 + 32 * 64 + 32 + 33 * P
            for r in recs:
                f = np.array(r["features"])
                pol, t = pkg.spmm_predict(f, w, P)
                best, ref = oracle.mlp_forward(f, w, P)
                assert pol == best
                np.testing.assert_allclose(t, ref, rtol=1e-9, atol=1e-9)


def test_permcache_key():
    """permcache keys: a function of the CSR structure, the policy and its parameters only (CPU, no GPU)."""
    import synthetic as syn
    from paper_conf_ispass_mehrabilcslo21_b200.permcache import cache_key
    a = syn.rmat(8, 4, 1)
    k = cache_key(a.rowidx, a.colidx, "cta_aware", {"window": 1024})
    assert k == cache_key(a.rowidx.copy(), a.colidx.copy(), "cta_aware", {"window": 1024})
    assert k != cache_key(a.rowidx, a.colidx, "hybrid_2_1", {"window": 1024})
    assert k != cache_key(a.rowidx, a.colidx, "cta_aware", {"window": 2048})
    c = a.colidx.copy()
    c[0] = (c[0] + 1) % a.N
    assert k != cache_key(a.rowidx, c, "cta_aware", {"window": 1024})
