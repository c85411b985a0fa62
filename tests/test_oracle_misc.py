"""Pins for the oracle's partition-by-nnz (c4, north star (4)) and predictor forward -- CPU."""
import numpy as np
import pytest
import torch

import oracle
import synthetic as syn


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_partition_properties(P):
    a = syn.rmat(10, 8, 3, "natural")
    b = oracle.partition_by_nnz(a.rowidx, P)
    nnz = a.nnz
    maxrow = int(np.diff(a.rowidx).max())
    assert b[0] == 0 and b[-1] == a.M and np.all(np.diff(b) >= 0)
    for p in range(P):
        assert a.rowidx[b[p + 1]] - a.rowidx[b[p]] <= -(-nnz // P) + maxrow
    # brute-force minimality of each cut
    for p in range(1, P):
        t = -(-p * nnz // P)
        r = next(r for r in range(a.M + 1) if a.rowidx[r] >= t)
        assert b[p] == r


def test_partition_degenerate():
    r = np.array([0, 0, 0], dtype=np.int64)
    assert oracle.partition_by_nnz(r, 4).tolist() == [0, 0, 0, 0, 2]


def test_mlp_forward_vs_torch():
    P = 6
    rng = np.random.default_rng(0)
    n = 48 + 64 * 24 + 64 + 32 * 64 + 32 + P * 32 + P
    w = rng.standard_normal(n).astype(np.float32) * 0.3
    w[24:48] = np.abs(w[24:48]) + 0.5        # sigma > 0
    feat = np.abs(rng.standard_normal(24)) * 100
    best, out = oracle.mlp_forward(feat, w, P)
    t = torch.from_numpy(w.astype(np.float64))
    mu, sg = t[:24], t[24:48]
    o = 48
    W1 = t[o:o + 1536].view(64, 24); o += 1536
    b1 = t[o:o + 64]; o += 64
    W2 = t[o:o + 2048].view(32, 64); o += 2048
    b2 = t[o:o + 32]; o += 32
    W3 = t[o:o + 32 * P].view(P, 32); o += 32 * P
    b3 = t[o:o + P]
    x = (torch.log1p(torch.from_numpy(feat)) - mu) / sg
    y = torch.nn.functional.linear(torch.relu(torch.nn.functional.linear(
        torch.relu(torch.nn.functional.linear(x, W1, b1)), W2, b2)), W3, b3)
    np.testing.assert_allclose(out, y.numpy(), rtol=1e-12, atol=1e-12)
    assert best == int(torch.argmin(y))
