"""C4 (BASELINE.json configs[3]): a synthetic corpus spanning the paper's feature ranges, every hot-path
policy timed on the B200 (the exhaustive-timing label) plus the 24 features and the
7 B200 platform features per K (f4, spmm_features_b200).

  python scripts/corpus.py --n-per-family 50 --out gpurun_out/corpus.jsonl

Families: power-law R-MAT (natural / local / random-label), banded random,
uniform random (Poisson degrees), block-clustered.  M log-uniform in [2^12, 2^max_log2m] (round 2: up to 2^22,
so that B at K >= 64 is far beyond the 126 MB L2 for a large part of the corpus), nnz/row log-uniform in [2, 64].
Half of the power-law (natural / local) and banded matrices get their rows randomly relabelled ("shuffled":
the original order then has no locality for the column-similarity orders to exploit).
Policies: all twelve of the C-ABI plus CTA-aware over the median-block pre-order ("cta_aware+md").  Seeds 0..4n-1.
"""
import argparse
import json
import math
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

FAMILIES = ["powerlaw", "banded", "uniform", "block"]


def shuffle_rows(a, seed):
    """Random row relabel (columns unchanged), as bench.make_matrix's shuffled configs."""
    q = np.random.default_rng(seed).permutation(a.M)
    lens = np.diff(a.rowidx)[q]
    r = np.zeros(a.M + 1, dtype=np.int64)
    np.cumsum(lens, out=r[1:])
    idx = np.repeat(a.rowidx[q] - r[:-1], lens) + np.arange(a.nnz, dtype=np.int64)
    return syn.CSR(a.M, a.N, r, a.colidx[idx], a.value[idx])


def draw(i, max_log2m):
    rng = np.random.default_rng(10_000 + i)
    fam = FAMILIES[i % 4]
    log2m = rng.uniform(12, max_log2m)
    M = int(round(2 ** log2m))
    d = float(math.exp(rng.uniform(math.log(2), math.log(64))))
    if fam == "powerlaw":
        S = int(round(log2m))
        variant = ["natural", "local", "random-label"][int(rng.integers(3))]
        a = syn.rmat(S, d, i, variant)
        params = dict(S=S, edge_factor=d, variant=variant)
    elif fam == "banded":
        w = int(max(d, d * 2 ** rng.uniform(0, 8)))
        a = syn.banded(M, int(round(d)), w, i)
        params = dict(d=int(round(d)), halfwidth=w)
    elif fam == "uniform":
        a = syn.uniform(M, M, d, i, poisson=True)
        params = dict(d=d)
    else:
        g = int(2 ** rng.integers(4, 9))
        c = int(2 ** rng.integers(1, 5))
        dd = int(min(round(d), c * 32))
        a = syn.blockcluster(M, M, g, c, dd, i)
        params = dict(g=g, c=c, d=dd)
    if fam == "banded" or (fam == "powerlaw" and params["variant"] != "random-label"):
        if rng.uniform() < 0.5:
            a = shuffle_rows(a, 20_000 + i)
            params["shuffled"] = True
    return fam, params, a


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n-per-family", type=int, default=50)
    ap.add_argument("--max-log2m", type=float, default=22.0)
    ap.add_argument("--K", default="32,64,128,256")
    ap.add_argument("--policies", default=",".join(list(pkg.POLICIES) + ["cta_aware+md"]))
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    ap.add_argument("--start", type=int, default=0)
    ap.add_argument("--stop", type=int, default=None)
    ap.add_argument("--out", default="gpurun_out/corpus.jsonl")
    args = ap.parse_args()
    Ks = [int(k) for k in args.K.split(",")]
    pols = args.policies.split(",")
    pkg.use_torch_allocator(True)
    flush = torch.empty(64 * 1024 * 1024, device="cuda")   # 256 MiB
    stream = torch.cuda.current_stream()
    out = open(args.out, "a")
    import bench
    n = 4 * args.n_per_family if args.stop is None else args.stop
    for i in range(args.start, n):
        t0 = time.perf_counter()
        fam, params, a = draw(i, args.max_log2m)
        h = pkg.SpMM.from_csr(a)
        feats = h.features().tolist()
        feats_b200 = {str(K): h.features_b200(K).tolist() for K in Ks}   # f4 platform features (g0..g6)
        Bs = {K: torch.from_numpy(syn.dense(a.N, K, 77 + i)).cuda() for K in Ks}
        C = torch.empty((a.M, max(Ks)), device="cuda")
        times = {K: {} for K in Ks}
        build = {}
        for pol in pols:
            tb = time.perf_counter()
            bench.permute_spec(h, pol, 1024)
            build[pol] = 1e3 * (time.perf_counter() - tb)
            for K in Ks:
                Ck = C[:, :K] if K == max(Ks) else torch.empty((a.M, K), device="cuda")
                for _ in range(args.warmup):
                    h.run(Bs[K], Ck)
                ts = []
                for _ in range(args.reps):
                    flush.fill_(1.0)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                    h.run(Bs[K], Ck)
                    e1.record(stream)
                    e1.synchronize()
                    ts.append(e0.elapsed_time(e1))
                times[K][pol] = statistics.median(ts)
        rec = dict(i=i, family=fam, params=params, name=a.name, M=a.M, N=a.N, nnz=a.nnz, features=feats,
                   features_b200=feats_b200,
                   times_ms={str(K): v for K, v in times.items()}, build_ms=build, seconds=time.perf_counter() - t0)
        out.write(json.dumps(rec) + "\n")
        out.flush()
        h.close()
        print(i, fam, a.M, a.nnz, f"{rec['seconds']:.1f}s", flush=True)


if __name__ == "__main__":
    main()
