"""A/B of row fusion (spmm_params.fuse_rows 1 = off, 0 = auto, 2 = forced) on the GPU box.

Per (matrix, K, policy): median CUDA-event time of spmm_run (L2 flushed between steps), the schedule's
union records per fused nnz, and a bit-identity check of C against the unfused run.

  python scripts/fuse_ab.py [--quick]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--quick", action="store_true")
ap.add_argument("--cases", default="")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "fuse_ab.jsonl"))
args = ap.parse_args()

flush_buf = torch.empty(64 * 1024 * 1024, device="cuda")
stream = torch.cuda.current_stream()


def shuffled(a, seed):
    """Same matrix with rows AND columns relabelled by one random permutation (locality destroyed)."""
    rng = np.random.default_rng(seed)
    p = rng.permutation(a.M)           # new id of old row/col i is inv... use gather form: new row r = old p[r]
    inv = np.empty_like(p)
    inv[p] = np.arange(a.M)
    rows = []
    vals = []
    for r in range(a.M):
        o = p[r]
        c = inv[a.colidx[a.rowidx[o]:a.rowidx[o + 1]]]
        v = a.value[a.rowidx[o]:a.rowidx[o + 1]]
        order = np.argsort(c)
        rows.append(c[order])
        vals.append(v[order])
    return syn.from_lists(a.M, a.N, rows, vals)


cases = [("c2_stencil100", lambda: bench.make_matrix(bench.CONFIGS["c2"]), [64, 32, 128], ["identity", "cta_aware"])]
if not args.quick:
    cases += [
        ("banded_1M_d27_w64", lambda: syn.banded(1 << 20, 27, 64, 11), [64, 128], ["identity", "cta_aware"]),
        ("stencil40_shuffled", lambda: shuffled(syn.stencil27(40, 12), 13), [64], ["identity", "cta_aware", "hybrid_2_1"]),
        ("c3_rmat22_local", lambda: bench.make_matrix(bench.CONFIGS["c3"]), [128], ["identity", "cta_aware"]),
    ]

if args.cases:
    cases = [c for c in cases if c[0] in args.cases.split(",")]
os.makedirs(os.path.dirname(args.out), exist_ok=True)
with open(args.out, "a") as fo:
    for name, gen, Ks, pols in cases:
        a = gen()
        h = pkg.SpMM.from_csr(a)
        for K in Ks:
            B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda()
            C = torch.empty((a.M, K), device="cuda")
            for pol in pols:
                ref = None
                for fuse in (1, 0, 2):
                    h.permute(pol, fuse_rows=fuse)
                    for _ in range(3):
                        h.run(B, C)
                    ts = bench.time_runs(torch, lambda: h.run(B, C), args.steps, lambda: flush_buf.fill_(1.0), stream)
                    out = C.cpu().numpy().view(np.int32)
                    same = True if ref is None else bool(np.array_equal(out, ref))
                    if ref is None:
                        ref = out.copy()
                    info = h.schedule_info()
                    rec = dict(matrix=name, M=a.M, nnz=a.nnz, K=K, policy=pol, fuse_rows=fuse, ms=statistics.median(ts),
                               gflops=2 * a.nnz * K / statistics.median(ts) / 1e6, bit_identical=same, **info)
                    print(json.dumps(rec), flush=True)
                    fo.write(json.dumps(rec) + "\n")
        h.close()
