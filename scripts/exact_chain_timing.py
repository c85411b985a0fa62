"""f3 measurement: paper-exact whole-matrix chains (W = 0, inverted-index builder k_chain_x) against the
windowed default (W = 1024): build time, SpMM step time (median of CUDA-event times, L2 flushed), and the
LRU-model L2 ceiling of the order.  python scripts/exact_chain_timing.py --configs c2,c3 --out FILE"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="c2")
ap.add_argument("--policies", default="cta_aware,hybrid_2_1")
ap.add_argument("--windows", default="1024,65536,0")
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "exact_chains.jsonl"))
args = ap.parse_args()
stream = torch.cuda.current_stream()
flush = torch.empty(64 * 1024 * 1024, device="cuda")
os.makedirs(os.path.dirname(args.out), exist_ok=True)
with open(args.out, "a") as fo:
    for cname in args.configs.split(","):
        cfg = bench.CONFIGS[cname]
        a = bench.make_matrix(cfg)
        K = cfg["K"]
        B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda()
        C = torch.empty((a.M, K), device="cuda")
        h = pkg.SpMM.from_csr(a)
        for pol in args.policies.split(","):
            for W in [int(x) for x in args.windows.split(",")]:
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                h.permute(pol, window=W)
                torch.cuda.synchronize()
                build_s = time.perf_counter() - t0
                for _ in range(3):
                    h.run(B, C)
                ts = bench.time_runs(torch, lambda: h.run(B, C), args.steps, lambda: flush.fill_(1.0), stream)
                rec = dict(config=cname, M=a.M, nnz=a.nnz, K=K, policy=pol, window=W, build_s=build_s,
                           ms=statistics.median(ts), gflops=2 * a.nnz * K / statistics.median(ts) / 1e6)
                import tools
                cap = int(torch.cuda.get_device_properties(0).L2_cache_size // (4 * K))
                rec["lru_b_row_misses"] = int(tools.lru_misses(a, h.perm(), cap))
                print(json.dumps(rec), flush=True)
                fo.write(json.dumps(rec) + "\n")
        h.close()
