"""Time spmm_run for (config, policy) under the current environment (A/B of SPMM_* knobs across processes):
median CUDA-event time, L2 flushed, and a hash of C's bytes for bit-identity across runs.
  SPMM_KSPLIT=2 python scripts/env_time.py --configs c5 --policies identity,cta_aware"""
import argparse
import hashlib
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="c3")
ap.add_argument("--policies", default="identity")
ap.add_argument("--steps", type=int, default=10)
args = ap.parse_args()
stream = torch.cuda.current_stream()
flush = torch.empty(64 * 1024 * 1024, device="cuda")
env = {k: v for k, v in os.environ.items() if k.startswith("SPMM_")}
for cname in args.configs.split(","):
    cfg = bench.CONFIGS[cname]
    a = bench.make_matrix(cfg)
    K = cfg["K"]
    B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda()
    C = torch.empty((a.M, K), device="cuda")
    h = pkg.SpMM.from_csr(a)
    h.set_kernel_timing(True)
    for pol in args.policies.split(","):
        h.permute(pol)
        for _ in range(3):
            h.run(B, C)
        ts = bench.time_runs(torch, lambda: h.run(B, C), args.steps, lambda: flush.fill_(1.0), stream)
        torch.cuda.synchronize()
        digest = hashlib.sha1(C.cpu().numpy().tobytes()).hexdigest()[:16]
        print(json.dumps(dict(env=env, config=cname, policy=pol, ms=statistics.median(ts), ms_min=min(ts),
                              launches=h.last_run_launches(), c_sha1=digest)), flush=True)
    h.close()
