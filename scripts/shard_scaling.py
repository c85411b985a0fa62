"""SpMM-phase strong scaling of the row-sharded mode, measured shard by shard on ONE B200 ("report
SpMM-phase scaling with B resident: t_1 / max_p t_p").  The matrix is partitioned by nnz into P shards exactly as
ShardedSpMM does (spmm_partition_by_nnz, compact columns: each shard holds only the B rows it references); each
shard's SpMM (permuted with the given policy) is timed alone with its own compact B resident, L2 flushed between
steps.  A rank of a P-GPU run executes exactly this kernel on its shard, so max_p t_p is the SpMM phase of that run
(communication excluded: that part needs the GPUs).  Also reports the compulsory-bytes ideal speedup
sum / max_p (8 nnz_p + 4K |cols_p| + 4K M_p).

  python scripts/shard_scaling.py --config c5 --policy cta_aware --P 1,2,4,8
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
from paper_conf_ispass_mehrabilcslo21_b200.sharded import compact_shard, make_shard, shard_columns  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--policy", default="cta_aware")
    ap.add_argument("--P", default="1,2,4,8")
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    cfg = bench.CONFIGS[args.config]
    a = bench.make_matrix(cfg)
    K = cfg["K"]
    bseed = (cfg["gen"][3] if cfg["gen"][0] == "rmat" else cfg["gen"][2]) + 1
    Bfull = torch.from_numpy(syn.dense(a.N, K, bseed)).cuda()
    pkg.use_torch_allocator(True)
    flush = torch.empty(64 * 1024 * 1024, device="cuda")
    res = {"config": cfg["desc"], "policy": args.policy, "per_P": {}}
    for P in [int(x) for x in args.P.split(",")]:
        bounds = pkg.spmm_partition_by_nnz(a.rowidx, P)
        shards = []
        for p in range(P):
            cols = shard_columns(a.rowidx, a.colidx, bounds, p)
            sh = compact_shard(make_shard(a.M, a.N, a.rowidx, a.colidx, a.value, bounds, p), cols)
            Bp = Bfull.index_select(0, torch.from_numpy(cols).cuda()).contiguous()
            C = torch.empty((sh.M, K), device="cuda")
            h = pkg.SpMM(sh.M, sh.N, sh.rowidx, sh.colidx, sh.value)
            h.permute(args.policy)
            h.prepare(K, Bp, C)
            for _ in range(3):
                h.run(Bp, C)
            ts = bench.time_runs(torch, lambda: h.run(Bp, C), args.steps, lambda: flush.fill_(1.0),
                                 torch.cuda.current_stream())
            h.set_kernel_timing(True)
            ks = []
            for _ in range(args.steps):
                flush.fill_(1.0)
                h.run(Bp, C)
                ks.append(h.last_kernel_ms())
            h.close()
            comp = 8 * sh.nnz + 4 * K * len(cols) + 4 * K * sh.M
            shards.append({"rows": sh.M, "nnz": sh.nnz, "cols": int(len(cols)), "step_ms": statistics.median(ts),
                           "kernel_ms": statistics.median(ks), "compulsory_bytes": comp})
            del Bp, C
            torch.cuda.empty_cache()
        tmax = max(s["step_ms"] for s in shards)
        res["per_P"][P] = {"shards": shards, "max_step_ms": tmax,
                           "compulsory_max_bytes": max(s["compulsory_bytes"] for s in shards),
                           "compulsory_sum_bytes": sum(s["compulsory_bytes"] for s in shards)}
        print(P, json.dumps({k: v for k, v in res["per_P"][P].items() if k != "shards"}), flush=True)
    t1 = res["per_P"][min(res["per_P"])]["max_step_ms"]
    for P, r in res["per_P"].items():
        r["spmm_phase_speedup"] = t1 / r["max_step_ms"]
        r["ideal_compulsory_speedup"] = r["compulsory_sum_bytes"] / r["compulsory_max_bytes"]
        r["gflops_aggregate"] = 2.0 * a.nnz * K / r["max_step_ms"] / 1e6
    print(json.dumps({P: {"speedup": round(r["spmm_phase_speedup"], 2), "ideal_compulsory": round(r["ideal_compulsory_speedup"], 2),
                          "max_step_ms": round(r["max_step_ms"], 3), "GFLOP/s": round(r["gflops_aggregate"])}
                      for P, r in res["per_P"].items()}))
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
