"""Build-time A/B of the two chain builders on the same window (k_chain vs k_chain_x via SPMM_CHAIN_EXACT),
with a bit-identity check of the two permutations.  python scripts/chain_builder_ab.py --configs c3,c5"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--configs", default="c3")
ap.add_argument("--policies", default="cta_aware,hybrid_2_1")
ap.add_argument("--windows", default="1024")
args = ap.parse_args()
for cname in args.configs.split(","):
    a = bench.make_matrix(bench.CONFIGS[cname])
    h = pkg.SpMM.from_csr(a)
    for pol in args.policies.split(","):
        for W in [int(x) for x in args.windows.split(",")]:
            res = {}
            for force in ("0", "1"):
                os.environ["SPMM_CHAIN_EXACT"] = force
                h.permute(pol, window=W)          # warm (allocations)
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                h.permute(pol, window=W)
                torch.cuda.synchronize()
                res[force] = (time.perf_counter() - t0, h.perm())
            os.environ.pop("SPMM_CHAIN_EXACT", None)
            print(json.dumps(dict(config=cname, M=a.M, policy=pol, window=W, k_chain_s=res["0"][0],
                                  k_chain_x_s=res["1"][0], identical=bool(np.array_equal(res["0"][1], res["1"][1])))),
                  flush=True)
    h.close()
