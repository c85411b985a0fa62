"""One k_spmm launch per policy in ONE process (for a single `ncu --set full -k regex:k_spmm` capture of all of
them: the i-th captured launch is the i-th policy).  Prints the policy order; scripts/collect_profiles.py maps the
rows of the exported raw page back to the policies.

  ncu --set full --clock-control none -k regex:k_spmm -c 8 -o gpurun_out/prof_multi_c5 \\
      python scripts/profile_policies.py --config c5 --policies identity,nnz_sort,...
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c5")
ap.add_argument("--policies", default=",".join(bench.HOT))
ap.add_argument("--window", type=int, default=1024)
args = ap.parse_args()
cfg = bench.CONFIGS[args.config]
a = bench.make_matrix(cfg)
K = cfg["K"]
bseed = (cfg["gen"][3] if cfg["gen"][0] == "rmat" else cfg["gen"][2]) + 1
pkg.use_torch_allocator(True)
B = torch.from_numpy(syn.dense(a.N, K, bseed)).cuda()
C = torch.empty((a.M, K), device="cuda")
h = pkg.SpMM.from_csr(a)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
pols = args.policies.split(",")
with open(os.path.join(ROOT, "gpurun_out", f"prof_multi_{args.config}.policies"), "w") as f:
    f.write("\n".join(pols) + "\n")
for pol in pols:
    bench.permute_spec(h, pol, args.window)
    h.prepare(K, B, C)
    flush.fill_(1.0)
    torch.cuda.synchronize()
    h.run(B, C)                  # the captured launch of this policy
    torch.cuda.synchronize()
    print("ok", pol, flush=True)
h.close()
