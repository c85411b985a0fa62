"""Run the SpMM of one policy a few times (for ncu captures on the GPU box).

  ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -o gpurun_out/prof \
      python scripts/profile_spmm.py --config c3 --policy identity
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
ap.add_argument("--config", default="c3")
ap.add_argument("--policy", default="identity")
ap.add_argument("--runs", type=int, default=3)
ap.add_argument("--window", type=int, default=1024)
ap.add_argument("--split", type=int, default=128)
ap.add_argument("--lib", default="", help="an A/B variant library (scripts/ab_lib.py) instead of the product build")
ap.add_argument("--define", action="append", default=[], help="build and load a variant with these -D defines")
args = ap.parse_args()
if args.define:
    from paper_conf_ispass_mehrabilcslo21_b200 import _build
    args.lib = _build.build_variant(args.define, "_".join(d.lower() for d in args.define))
if args.lib:
    pkg.load_library(args.lib)
cfg = bench.CONFIGS[args.config]
a = bench.make_matrix(cfg)
K = cfg["K"]
B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda()
C = torch.empty((a.M, K), device="cuda")
h = pkg.SpMM.from_csr(a)
bench.permute_spec(h, args.policy, args.window)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
for _ in range(args.runs):
    flush.fill_(1.0)
    h.run(B, C)
torch.cuda.synchronize()
print("ok", args.policy, h.info())
