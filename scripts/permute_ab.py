"""Build-time A/B of a compile-time library variant against the product build: spmm_permute wall time (stream
synchronised) per policy, and a SHA-256 of each permutation (the two builds must agree bit for bit).

  python scripts/permute_ab.py --define SPMM_EXP_NO_XRANGE --configs c3,c5 --policies cta_aware,hybrid_2_1
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CHILD = r"""
import sys, json, time, hashlib, torch
sys.path.insert(0, {root!r})
import bench, paper_conf_ispass_mehrabilcslo21_b200 as pkg
if {lib!r}:
    pkg.load_library({lib!r})
a = bench.make_matrix(bench.CONFIGS[{config!r}])
pkg.use_torch_allocator(True)
h = pkg.SpMM.from_csr(a)
res = {{}}
for pol in {policies!r}:
    ts = []
    for rep in range(3):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        bench.permute_spec(h, pol, {window})
        torch.cuda.synchronize(); ts.append((time.perf_counter() - t0) * 1e3)
    perm = h.perm()
    res[pol] = {{"ms": sorted(ts)[1], "all_ms": ts, "sha": hashlib.sha256(perm.tobytes()).hexdigest()[:16]}}
print(json.dumps(res))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--define", action="append", required=True)
    ap.add_argument("--configs", default="c3")
    ap.add_argument("--policies", default="cta_aware,hybrid_2_1")
    ap.add_argument("--window", type=int, default=1024)
    args = ap.parse_args()
    from paper_conf_ispass_mehrabilcslo21_b200 import _build
    lib_b = _build.build_variant(args.define, "_".join(d.lower() for d in args.define))
    pols = args.policies.split(",")
    out = {}
    for c in args.configs.split(","):
        r = {}
        for name, lib in (("product", ""), ("variant", lib_b)):
            p = subprocess.run([sys.executable, "-c", CHILD.format(root=ROOT, lib=lib, config=c, policies=pols, window=args.window)],
                               capture_output=True, text=True, timeout=3600)
            line = [l for l in p.stdout.splitlines() if l.startswith("{")]
            if not line:
                print(f"{c} {name}: child failed: {p.stderr[-1500:]}", file=sys.stderr, flush=True)
            r[name] = json.loads(line[-1]) if line else {}
        out[c] = {pol: {"product_ms": r["product"].get(pol, {}).get("ms"), "variant_ms": r["variant"].get(pol, {}).get("ms"),
                        "identical": r["product"].get(pol, {}).get("sha") == r["variant"].get(pol, {}).get("sha")}
                  for pol in pols}
        print(c, json.dumps(out[c]), flush=True)
    print(json.dumps({"defines": args.define, "window": args.window, "results": out}))


if __name__ == "__main__":
    main()
