"""A/B of a compile-time library variant against the product build: the k_spmm kernel time (library events,
spmm_set_kernel_timing) of one policy on one config, alternating the two libraries in separate processes.

  python scripts/ab_lib.py --define SPMM_EXP_A_POLICY --configs c3,c5 --policy cta_aware
"""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CHILD = r"""
import sys, json, statistics, torch
sys.path.insert(0, {root!r})
import bench, synthetic as syn, paper_conf_ispass_mehrabilcslo21_b200 as pkg
if {lib!r}:
    pkg.load_library({lib!r})
cfg = bench.CONFIGS[{config!r}]
a = bench.make_matrix(cfg); K = cfg["K"]
pkg.use_torch_allocator(True)
B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda(); C = torch.empty((a.M, K), device="cuda")
h = pkg.SpMM.from_csr(a); h.permute({policy!r}); h.prepare(K, B, C)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
for _ in range(3): h.run(B, C)
h.set_kernel_timing(True)
import threading, pynvml
pynvml.nvmlInit(); _hd = pynvml.nvmlDeviceGetHandleByIndex(0); _smp = []; _stop = threading.Event()
def _sample():
    while not _stop.is_set():
        _smp.append((pynvml.nvmlDeviceGetPowerUsage(_hd) / 1000.0, pynvml.nvmlDeviceGetClockInfo(_hd, pynvml.NVML_CLOCK_SM)))
        _stop.wait(0.005)
_th = threading.Thread(target=_sample, daemon=True); _th.start()
ks = []; st = []
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
for _ in range(15):
    flush.fill_(1.0); e0.record(); h.run(B, C); e1.record(); e1.synchronize()
    ks.append(h.last_kernel_ms()); st.append(e0.elapsed_time(e1))
_stop.set(); _th.join()
w = torch.arange(C.numel(), device="cuda", dtype=torch.int64) % 1000003 + 1
crc = int(((C.reshape(-1).view(torch.int32).to(torch.int64) & 0xffffffff) * w).sum().item())   # bits of C
print(json.dumps({{"ms": statistics.median(ks), "step_ms": statistics.median(st), "crc": crc, "power_w": statistics.median([x[0] for x in _smp]), "sm_mhz": statistics.median([x[1] for x in _smp])}}))
"""


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--define", action="append", required=True)
    ap.add_argument("--configs", default="c3")
    ap.add_argument("--policy", default="cta_aware")
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("--base", action="append", default=[], help="defines of the baseline build (default: product)")
    args = ap.parse_args()
    from paper_conf_ispass_mehrabilcslo21_b200 import _build
    lib_b = _build.build_variant(args.define, "_".join(d.lower() for d in args.define))
    lib_a = _build.build_variant(args.base, "_".join(d.lower() for d in args.base)) if args.base else ""
    res = {}
    for c in args.configs.split(","):
        t = {"product": [], "variant": []}
        steps = {"product": [], "variant": []}
        pw = {"product": [], "variant": []}
        crcs = {}
        for _ in range(args.rounds):
            for name, lib in (("product", lib_a), ("variant", lib_b)):
                out = subprocess.run([sys.executable, "-c", CHILD.format(root=ROOT, lib=lib, config=c, policy=args.policy)],
                                     capture_output=True, text=True, timeout=1200)
                line = [l for l in out.stdout.splitlines() if l.startswith("{")]
                if not line:
                    print(f"{c} {name}: child failed: {out.stderr[-1500:]}", file=sys.stderr, flush=True)
                d = json.loads(line[-1]) if line else {}
                t[name].append(d.get("ms"))
                steps[name].append(d.get("step_ms"))
                pw[name].append((d.get("power_w"), d.get("sm_mhz")))
                crcs.setdefault(name, set()).add(d.get("crc"))
        res[c] = {k: v for k, v in t.items()}
        res[c]["median"] = {k: statistics.median([x for x in v if x]) for k, v in t.items()}
        res[c]["power_w_sm_mhz"] = pw
        res[c]["step_median"] = {k: statistics.median([x for x in v if x]) for k, v in steps.items()}
        res[c]["C_bit_identical"] = crcs.get("product") == crcs.get("variant") and len(crcs.get("product", ())) == 1
        print(c, json.dumps(res[c]), flush=True)
    print(json.dumps({"defines": args.define, "base": args.base, "policy": args.policy, "results": res}))


if __name__ == "__main__":
    main()
