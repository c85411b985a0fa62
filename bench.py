#!/usr/bin/env python
"""bench.py -- SpMM GFLOP/s and % HBM roofline per row-permutation policy on B200 (BASELINE.json metric).

A "step" is one SpMM C = A.B on the row-permuted CSR (a8, the timed hot path) for the policy chosen by
exhaustive timing (a10: every hot-path policy incl. the original order is built (a2-a7) and timed,
the fastest wins).  The permutation builds are offline / amortised and reported per policy as
build_ms; features (a9) are timed and reported as features_ms.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl ours|reference]

N>1 (torchrun): A is row-sharded by equal nnz (spmm_partition_by_nnz), each rank permutes its shard,
B is broadcast with NCCL (outside the timed region, "B resident"), C stays row-sharded; value = total
flops / max-over-ranks time (strong scaling: the matrix is fixed).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synthetic as syn  # noqa: E402

CONFIGS = {
    # BASELINE.json configs[i] -> synthetic recipe
    "c1": dict(desc="configs[0]: power-law R-MAT S=12 natural, M=N=4096, nnz~40k, K=32", gen=("rmat", 12, 12, 1000, "natural"), K=32),
    "c2": dict(desc="configs[1]: banded FEM-like 27-point stencil 100^3, M=N=1M, ~27 nnz/row, K=64", gen=("stencil", 100, 2000), K=64),
    "c3": dict(desc="configs[2]: power-law R-MAT S=22 'local' (80% in-community columns), M=N=4M, nnz~100M, K=128",
               gen=("rmat", 22, 28, 3000, "local"), K=128),
    "c3rl": dict(desc="configs[2] stress variant: power-law R-MAT S=22 random-label, M=N=4M, nnz~100M, K=128",
                 gen=("rmat", 22, 28, 3001, "random-label"), K=128),
    "c5": dict(desc="configs[4]: power-law R-MAT S=24 'local', M=N=16M, nnz~500M, K=128", gen=("rmat", 24, 38, 5000, "local"), K=128),
    "c3sh": dict(desc="configs[2] with its rows randomly relabelled (seeded shuffle; columns unchanged): the original "
                      "order has no locality, the column-similarity orders must recover the communities",
                 gen=("rmat", 22, 28, 3000, "local"), shuffle=3002, K=128),
    "c5rl": dict(desc="configs[4] stress variant: power-law R-MAT S=24 random-label, M=N=16M, nnz~500M, K=128",
                 gen=("rmat", 24, 38, 5001, "random-label"), K=128),
    "c5sh": dict(desc="configs[4] with its rows randomly relabelled (seeded shuffle; columns unchanged)",
                 gen=("rmat", 24, 38, 5000, "local"), shuffle=5002, K=128),
}
HOT = ["identity", "nnz_sort", "plain_sort", "cta_aware", "hybrid_1", "hybrid_2_1", "cta_aware+mh", "cta_aware+md"]
# "+mh" / "+md": the chain policy with its windows over the MinHash / median-block pre-order (spmm_params.preorder
# = 1 / 2)
METRIC = "SpMM GFLOP/s and % HBM roofline per permutation policy at 1/2/4/8 B200"


def make_matrix(cfg):
    g = cfg["gen"]
    a = syn.rmat(g[1], g[2], g[3], g[4]) if g[0] == "rmat" else syn.stencil27(g[1], g[2])
    if cfg.get("shuffle") is not None:   # row relabel: new row r = old row q[r]
        q = np.random.default_rng(cfg["shuffle"]).permutation(a.M)
        lens = np.diff(a.rowidx)[q]
        r = np.zeros(a.M + 1, dtype=np.int64)
        np.cumsum(lens, out=r[1:])
        idx = np.repeat(a.rowidx[q] - r[:-1], lens) + np.arange(a.nnz, dtype=np.int64)
        a = syn.CSR(a.M, a.N, r, a.colidx[idx], a.value[idx])
    return a


def permute_spec(h, pol, window):
    """A policy name, optionally with '+mh' / '+md': chain windows over the MinHash / median-block pre-order
    (spmm_params.preorder = 1 / 2; parsed by the binding's SpMM.permute)."""
    return h.permute(pol, window=window)


def algorithmic_bytes(a, K):
    """4(M+1) + 8 nnz + 4K|cols(A)| + 4MK  (BASELINE.json north star)."""
    seen = np.zeros(a.N, dtype=bool)
    seen[a.colidx] = True
    ncols = int(seen.sum())
    return 4 * (a.M + 1) + 8 * a.nnz + 4 * K * ncols + 4 * a.M * K, ncols


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """SM clock + clock-event (throttle) reasons sampled during the timed region: NVML every 10 ms (pynvml, the
    device matched by PCI bus id), else nvidia-smi every 200 ms."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
    # NVML clocks-event reason bits for NAMES (nvmlClocksEventReason*: HwSlowdown 0x8, HwThermalSlowdown 0x40,
    # SwThermalSlowdown 0x20, SwPowerCap 0x4)
    BITS = [0x8, 0x40, 0x20, 0x4]

    def __init__(self, index=0):
        self.index = index
        self.samples = []          # (sm_mhz, max_mhz, [reason flags])
        self.power = []            # board power draw, W (NVML only)
        self.power_limit = None
        self.source = None
        self._stop = threading.Event()
        self._t = None

    def _nvml_handle(self):
        import pynvml
        import torch
        pynvml.nvmlInit()
        try:
            pr = torch.cuda.get_device_properties(self.index)
            bus = f"{pr.pci_domain_id:08x}:{pr.pci_bus_id:02x}:{pr.pci_device_id:02x}.0"
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:  # noqa: BLE001
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def start(self):
        try:
            nv, hd = self._nvml_handle()
            mx = float(nv.nvmlDeviceGetMaxClockInfo(hd, nv.NVML_CLOCK_SM))
            self.source = "nvml 10 ms"
            try:
                self.power_limit = nv.nvmlDeviceGetEnforcedPowerLimit(hd) / 1000.0
            except Exception:  # noqa: BLE001
                self.power_limit = None
        except Exception:  # noqa: BLE001
            nv = hd = None
            self.source = "nvidia-smi 200 ms"

        def run():
            while not self._stop.is_set():
                try:
                    if nv is not None:
                        sm = float(nv.nvmlDeviceGetClockInfo(hd, nv.NVML_CLOCK_SM))
                        r = int(nv.nvmlDeviceGetCurrentClocksEventReasons(hd))
                        self.samples.append((sm, mx, [bool(r & b) for b in self.BITS]))
                        try:
                            self.power.append(nv.nvmlDeviceGetPowerUsage(hd) / 1000.0)
                        except Exception:  # noqa: BLE001
                            pass
                    else:
                        out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                              "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                             timeout=5).stdout.strip()
                        f = [x.strip() for x in out.split(",")]
                        if len(f) >= 6 and f[0].replace(".", "").isdigit():
                            self.samples.append((float(f[0]), float(f[1]),
                                                 ["Active" in x and "Not" not in x for x in f[2:6]]))
                except Exception:  # noqa: BLE001
                    pass
                self._stop.wait(0.01 if nv is not None else 0.2)
        self._t = threading.Thread(target=run, daemon=True)
        self._t.start()

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)
        sm = [s[0] for s in self.samples]
        mx = [s[1] for s in self.samples]
        reasons = sorted({self.NAMES[i] for s in self.samples for i in range(4) if s[2][i]})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples), "source": self.source,
                "power_w": statistics.median(self.power) if self.power else None, "power_limit_w": self.power_limit}


def time_runs(torch, fn, steps, flush, stream, after=None):
    """Per-step CUDA-event times (ms) on `stream`, L2 flushed before each step (outside the events).
    `after()` (optional) is called once per step after the step's end event completed."""
    ts = []
    for _ in range(steps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
        if after is not None:
            after()
    return ts


def oracle_sample_rows(a, target_nnz, seed=7):
    """Seeded sample of whole rows with about target_nnz non-zeros (bounded CPU baseline work)."""
    rng = np.random.default_rng(seed)
    order = rng.permutation(a.M)
    lens = np.diff(a.rowidx)[order]
    cut = int(np.searchsorted(np.cumsum(lens), target_nnz)) + 1
    rows = np.sort(order[:cut])
    return rows, int(np.diff(a.rowidx)[rows].sum())


def cpu_baseline(a, B, K, budget_s=15.0, single_thread=False):
    """The oracle (oracle.c, float64, OpenMP) as it stands, on a bounded row sample, on this host's cores."""
    import oracle
    # every core of this process's affinity set, replacing any inherited OMP_NUM_THREADS (torchrun sets 1);
    # `cores` is the thread count OpenMP reports in effect
    cores = oracle.set_threads(len(os.sched_getaffinity(0)))
    rows, snnz = oracle_sample_rows(a, 200_000)
    t0 = time.perf_counter()
    oracle.spmm(a, B, rows=rows)
    dt = time.perf_counter() - t0
    # scale the sample so the measured work lasts about budget_s (capped at the whole matrix)
    scale = min(max(budget_s / max(dt, 1e-3), 1.0), a.nnz / max(snnz, 1))
    if scale > 1.5:
        rows, snnz = oracle_sample_rows(a, int(snnz * scale))
        t0 = time.perf_counter()
        oracle.spmm(a, B, rows=rows)
        dt = time.perf_counter() - t0
    res = {"value": 2.0 * snnz * K / dt / 1e9, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
           "sample": f"{len(rows)} seeded random whole rows ({snnz} nnz of {a.nnz}), K={K}, float64 oracle_spmm_rows",
           "seconds": dt}
    if single_thread:   # a 1-thread number beside the all-core one (C1 / C2)
        oracle.set_threads(1)
        rows1, snnz1 = oracle_sample_rows(a, max(1, snnz // max(cores, 1)))
        t0 = time.perf_counter()
        oracle.spmm(a, B, rows=rows1)
        dt1 = time.perf_counter() - t0
        oracle.set_threads(cores)
        res["single_thread"] = {"value": 2.0 * snnz1 * K / dt1 / 1e9, "unit": "GFLOP/s", "cores": 1,
                                "sample": f"{len(rows1)} rows ({snnz1} nnz)", "seconds": dt1}
    return res


def run_reference(args):
    """--impl reference: the CPU oracle timed as it stands (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cfg = CONFIGS[args.config]
    a = make_matrix(cfg)
    K = cfg["K"]
    B = syn.dense(a.N, K, cfg["gen"][-2] + 1 if cfg["gen"][0] == "rmat" else cfg["gen"][2] + 1)
    import oracle
    cores = oracle.set_threads(len(os.sched_getaffinity(0)))   # overrides torchrun's OMP_NUM_THREADS=1
    rows, snnz = oracle_sample_rows(a, args.ref_sample_nnz)
    for _ in range(args.warmup):
        oracle.spmm(a, B, rows=rows[: max(1, len(rows) // 10)])
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.spmm(a, B, rows=rows)
        ts.append(time.perf_counter() - t0)
    tot = sum(ts)
    val = 2.0 * snnz * K * args.steps / tot / 1e9
    sample = f"each step: {len(rows)} seeded random whole rows ({snnz} nnz of {a.nnz}), K={K}, float64 oracle"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * tot / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": cfg["desc"], "M": a.M, "N": a.N, "nnz": a.nnz, "K": K},
        "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }))


def timed_max(torch, dist, world, fn, reps, stream):
    """Mean CUDA-event time (ms) of fn() on `stream`, barrier before each rep, max over ranks."""
    ts = []
    for _ in range(reps):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    t = torch.tensor([statistics.mean(ts)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def measure_exchange(torch, dist, sh, h, Bd, Cd, Bfull, K, compact, stream, reps=5, chunks=None, multicast=False):
    """N>1: the data-path communication of the sharded mode, timed on the device (max over
    ranks) and reported in GB/s of bytes moved between GPUs:
      b_exchange   -- per-rank B rows (distribute_B) or the broadcast of all of B;
      c_allgather  -- NCCL all_gather of the C shards (allgather_C);
      fused        -- the SpMM with its epilogue storing every row into every rank's symmetric-memory full-C
                      buffer (spmm_run_to), against the plain SpMM: the all-gather's added cost;
      multicast    -- the same through the NVLS multicast address (spmm_run_multicast), where the group has one;
      pipelined    -- one end-to-end step with B sent in column chunks, the SpMM of chunk c overlapping the
                      transfer of chunk c + 1 (run_pipelined), against the sequential exchange + SpMM."""
    world = sh.world
    out = {}
    mine = torch.tensor([Bd.shape[0]], dtype=torch.int64, device="cuda")
    every = [torch.empty_like(mine) for _ in range(world)]
    dist.all_gather(every, mine)
    b_rows = [int(t.item()) for t in every]          # B rows each rank holds
    b_bytes = (sum(b_rows) - b_rows[0]) * K * 4 if compact else (world - 1) * sh.N * K * 4   # sent by rank 0
    if compact:
        fn_b = lambda: sh.distribute_B(Bfull, K=K, src=0, device=Bd.device)  # noqa: E731
    else:
        fn_b = lambda: sh.broadcast_B(Bd, src=0)  # noqa: E731
    tb = timed_max(torch, dist, world, fn_b, reps, stream)
    out["b_exchange"] = {"ms": tb, "bytes": b_bytes, "GBps": b_bytes / (tb * 1e-3) / 1e9,
                         "how": "distribute_B (NCCL sends of B[cols_p])" if compact else "NCCL broadcast"}
    if compact:
        # B arriving row-sharded (rank q owns rows [bo[q], bo[q+1])): one all-to-allv of exactly the referenced rows
        bo = sh.b_owner_bounds()
        n_q = int(bo[sh.rank + 1] - bo[sh.rank])
        if sh.rank == 0:
            for q in range(1, world):
                sh.comm.send(Bfull[int(bo[q]):int(bo[q + 1])], q)
            Bsl = Bfull[:n_q].contiguous()
        else:
            Bsl = torch.empty((n_q, K), dtype=torch.float32, device=Bd.device)
            sh.comm.recv(Bsl, 0)
        sh.setup_alltoall(Bd.device)
        Ba = sh.exchange_B_alltoall(Bsl, K)
        same = bool(torch.equal(Ba, Bd))
        ta = timed_max(torch, dist, world, lambda: sh.exchange_B_alltoall(Bsl, K), reps, stream)
        moved = torch.tensor([Bd.shape[0] - sh._a2a_need[sh.rank]], dtype=torch.int64, device=Bd.device)
        dist.all_reduce(moved)       # rows that crossed GPUs (a rank's own slice stays local)
        out["b_alltoall"] = {"ms": ta, "bytes": int(moved.item()) * K * 4,
                             "GBps_aggregate": int(moved.item()) * K * 4 / (ta * 1e-3) / 1e9,
                             "equals_distribute_B": same,
                             "how": "B row-sharded over the ranks; exchange_B_alltoall (one all-to-allv of B[cols_p])"}
        del Bsl, Ba
    c_bytes = (sh.M - Cd.shape[0]) * K * 4      # the other ranks' C rows this rank receives
    tc = timed_max(torch, dist, world, lambda: sh.allgather_C(Cd), reps, stream)
    out["c_allgather"] = {"ms": tc, "bytes_received_rank": c_bytes, "GBps_received_rank": c_bytes / (tc * 1e-3) / 1e9,
                          "how": "NCCL all_gather of padded shards (allgather_C)"}
    t_plain = timed_max(torch, dist, world, lambda: h.run(Bd, Cd), reps, stream)
    out["spmm_ms"] = t_plain
    if sh.comm.nccl:
        try:
            buf, ptrs, hdl = sh.symmetric_C(K)
            t_f = timed_max(torch, dist, world, lambda: sh.run_allgather_fused(Bd, ptrs), reps, stream)
            out["fused"] = {"ms": t_f, "allgather_added_ms": t_f - t_plain,
                            "GBps_per_rank_out": (world - 1) * Cd.shape[0] * K * 4 / max(t_f * 1e-3, 1e-9) / 1e9,
                            "how": "spmm_run_to: per-peer stores into the symmetric-memory full-C buffers"}
            mc = int(getattr(hdl, "multicast_ptr", 0) or 0)
            if mc and multicast:        # opt-in (--multicast): the NVLS store path has not run on hardware yet
                t_m = timed_max(torch, dist, world, lambda: sh.run_allgather_multicast(Bd, mc), reps, stream)
                out["multicast"] = {"ms": t_m, "allgather_added_ms": t_m - t_plain,
                                    "how": "spmm_run_multicast: one multimem.st per element (NVLS)"}
            else:
                out["multicast"] = {"skipped": "no multicast address" if not mc else "not requested (--multicast)"}
            del buf
        except Exception as e:  # noqa: BLE001
            out["fused"] = {"error": str(e)[:200]}
    else:
        out["fused"] = {"skipped": "symmetric memory needs NCCL"}
    if compact:
        Cp = torch.empty_like(Cd)
        t_seq = timed_max(torch, dist, world, lambda: h.run(fn_b(), Cd), reps, stream)
        t_pipe = timed_max(torch, dist, world, lambda: sh.run_pipelined(Bfull, K=K, chunks=chunks, C_local=Cp,
                                                                         src=0, device=Bd.device), reps, stream)
        torch.cuda.synchronize()
        out["pipelined"] = {"ms": t_pipe, "sequential_ms": t_seq, "chunks": chunks or max(1, K // 64),
                            "bit_identical_to_run": bool(torch.equal(Cp.view(torch.int32), Cd.view(torch.int32)))}
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="c5", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--policies", default=",".join(HOT))
    ap.add_argument("--window", type=int, default=1024)
    ap.add_argument("--policy-steps", type=int, default=5, help="timed steps per policy for the exhaustive selection")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--e2e-pipe-steps", type=int, default=16,
                    help="right-hand sides per pipelined end-to-end measurement (fill and drain amortised over them)")
    ap.add_argument("--ref-sample-nnz", type=int, default=10_000_000)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-cusparse", action="store_true")
    ap.add_argument("--no-ceiling", action="store_true", help="skip the host LRU model of L2 reuse")
    ap.add_argument("--out", default=None, help="also write the JSON line to this file")
    ap.add_argument("--multicast", action="store_true",
                    help="N>1: also time the C all-gather through NVLS multicast stores (spmm_run_multicast)")
    ap.add_argument("--b-exchange", default="rows", choices=["rows", "broadcast"],
                    help="N>1: send each rank only the B rows its shard references (rows) or broadcast all of B")
    args = ap.parse_args()
    assert args.warmup >= 3, "timing rules: at least 3 warm-up steps"
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    import paper_conf_ispass_mehrabilcslo21_b200 as pkg

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # BENCH_GPU_INDEX / BENCH_DIST_BACKEND: test hooks only (dry-run of the N>1 path with several ranks on one
    # GPU over gloo); the driver's runs use one GPU per rank and NCCL
    local = int(os.environ.get("BENCH_GPU_INDEX", local))
    torch.cuda.set_device(local)
    if world > 1:
        backend = os.environ.get("BENCH_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    cfg = CONFIGS[args.config]
    K = cfg["K"]
    bseed = (cfg["gen"][3] if cfg["gen"][0] == "rmat" else cfg["gen"][2]) + 1

    t0 = time.perf_counter()
    a_full = make_matrix(cfg) if rank == 0 else None
    gen_s = time.perf_counter() - t0
    compact = world > 1 and args.b_exchange == "rows"
    pkg.use_torch_allocator(True)
    sh = None
    if world == 1:
        h = pkg.SpMM.from_csr(a_full)
        Mr, lo, N, N_loc, nnz_r, nnz_total = a_full.M, 0, a_full.N, a_full.N, a_full.nnz, a_full.nnz
        seen = np.zeros(a_full.N, dtype=bool)
        seen[a_full.colidx] = True
        ncols = int(seen.sum())
        del seen
    else:
        # one sharding path (sharded.py): rank 0 partitions by nnz and sends every rank its own shard (NCCL p2p of
        # device tensors; compact columns with --b-exchange rows); no rank holds another rank's rows
        from paper_conf_ispass_mehrabilcslo21_b200.sharded import ShardedSpMM
        sh = ShardedSpMM.scatter(a_full if rank == 0 else None, src=0, compact_B=compact, device=dev)
        h = sh.local
        Mr, lo, N, N_loc, nnz_r = sh.shard.M, sh.row_offset, sh.N, sh.shard.N, sh.shard.nnz
        cidx = torch.as_tensor(sh.shard.colidx).to(dev).long()
        seen = torch.zeros(N_loc, dtype=torch.bool, device=dev)
        seen[cidx] = True
        ncols = int(seen.sum().item())
        del seen, cidx
        nt = torch.tensor([nnz_r], dtype=torch.int64, device=dev)
        dist.all_reduce(nt)
        nnz_total = int(nt.item())
    alg_bytes = 4 * (Mr + 1) + 8 * nnz_r + 4 * K * ncols + 4 * Mr * K   # north star, this rank's shard
    flops = 2.0 * nnz_r * K
    total_flops = 2.0 * nnz_total * K

    # B: drawn on rank 0 (host); N>1: broadcast over NCCL, or (--b-exchange rows, default) each rank receives
    # only the rows its shard references (sharded.py distribute_B: NCCL sends of B[cols_p]) -- outside the timed region
    B_host = torch.from_numpy(syn.dense(N, K, bseed)) if rank == 0 else None
    Bfull = None
    if world == 1:
        Bd = B_host.to(dev)
    elif compact:
        Bfull = B_host.to(dev) if rank == 0 else None
        Bd = sh.distribute_B(Bfull, K=K, src=0, device=dev)
    else:
        Bd = B_host.to(dev) if rank == 0 else torch.empty((N, K), dtype=torch.float32, device=dev)
        sh.broadcast_B(Bd, src=0)
    Cd = torch.empty((Mr, K), dtype=torch.float32, device=dev)
    flush_buf = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)   # 256 MiB > 126 MB L2

    def flush():
        flush_buf.fill_(1.0)

    torch.cuda.synchronize()
    feat_t0 = time.perf_counter()
    feats = h.features()
    features_ms = 1e3 * (time.perf_counter() - feat_t0)
    a_host = None
    if rank == 0 and not args.no_ceiling:
        r0, r1 = int(a_full.rowidx[0]), int(a_full.rowidx[Mr])
        a_host = syn.CSR(Mr, N, a_full.rowidx[:Mr + 1] - r0, a_full.colidx[r0:r1], a_full.value[r0:r1])

    # ---- exhaustive per-policy timing (a10) ----
    pol_res = {}
    for pol in args.policies.split(","):
        torch.cuda.synchronize()
        tb = time.perf_counter()
        permute_spec(h, pol, args.window)
        build_ms = 1e3 * (time.perf_counter() - tb)
        for _ in range(args.warmup):
            h.run(Bd, Cd)
        ts = time_runs(torch, lambda: h.run(Bd, Cd), args.policy_steps, flush, stream)
        ms = statistics.median(ts)
        pol_res[pol] = {"ms": ms, "gflops": flops / ms / 1e6, "build_ms": build_ms, "launches": h.last_run_launches(),
                        "info": h.info(), "schedule": h.schedule_info()}
        if a_host is not None:
            # L2-capacity ceiling: B-row misses of an LRU of L2 size in this order
            import tools
            cap = int(torch.cuda.get_device_properties(dev).L2_cache_size // (4 * K))
            miss = tools.lru_misses(a_host, h.perm(), cap)
            traffic = alg_bytes - 4 * K * ncols + 4 * K * miss
            pol_res[pol]["lru_model"] = {"l2_rows": cap, "b_row_misses": miss, "model_bytes": traffic,
                                         "ceiling_frac": alg_bytes / traffic}
    # choose the fastest (max over ranks of each policy's time)
    names = list(pol_res)
    tvec = torch.tensor([pol_res[n]["ms"] for n in names], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tvec, op=dist.ReduceOp.MAX)
    best = names[int(torch.argmin(tvec))]
    permute_spec(h, best, args.window)

    # ---- the timed region: `steps` steps of the selected policy ----
    for _ in range(args.warmup):
        h.run(Bd, Cd)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = ClockSampler(local)
    clk.start()
    h.set_kernel_timing(True)      # library CUDA events around the main SpMM kernel (dominant-kernel roofline)
    kms = []
    torch.cuda.synchronize()
    ts = time_runs(torch, lambda: h.run(Bd, Cd), args.steps, flush, stream, after=lambda: kms.append(h.last_kernel_ms()))
    torch.cuda.synchronize()
    h.set_kernel_timing(False)
    if world > 1:
        dist.barrier()
    clocks = clk.stop()
    launches = h.last_run_launches() * args.steps
    tot_ms = torch.tensor([sum(ts)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot_ms, op=dist.ReduceOp.MAX)
    ms_step = float(tot_ms.item()) / args.steps
    value = total_flops / ms_step / 1e6   # GFLOP/s, whole job
    peak, peak_src = peaks()
    # dominant kernel (the row-group SpMM kernel): its algorithmic bytes exclude the empty rows' C rows,
    # which the separate zero-fill launch writes; the whole step is reported beside it
    n_empty_r = int(pol_res[best]["info"]["empty_rows"])
    kern_bytes = alg_bytes - 4 * K * n_empty_r
    kern_ms = statistics.mean(kms) if kms and min(kms) > 0 else None
    achieved = kern_bytes / (kern_ms * 1e-3) / 1e9 if kern_ms else alg_bytes / (statistics.mean(ts) * 1e-3) / 1e9
    step_achieved = alg_bytes / (statistics.mean(ts) * 1e-3) / 1e9
    l2 = None
    if rank == 0:
        # second ceiling: the SM load path.  Every B-row load (one per nnz, or one per union record of a fused row
        # group) brings 4K bytes into registers; tools/ldpathprobe.cu measures how many bytes per SM clock k_spmm's
        # load shape (8-lane groups x one 256-bit load per lane, random rows) can gather from an L2-resident window
        # and from an L1-resident one.  At the clock sampled in the timed region, 4K * loads / that rate bounds the
        # kernel whatever HBM does.
        try:
            import tools
            sch = pol_res[best]["schedule"]
            loads = (nnz_r - sch["fused_nnz"] + sch["records"]) if sch["fuse"] > 1 else nnz_r
            g_bytes = 4.0 * K * loads
            l2_gbs, l2_bpc = tools.ldpath_gather(0, 16 << 20, 4 * K)
            l1_gbs, l1_bpc = tools.ldpath_gather(0, 32 << 10, 4 * K)
            nsm = torch.cuda.get_device_properties(dev).multi_processor_count
            mhz = clocks.get("sm_mhz") or clocks.get("sm_max_mhz") or 1965.0
            l2_at_clk = l2_bpc * nsm * mhz * 1e6 / 1e9
            l2 = {"gather_l2_gbs": l2_gbs, "gather_l2_bytes_per_sm_clk": l2_bpc,
                  "gather_l1_gbs": l1_gbs, "gather_l1_bytes_per_sm_clk": l1_bpc,
                  "b_row_loads_per_launch": loads, "b_row_bytes_per_launch": g_bytes,
                  "timed_region_sm_mhz": mhz, "gather_l2_gbs_at_timed_clock": l2_at_clk,
                  "kernel_frac_of_l2_gather_ceiling": (g_bytes / (kern_ms * 1e-3) / 1e9) / l2_at_clk if kern_ms else None,
                  "hbm_ceiling_frac_without_l1_reuse": (kern_bytes / peak) / (g_bytes / l2_at_clk),
                  "how": "tools/ldpathprobe.cu shape 0 (k_spmm's load shape) over a 16 MiB (L2) / 32 KiB (L1) window of "
                         f"random {4 * K}-byte rows; bytes per SM clock x SMs x the timed region's median SM clock"}
        except Exception as e:  # noqa: BLE001
            l2 = {"error": str(e)[:200]}

    multi = (measure_exchange(torch, dist, sh, h, Bd, Cd, Bfull, K, compact, stream, multicast=args.multicast)
             if world > 1 else None)

    # ---- e2e through the public API with host buffers ----
    # N=1: spmm_run_host (H2D of B, SpMM, D2H of C).  N>1: rank 0 H2D of B, NCCL broadcast, SpMM on every
    # shard, D2H of every C shard; max over ranks.
    # N>1 with per-rank B rows: every rank's step starts from ITS rows of B in pinned host memory (the host keeps
    # the input partitioned per GPU, prepared outside the timed region like any input) and copies them over its
    # own PCIe link; with --b-exchange broadcast, rank 0 copies all of B and NCCL broadcasts it.
    Cp = torch.empty((Mr, K), dtype=torch.float32).pin_memory()
    if world == 1 or not compact:
        Bp = B_host.pin_memory() if rank == 0 else None
    else:
        Bp = Bd.cpu().pin_memory()

    def e2e_step():
        if world == 1:
            h.run_host(Bp, Cp)
        else:
            if compact:
                Bd.copy_(Bp, non_blocking=True)
            else:
                if rank == 0:
                    Bd.copy_(Bp, non_blocking=True)
                sh.broadcast_B(Bd, src=0)
            h.run(Bd, Cd)
            Cp.copy_(Cd, non_blocking=True)
            torch.cuda.current_stream().synchronize()
    e2e_step()
    e2e_ts = []
    for _ in range(max(3, args.e2e_steps)):
        if world > 1:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        e2e_step()
        e1.record(stream)
        e1.synchronize()
        e2e_ts.append(e0.elapsed_time(e1))
    e2e_t = torch.tensor([statistics.mean(e2e_ts)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    # pipelined e2e (N=1): spmm_run_host_batch over the timed steps -- every step still copies its whole B in
    # and its whole C out, but the H2D of step i+1 and the D2H of step i-1 overlap the SpMM of step i
    e2e_pipe = None
    if world == 1:
        try:
            nst = max(3, args.e2e_pipe_steps)
            Cp2 = [Cp, torch.empty((Mr, K), dtype=torch.float32).pin_memory()]
            Bs, Cs = [Bp] * nst, [Cp2[i % 2] for i in range(nst)]
            h.run_host_batch(Bs[:2], Cs[:2])          # warm-up (slots, streams)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            h.run_host_batch(Bs, Cs)
            e1.record(stream)
            e1.synchronize()
            pms = e0.elapsed_time(e1) / nst
            e2e_pipe = {"value": total_flops / pms / 1e6, "unit": "GFLOP/s", "ms_per_step": pms, "steps": nst,
                        "path": "spmm_run_host_batch (double-buffered, H2D/D2H overlapped with the SpMM)"}
            del Cp2
        except Exception as e:  # noqa: BLE001
            e2e_pipe = {"error": str(e)[:200]}
    rows_tot = torch.tensor([N_loc, Mr], dtype=torch.int64, device=dev)   # B rows copied in, C rows copied out
    if world > 1:
        dist.all_reduce(rows_tot)
    h2d = int(rows_tot[0].item()) * K * 4 if compact else N * K * 4
    e2e = {"value": total_flops / float(e2e_t.item()) / 1e6, "unit": "GFLOP/s",
           "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(rows_tot[1].item()) * K * 4,
           "ms_per_step": float(e2e_t.item()),
           "path": "spmm_run_host" if world == 1 else
           ("per-rank H2D of its B rows (pinned) + spmm_run + D2H of its C shard" if compact else
            "H2D(B) on rank 0 + NCCL broadcast + spmm_run + D2H(C shards)")}
    if e2e_pipe is not None:
        e2e["pipelined"] = e2e_pipe
        # headline E = the pipelined public API when it ran: still every step copies its whole B in and its whole
        # C out inside the timed region; the one-call-at-a-time number stays under "sequential"
        if "value" in e2e_pipe and e2e_pipe["value"] > e2e["value"]:
            e2e["sequential"] = {"value": e2e["value"], "ms_per_step": e2e["ms_per_step"], "path": e2e["path"]}
            e2e["value"] = e2e_pipe["value"]
            e2e["ms_per_step"] = e2e_pipe["ms_per_step"]
            e2e["path"] = e2e_pipe["path"]

    # ---- cuSPARSE comparator: cusparseSpMM CSR ALG1/ALG2/ALG3 and the default algorithm, row-major B and C,
    # best-of (tools/cusparse_ref.cu), same inputs, same L2 flush, rank 0 shard ----
    cus = None
    if not args.no_cusparse and rank == 0:
        import tools
        src_csr = a_full if world == 1 else sh.shard
        rp32 = torch.as_tensor(np.asarray(src_csr.rowidx)).to(dev).to(torch.int32)
        colidx_d = torch.as_tensor(np.asarray(src_csr.colidx)).to(dev)
        value_d = torch.as_tensor(np.asarray(src_csr.value)).to(dev)
        Cc = torch.empty_like(Cd)
        h.run(Bd, Cd)                 # our C of the selected policy, for the sanity diff
        torch.cuda.synchronize()
        per_alg = {}
        for alg, name in ((0, "default"), (1, "csr_alg1"), (2, "csr_alg2"), (3, "csr_alg3")):
            try:
                cts = tools.cusparse_spmm_times(Mr, N_loc, nnz_r, rp32.data_ptr(), colidx_d.data_ptr(), value_d.data_ptr(),
                                                Bd.data_ptr(), K, Cc.data_ptr(), alg, max(3, args.policy_steps),
                                                (flush_buf.data_ptr(), flush_buf.numel() * 4), stream.cuda_stream)
                torch.cuda.synchronize()
                # sanity: the library's C against ours (both fp32; reported, not asserted)
                diff = float((Cc - Cd).abs().max().item())
                per_alg[name] = {"ms": statistics.median(cts), "max_abs_diff_vs_ours": diff}
            except Exception as e:  # noqa: BLE001
                per_alg[name] = {"error": str(e)[:160]}
        ok = {k: v for k, v in per_alg.items() if "ms" in v}
        if ok:
            bname = min(ok, key=lambda k: ok[k]["ms"])
            cms = ok[bname]["ms"]
            cus = {"ms": cms, "gflops": flops / cms / 1e6, "best_alg": bname, "per_alg": per_alg,
                   "speedup_best_vs_cusparse": cms / pol_res[best]["ms"],
                   "speedup_identity_vs_cusparse": cms / pol_res["identity"]["ms"] if "identity" in pol_res else None,
                   "via": "cusparseSpMM (CUSPARSE_SPMM_CSR_ALG1/2/3, default), row-major, best-of, rank 0 shard"}
        else:
            cus = {"error": "no cuSPARSE algorithm ran", "per_alg": per_alg}
        del Cc, rp32, colidx_d, value_d

    if rank != 0:
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        h.close()
        return
    cpu = None
    if not args.no_cpu_baseline and world == 1:
        cpu = cpu_baseline(a_full, B_host.numpy(), K, single_thread=args.config in ("c1", "c2"))
    # DRAM bytes of one k_spmm launch of the SELECTED policy on this config, from the committed ncu --set full
    # capture (scripts/profile_policies.py -> scripts/collect_profiles.py); null when that policy has none
    traffic, traffic_from = None, f"no committed ncu capture of {args.config}/{best}"
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof) and world == 1:
        d = json.load(open(prof)).get(f"{args.config}/{best}")
        if d:
            traffic = d.get("dram_bytes_per_launch")
            traffic_from = f"ncu --set full of {d.get('kernel', 'k_spmm')} on {args.config}/{best} ({d.get('round')})"

    for pol, r in pol_res.items():
        r["roofline_frac"] = alg_bytes / (r["ms"] * 1e-3) / 1e9 / peak
        r["speedup_vs_identity"] = pol_res["identity"]["ms"] / r["ms"] if "identity" in pol_res else None
    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": cfg["desc"], "M": a_full.M if world == 1 else sh.M, "N": N, "nnz": nnz_total, "K": K,
                   "policy": best, "window": args.window, "parallelism": f"rows sharded by nnz over {world} GPU(s)",
                   "b_exchange": ("per-rank B rows (compact shards)" if compact else "broadcast") if world > 1 else None,
                   "l2": "256 MiB scratch written between timed steps (L2 flush); B, C also > L2",
                   "selection": "exhaustive timing over " + ",".join(pol_res),
                   "schedule": h.schedule_info()},
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic, "traffic_from": traffic_from,
                     "algorithmic_bytes_per_launch": kern_bytes, "distinct_columns": ncols,
                     "kernel": "k_spmm (row-group SpMM, rank 0 shard): CUDA events recorded by the library on the "
                               "launch stream around the kernel (spmm_set_kernel_timing), mean over the timed steps",
                     "kernel_ms": kern_ms, "share_of_step": (kern_ms / statistics.mean(ts)) if kern_ms else None,
                     "step": {"achieved": step_achieved, "frac": step_achieved / peak, "algorithmic_bytes": alg_bytes,
                              "what": "whole spmm_run = k_zero_rows + k_spmm + k_combine"},
                     "peak_source": peak_src, "l2": l2},
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": launches,
        "multi_gpu": multi,
        "clocks": clocks,
        "policies": pol_res,
        "cusparse": cus,
        "features_ms": features_ms, "features": dict(zip(pkg.FEATURE_NAMES, map(float, feats))),
        "gen_seconds": gen_s,
        "paper_context": "paper (GV100/2080 Ti, FP32, K=N<=30K): best permutation 1.4x over plain CSR, 2.6x over cuSPARSE",
    }
    print(json.dumps(line))
    if args.out:
        with open(args.out, "w") as f:
            f.write(json.dumps(line) + "\n")
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    h.close()


if __name__ == "__main__":
    main()
