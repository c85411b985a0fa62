import sys, statistics, torch, json
sys.path.insert(0, '.')
import bench, synthetic as syn, paper_conf_ispass_mehrabilcslo21_b200 as pkg
cfg = bench.CONFIGS["c2"]; a = bench.make_matrix(cfg); K = cfg["K"]
pkg.use_torch_allocator(True)
B = torch.from_numpy(syn.dense(a.N, K, 2001)).cuda(); C = torch.empty((a.M, K), device="cuda")
h = pkg.SpMM.from_csr(a); h.permute("cta_aware"); h.prepare(K, B, C)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
lib = pkg.load_library(); s = torch.cuda.current_stream()
def direct(): lib.spmm_run(h._h, B.data_ptr(), K, C.data_ptr(), s.cuda_stream)
res = {}
for name, fn in (("h.run", lambda: h.run(B, C)), ("direct", direct), ("h.run", lambda: h.run(B, C)), ("direct", direct)):
    for _ in range(5): fn()
    ts = bench.time_runs(torch, fn, 30, lambda: flush.fill_(1.0), s)
    res.setdefault(name, []).append(statistics.median(ts))
h.set_kernel_timing(True); ks = []
for _ in range(20):
    flush.fill_(1.0); h.run(B, C); ks.append(h.last_kernel_ms())
res["kernel"] = statistics.median(ks)
print(json.dumps(res))

# the same steps under bench.py's conditions: NVML clock sampling thread + library kernel-timing events
clk = bench.ClockSampler(0)
clk.start()
h.set_kernel_timing(True)
res2 = {}
for name, fn in (("h.run+clocks+timing", lambda: h.run(B, C)),):
    ts = bench.time_runs(torch, fn, 30, lambda: flush.fill_(1.0), s, after=lambda: h.last_kernel_ms())
    res2[name] = statistics.median(ts)
h.set_kernel_timing(False)
ts = bench.time_runs(torch, lambda: h.run(B, C), 30, lambda: flush.fill_(1.0), s)
res2["h.run+clocks"] = statistics.median(ts)
clk.stop()
print(json.dumps(res2))
