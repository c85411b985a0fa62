import sys, json, statistics, torch
sys.path.insert(0, '.')
import bench, synthetic as syn, paper_conf_ispass_mehrabilcslo21_b200 as pkg
cfg = bench.CONFIGS["c2"]; a = bench.make_matrix(cfg); K = cfg["K"]
pkg.use_torch_allocator(True)
B = torch.from_numpy(syn.dense(a.N, K, 2001)).cuda(); C = torch.empty((a.M, K), device="cuda")
h = pkg.SpMM.from_csr(a)
flush = torch.empty(64 * 1024 * 1024, device="cuda")
res = []
for pol in ("identity", "cta_aware", "hybrid_2_1", "cta_aware+md"):
    for bw in (32, 16, 8, 4, 2, 1):
        if pol == "identity" and bw != 32: continue
        h.permute(pol, bw=bw, window=1024); h.prepare(K, B, C)
        for _ in range(3): h.run(B, C)
        h.set_kernel_timing(True); ks = []
        for _ in range(15):
            flush.fill_(1.0); h.run(B, C); ks.append(h.last_kernel_ms())
        h.set_kernel_timing(False)
        si = h.schedule_info()
        res.append(dict(policy=pol, bw=bw, ms=statistics.median(ks), records_per_nnz=si["records"] / max(si["fused_nnz"], 1)))
        print(json.dumps(res[-1]), flush=True)
