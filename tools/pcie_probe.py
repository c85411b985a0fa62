"""Measurement helper (not the method): pinned host <-> device copy bandwidth on this box, one direction alone and
both directions at once (single copies and chunked over several streams) -- the ceiling of bench.py's e2e."""
import torch, time, json

n = 1 << 29                 # 2 GiB
h_in = torch.empty(n, dtype=torch.float32).pin_memory()
h_out = torch.empty(n, dtype=torch.float32).pin_memory()
d_in = torch.empty(n, device="cuda")
d_out = torch.empty(n, device="cuda")
res = {}
def timeit(fn, reps=3):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize(); t = time.perf_counter(); fn(); torch.cuda.synchronize(); best = min(best, time.perf_counter() - t)
    return best
gb = n * 4 / 1e9
res["h2d_alone_GBps"] = gb / timeit(lambda: d_in.copy_(h_in, non_blocking=True))
res["d2h_alone_GBps"] = gb / timeit(lambda: h_out.copy_(d_out, non_blocking=True))
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def both():
    with torch.cuda.stream(s1): d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2): h_out.copy_(d_out, non_blocking=True)
res["bidir_each_GBps"] = gb / timeit(both)
for nch in (2, 4, 8):
    ss = [torch.cuda.Stream() for _ in range(2 * nch)]
    c = n // nch
    def chunked():
        for i in range(nch):
            with torch.cuda.stream(ss[i]): d_in[i*c:(i+1)*c].copy_(h_in[i*c:(i+1)*c], non_blocking=True)
            with torch.cuda.stream(ss[nch+i]): h_out[i*c:(i+1)*c].copy_(d_out[i*c:(i+1)*c], non_blocking=True)
    res[f"bidir_each_GBps_{nch}chunks"] = gb / timeit(chunked)
    def h2d_chunked():
        for i in range(nch):
            with torch.cuda.stream(ss[i]): d_in[i*c:(i+1)*c].copy_(h_in[i*c:(i+1)*c], non_blocking=True)
    res[f"h2d_alone_GBps_{nch}chunks"] = gb / timeit(h2d_chunked)
print(json.dumps(res))
