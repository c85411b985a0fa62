"""Round-2 entry points only (for racecheck, which is too slow for the whole sanitize_driver.py within the box's
limits): run_ld, run_to, concurrent runs through the scratch slots, set_perm, median-block pre-order, nw = 1 exact
chains, spmm_prepare + CUDA-graph capture."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

# round 2: run_ld column blocks, run_to, concurrent runs on 4 streams through the scratch slots, set_perm, the
# median-block pre-order, nw = 1 exact chains, spmm_prepare + CUDA-graph capture and replay
a5 = syn.rmat(11, 10, 1001, "local")
h5 = pkg.SpMM.from_csr(a5)
h5.permute("cta_aware+md")
B5 = torch.from_numpy(syn.dense(a5.N, 128, 5)).cuda()
C5 = torch.empty((a5.M, 128), device="cuda")
for c0 in (0, 64):
    h5.run_ld(B5[:, c0:c0 + 64].contiguous(), C5, col_offset=c0)
h5.run_to(B5, [torch.empty((a5.M + 8, 128), device="cuda") for _ in range(3)], row_offset=8)
streams = [torch.cuda.Stream() for _ in range(4)]
torch.cuda.synchronize()
outs = [torch.empty((a5.M, 128), device="cuda") for _ in range(6)]
for i, Co in enumerate(outs):
    with torch.cuda.stream(streams[i % 4]):
        h5.run(B5, Co, stream=streams[i % 4])
torch.cuda.synchronize()
h5.set_perm(h5.perm()[::-1].copy())
h5.run(B5, C5)
os.environ["SPMM_CHAIN_EXACT"] = "1"
for pol in ("warp_aware", "hybrid_2_3", "hybrid_2_2"):
    h5.permute(pol, window=0, nw=1)
os.environ.pop("SPMM_CHAIN_EXACT")
h5.permute("hybrid_2_1")
h5.prepare(128, B5, C5)
torch.cuda.synchronize()
g = torch.cuda.CUDAGraph()
sg = torch.cuda.Stream()
with torch.cuda.stream(sg):
    with torch.cuda.graph(g, stream=sg):
        h5.run(B5, C5, stream=sg)
g.replay()
torch.cuda.synchronize()
h5.close()
print("sanitize driver done")
