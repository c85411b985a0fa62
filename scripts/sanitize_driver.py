"""Small pass over every entry point and policy (for compute-sanitizer)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synthetic as syn  # noqa: E402
import paper_conf_ispass_mehrabilcslo21_b200 as pkg  # noqa: E402

a = syn.rmat(11, 10, 1000, "natural")
h = pkg.SpMM.from_csr(a)
h.features()
for pol in pkg.POLICIES:
    h.permute(pol, window=256, split_nnz=64)
    for K in (32, 128, 36):
        B = torch.from_numpy(syn.dense(a.N, K, 1)).cuda()
        C = h.run(B)
    h.features(current_order=True)
torch.cuda.synchronize()
h2 = pkg.SpMM.from_csr(syn.blockcluster(3000, 5000, 32, 4, 12, 3))
h2.permute("hybrid_2_2", window=512, preorder=1, seed=3)
h2.run(torch.zeros((5000, 64), device="cuda"))
torch.cuda.synchronize()
# row fusion (forced, K = 64 -> R = 4, K = 128 -> R = 2) with a split row, the pipelined host API, B200 features
st = syn.stencil27(10, 4)
rows = [st.colidx[st.rowidx[i]:st.rowidx[i + 1]].tolist() for i in range(st.M)]
rows[7] = list(range(0, st.N, 3))
st = syn.from_lists(st.M, st.N, rows)
h3 = pkg.SpMM.from_csr(st)
for pol in ("identity", "cta_aware"):
    h3.permute(pol, fuse_rows=2)
    for K in (64, 128):
        h3.run(torch.from_numpy(syn.dense(st.N, K, 2)).cuda())
        Bs = [torch.from_numpy(syn.dense(st.N, K, 3 + i)).pin_memory() for i in range(3)]
        Cs = [torch.empty((st.M, K)).pin_memory() for _ in range(3)]
        h3.run_host_batch(Bs, Cs)
    for K in (32, 128):
        h3.features_b200(K, current_order=True)
h.features_b200(64)
torch.cuda.synchronize()
# inverted-index exact chains (k_chain_x): whole matrix and multi-window, both modes, an empty-row-rich input
os.environ["SPMM_CHAIN_EXACT"] = "1"
for wide in ("0", "1"):
    os.environ["SPMM_CHAIN_WIDE"] = wide
    for a4 in (syn.uniform(1500, 2000, 3, 5, poisson=True), syn.rmat(10, 8, 6, "local")):
        h4 = pkg.SpMM.from_csr(a4)
        for pol in ("cta_aware", "hybrid_2_1", "warp_aware", "hybrid_2_3", "hybrid_2_2", "hybrid_1"):
            for W in (0, 256):
                h4.permute(pol, window=W)
        h4.close()
os.environ.pop("SPMM_CHAIN_EXACT")
os.environ.pop("SPMM_CHAIN_WIDE")
torch.cuda.synchronize()
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
