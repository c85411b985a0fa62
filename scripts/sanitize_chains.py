"""compute-sanitizer driver for the inverted-index chain builders k_chain_x / k_chain_xl (every mode, both prefix
widths, whole-matrix and windowed) and the warp-cooperative adjacent-distance feature pass (rows > 256 nnz)."""
import os, sys
sys.path.insert(0, os.getcwd())
import torch, synthetic as syn, paper_conf_ispass_mehrabilcslo21_b200 as pkg
os.environ["SPMM_CHAIN_EXACT"] = "1"
for wide in ("0", "1"):
    os.environ["SPMM_CHAIN_WIDE"] = wide
    for a4 in (syn.uniform(600, 900, 3, 5, poisson=True), syn.rmat(9, 8, 6, "local")):
        h4 = pkg.SpMM.from_csr(a4)
        for pol in ("cta_aware", "hybrid_2_1", "warp_aware", "hybrid_2_3", "hybrid_2_2", "hybrid_1"):
            for W in (0, 128):
                h4.permute(pol, window=W)
        h4.close()
# long adjacent row pairs (> 256 nnz together) for k_adjacent's warp path, with hub-like rows
import numpy as np
rng = np.random.default_rng(3)
rows = [sorted(rng.choice(4000, size=int(n), replace=False).tolist()) for n in rng.integers(0, 700, size=300)]
hl = pkg.SpMM.from_csr(syn.from_lists(300, 4000, rows))
hl.features()
hl.permute("cta_aware", window=64)
hl.features(current_order=True)
hl.close()
torch.cuda.synchronize()
print("chain sanitize done")
