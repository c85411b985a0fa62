"""compute-sanitizer driver for the inverted-index chain builder k_chain_x (every mode, both prefix widths)."""
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
torch.cuda.synchronize()
print("chain sanitize done")
