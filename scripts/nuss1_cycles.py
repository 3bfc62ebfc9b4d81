"""Config-1 probe: one 64-nt fold through the C ABI with DP_NUSS_TIMING=1 (k_nuss_small's cycle split)."""
import os
import numpy as np
import torch
import dpgen
import paper_conf_pldi_carteylm12_b200 as dp

os.environ["DP_NUSS_TIMING"] = "1"
x = dpgen.config1_rna64()
cat, off = dpgen.pack([x])
cu = lambda v: torch.from_numpy(np.ascontiguousarray(v)).cuda()
with dp.Plan(dp.NUSSINOV, 64, pair_mask=dpgen.rna_pair_mask(), min_hairpin=dpgen.NUSS_HAIRPIN, want_traceback=True) as p:
    for _ in range(3):
        p.solve_batch(cu(cat), cu(off), max_len_a=64)
        torch.cuda.synchronize()
