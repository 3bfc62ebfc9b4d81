import os, sys
import numpy as np, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dpgen, paper_conf_pldi_carteylm12_b200 as dp
x = dpgen.config1_rna64(); cat, off = dpgen.pack([x])
c, o = torch.from_numpy(cat).cuda(), torch.from_numpy(off).cuda()
with dp.Plan(dp.NUSSINOV, 64, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
    for _ in range(3):
        p.solve_batch(c, o, max_len_a=64)
    torch.cuda.synchronize()
