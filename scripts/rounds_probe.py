import os, sys, numpy as np, torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import dpgen, paper_conf_pldi_carteylm12_b200 as dp
g = np.random.default_rng(5)
x = g.integers(0, 4, size=1000).astype(np.uint8)
cat, off = dpgen.pack([x])
c, o = torch.from_numpy(cat).cuda(), torch.from_numpy(off).cuda()
with dp.Plan(dp.NUSSINOV, 1000, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
    out = torch.empty(1, dtype=torch.int32, device="cuda")
    p.solve_batch(c, o, max_len_a=1000, out=out); torch.cuda.synchronize()
    os.environ["DP_NUSS_ROUNDS"] = "1"; os.environ["DP_NUSS_TIMING"] = "1"
with dp.Plan(dp.NUSSINOV, 1000, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
    p.solve_batch(c, o, max_len_a=1000, out=out); torch.cuda.synchronize()
