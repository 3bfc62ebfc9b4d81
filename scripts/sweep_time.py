import sys, numpy as np, torch
sys.path.insert(0, '.')
import dpgen, paper_conf_pldi_carteylm12_b200 as dp
a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(100_000)
cu = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
A = (cu(a_cat), cu(a_off), cu(b_cat), cu(b_off))
p = dp.Plan(dp.SW_LINEAR, 256, 256, sigma=dpgen.blosum62(), gap=dpgen.SW_GAP, want_traceback=True)
for _ in range(3): p.solve_batch(*A, max_len_a=256, max_len_b=256)
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(20): p.solve_batch(*A, max_len_a=256, max_len_b=256)
e1.record(); torch.cuda.synchronize()
print("sweep ms", e0.elapsed_time(e1) / 20)
