# Probe: Nussinov fill with and without the in-kernel traceback (timing only).
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import dpgen
import paper_conf_pldi_carteylm12_b200 as dp
for which in sys.argv[1:]:
    if which == "nuss4":
        cat, off = dpgen.pack([dpgen.config4_rna8192()])
    else:
        cat, off = dpgen.config5_rna_batch(int(which))
    ml = int(np.diff(off).max())
    a, o = torch.from_numpy(cat).cuda(), torch.from_numpy(off).cuda()
    for tb in (False, True):
        p = dp.Plan(dp.NUSSINOV, ml, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=tb)
        p.solve_batch(a, o, max_len_a=ml); torch.cuda.synchronize()
        t = time.time(); p.solve_batch(a, o, max_len_a=ml); torch.cuda.synchronize()
        print(f"{which} traceback={tb}: {1e3*(time.time()-t):.1f} ms", flush=True)
