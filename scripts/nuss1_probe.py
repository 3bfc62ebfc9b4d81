"""Config-1 latency probe: kernel time of the Nussinov paths for one 64-nt RNA (with and without
the traceback), CUDA events over 200 back-to-back solves."""
import os
import sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dpgen
import paper_conf_pldi_carteylm12_b200 as dp

x = dpgen.config1_rna64()
cat, off = dpgen.pack([x])
c, o = torch.from_numpy(cat).cuda(), torch.from_numpy(off).cuda()
for env in ({}, {"DP_NUSS_CELL": "1"}, {"DP_NUSS_TILED_MIN": "31"}):
    for tb in (False, True):
        os.environ.pop("DP_NUSS_CELL", None)
        os.environ.pop("DP_NUSS_TILED_MIN", None)
        os.environ.update(env)
        with dp.Plan(dp.NUSSINOV, 64, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=tb) as p:
            out = torch.empty(1, dtype=torch.int32, device="cuda")
            for _ in range(20):
                p.solve_batch(c, o, max_len_a=64, out=out)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(200):
                p.solve_batch(c, o, max_len_a=64, out=out)
            e1.record()
            torch.cuda.synchronize()
            print(env, "tb" if tb else "score", f"{e0.elapsed_time(e1) / 200 * 1000:.1f} us per solve", int(out[0]))
