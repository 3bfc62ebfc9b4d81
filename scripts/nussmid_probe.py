"""NEXT 4 probe: a few mid-length Nussinov problems on the cluster kernel vs the batch / grid
kernels (DP_NUSS_NO_CLUSTER=1), CUDA events over back-to-back solves with traceback."""
import os
import sys
import numpy as np
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dpgen
import paper_conf_pldi_carteylm12_b200 as dp

g = np.random.default_rng(5)
for name, lens in (("1x1000", [1000]), ("9x1000", [1000] * 9), ("18xU[512,1024]", list(g.integers(512, 1025, 18))),
                   ("36x512", [512] * 36)):
    seqs = [g.integers(0, 4, size=int(l)).astype(np.uint8) for l in lens]
    cat, off = dpgen.pack(seqs)
    c, o = torch.from_numpy(cat).cuda(), torch.from_numpy(off).cuda()
    ml = max(lens)
    res = {}
    for env in ({}, {"DP_NUSS_NO_CLUSTER": "1"}):
        os.environ.pop("DP_NUSS_NO_CLUSTER", None)
        os.environ.update(env)
        with dp.Plan(dp.NUSSINOV, ml, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
            out = torch.empty(len(lens), dtype=torch.int32, device="cuda")
            for _ in range(2):
                p.solve_batch(c, o, max_len_a=ml, out=out)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(5):
                p.solve_batch(c, o, max_len_a=ml, out=out)
            e1.record()
            torch.cuda.synchronize()
            res["cluster" if not env else "batch"] = (e0.elapsed_time(e1) / 5, out.cpu().numpy().copy())
    cells = sum(l * (l - 1) // 2 for l in lens)
    same = (res["cluster"][1] == res["batch"][1]).all()
    print(f"{name}: cluster {res['cluster'][0]:.3f} ms ({cells / res['cluster'][0] / 1e6:.2f} GCUPS), "
          f"no-cluster {res['batch'][0]:.3f} ms, scores equal {same}", flush=True)
