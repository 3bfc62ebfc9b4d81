"""Small packed-SW traceback repro (multi-strip lengths) for compute-sanitizer runs."""
import sys
import numpy as np
import torch
import dpgen
import paper_conf_pldi_carteylm12_b200 as dp

n, L = int(sys.argv[1]) if len(sys.argv) > 1 else 4, int(sys.argv[2]) if len(sys.argv) > 2 else 300
g = np.random.default_rng(5)
a = [g.integers(0, 24, size=L).astype(np.uint8) for _ in range(n)]
b = [g.integers(0, 24, size=L).astype(np.uint8) for _ in range(n)]
ac, ao = dpgen.pack(a); bc, bo = dpgen.pack(b)
cu = lambda x: torch.from_numpy(np.ascontiguousarray(x)).cuda()
with dp.Plan(dp.SW_LINEAR, L, L, sigma=dpgen.blosum62(), gap=4, alphabet_size=24, want_traceback=True) as p:
    sc = p.solve_batch(cu(ac), cu(ao), cu(bc), cu(bo), max_len_a=L, max_len_b=L)
    torch.cuda.synchronize(); print("solve ok", p.last_variant, sc.cpu().numpy()[:4])
    out, ln, co = p.traceback(0, n, 2 * L + 1)
    torch.cuda.synchronize(); print("tb ok", ln.cpu().numpy()[:4])
