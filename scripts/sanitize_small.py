"""Small invocations of every kernel family for compute-sanitizer (memcheck / racecheck / synccheck):
SURVEY §5 "race detection" — the runtime counterpart of eq.(2) (cells of one partition are
independent, L318-L322) and Fig.8's `sync` (L251-L253). Sizes are tiny (racecheck is ~100x slower)
but span several tiles, strips, warps and the ragged tails."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import dpgen  # noqa: E402
import paper_conf_pldi_carteylm12_b200 as dp  # noqa: E402


def cu(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def main(which):
    g = np.random.default_rng(3)
    sig = dpgen.blosum62()
    if which in ("all", "align"):
        a = [g.integers(0, 20, int(l)).astype(np.uint8) for l in g.integers(1, 300, 12)]
        b = [g.integers(0, 20, int(l)).astype(np.uint8) for l in g.integers(1, 300, 12)]
        (ac, ao), (bc, bo) = dpgen.pack(a), dpgen.pack(b)
        la, lb = max(map(len, a)), max(map(len, b))
        for kind, kw in ((dp.SW_LINEAR, dict(gap=4)), (dp.SW_AFFINE, dict(gap_open=11, gap_extend=1)),
                         (dp.EDIT, dict(alphabet_size=24))):
            with dp.Plan(kind, la, lb, sigma=None if kind == dp.EDIT else sig, want_traceback=True, **kw) as p:
                sc = p.solve_batch(cu(ac), cu(ao), cu(bc), cu(bo), max_len_a=la, max_len_b=lb)  # kept: the
                p.traceback(0, len(a), la + lb + 1)                                           # traceback reads it
                del sc
        with dp.Plan(dp.DIAG_LCS, la, lb, alphabet_size=4) as p:
            a4 = [x % 4 for x in a]
            b4 = [x % 4 for x in b]
            (ac, ao), (bc, bo) = dpgen.pack(a4), dpgen.pack(b4)
            p.solve_batch(cu(ac), cu(ao), cu(bc), cu(bo), max_len_a=la, max_len_b=lb)
    if which in ("all", "inter"):   # short pairs: the inter-task kernel (one pair per thread)
        a = [g.integers(0, 20, int(l)).astype(np.uint8) for l in g.integers(0, 65, 300)]
        b = [g.integers(0, 20, int(l)).astype(np.uint8) for l in g.integers(0, 65, 300)]
        (ac, ao), (bc, bo) = dpgen.pack(a), dpgen.pack(b)
        with dp.Plan(dp.SW_LINEAR, 64, 64, sigma=sig, gap=4, want_traceback=True) as p:
            sc = p.solve_batch(cu(ac), cu(ao), cu(bc), cu(bo), max_len_a=64, max_len_b=64)
            p.traceback(0, len(a), 129)
            del sc
    if which in ("all", "nuss"):
        for lens in ((1, 20, 64, 100, 128),                        # k_nuss_small (a few problems <= 128 nt)
                     tuple(int(l) for l in g.integers(0, 200, 70))):  # k_nuss_batch (more than 64 problems)
            seqs = [g.integers(0, 4, int(l)).astype(np.uint8) for l in lens]
            c, o = dpgen.pack(seqs)
            ml = max(lens)
            with dp.Plan(dp.NUSSINOV, ml, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
                p.solve_batch(cu(c), cu(o), max_len_a=ml)
                p.traceback(0, len(seqs), ml, coords=False)
        # k_nuss_cluster (a few problems of 129..1024 nt)
        seqs = [g.integers(0, 4, int(l)).astype(np.uint8) for l in (1, 20, 33, 64, 100, 130, 200)]
        c, o = dpgen.pack(seqs)
        with dp.Plan(dp.NUSSINOV, 200, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
            p.solve_batch(cu(c), cu(o), max_len_a=200)
            p.traceback(0, len(seqs), 200, coords=False)
        x = g.integers(0, 4, 1100).astype(np.uint8)   # the grid-wide sweep (n > 1024)
        c, o = dpgen.pack([x])
        with dp.Plan(dp.NUSSINOV, 1100, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
            p.solve_batch(cu(c), cu(o), max_len_a=1100)
            p.traceback(0, 1, 1100, coords=False)
    if which in ("all", "hmm"):
        pi, A, E = (v.astype(np.float32) for v in dpgen.hmm_params(g, 64, 4))
        seqs = [dpgen.sample_hmm(g, pi, A, E, 1, int(t))[0] for t in (0, 1, 50, 300)] * 40
        c, o = dpgen.pack(seqs)
        with dp.Plan(dp.HMM_FORWARD, 300, pi=pi, A=A, E=E) as p:
            p.solve_batch(cu(c), cu(o), max_len_a=300)
        with dp.Plan(dp.HMM_VITERBI, 300, lpi=dpgen.millibits(pi), lA=dpgen.millibits(A), lE=dpgen.millibits(E),
                     want_traceback=True) as p:
            p.solve_batch(cu(c), cu(o), max_len_a=300)
            p.traceback(0, len(seqs), 300, coords=False)
        tr, eM, eI = (v.astype(np.float32) for v in dpgen.profile_hmm_params(g, 300, 20))
        seqs = [g.integers(0, 20, int(l)).astype(np.uint8) for l in (0, 1, 40, 310)]
        c, o = dpgen.pack(seqs)
        with dp.Plan(dp.PROFILE_FORWARD, 310, trans=tr, emit_m=eM, emit_i=eI) as p:
            p.solve_batch(cu(c), cu(o), max_len_a=310)
    torch.cuda.synchronize()
    print("ok", which)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "all")
