"""Pins for the oracle's affine-gap Smith–Waterman (SURVEY.md §8(f) NEXT rank 1,
Gotoh; DESIGN.md R-SW-AFFINE / R-TB-SWA).

* brute force: max over every local alignment scored with gap(k) = go + k*ge;
* special case go = 0: a gap of length k costs k*ge, i.e. linear SW with g = ge;
* special case go -> large: only gap-free local alignments (best diagonal run);
* the traceback spells a local alignment whose affine score is the optimum and
  whose coordinates match the ops."""
import numpy as np

import dpgen
from tests import brute


def _affine_score(s, t, ops, co, sigma, go, ge):
    i0, j0, i1, j1 = co
    return brute.score_alignment_affine(s[i0:i1], t[j0:j1], ops, lambda a, b: int(sigma[a][b]), go, ge)


def test_affine_brute_force_random(orc):
    g = np.random.default_rng(31)
    for trial in range(60):
        asz = int(g.integers(2, 5))
        sig = g.integers(-4, 6, size=(asz, asz)).astype(np.int8)
        go, ge = int(g.integers(0, 6)), int(g.integers(1, 4))
        s = g.integers(0, asz, size=g.integers(0, 5)).astype(np.uint8)
        t = g.integers(0, asz, size=g.integers(0, 5)).astype(np.uint8)
        sc, _, _ = orc.sw_affine(s, t, sig, go, ge)
        assert sc == brute.brute_local_affine(list(s), list(t), sig, go, ge), (trial, s, t, go, ge)


def test_affine_brute_force_blosum(orc):
    g = np.random.default_rng(32)
    sig = dpgen.blosum62()
    for trial in range(25):
        s = g.integers(0, 20, size=g.integers(1, 6)).astype(np.uint8)
        t = g.integers(0, 20, size=g.integers(1, 6)).astype(np.uint8)
        for go, ge in ((11, 1), (2, 1), (0, 4)):
            sc, _, _ = orc.sw_affine(s, t, sig, go, ge)
            assert sc == brute.brute_local_affine(list(s), list(t), sig, go, ge)


def test_affine_reduces_to_linear(orc):
    # go = 0: gap(k) = k*ge = linear gap ge
    g = np.random.default_rng(33)
    sig = dpgen.blosum62()
    for _ in range(40):
        s = g.integers(0, 20, size=g.integers(0, 40)).astype(np.uint8)
        t = g.integers(0, 20, size=g.integers(0, 40)).astype(np.uint8)
        ge = int(g.integers(1, 8))
        assert orc.sw_affine(s, t, sig, 0, ge)[0] == orc.sw(s, t, sig, ge)[0]


def test_affine_gap_free_limit(orc):
    # a prohibitive open cost leaves only gap-free alignments: the best diagonal segment
    g = np.random.default_rng(34)
    sig = dpgen.blosum62()
    for _ in range(30):
        s = g.integers(0, 20, size=g.integers(1, 25)).astype(np.uint8)
        t = g.integers(0, 20, size=g.integers(1, 25)).astype(np.uint8)
        best = 0
        for d in range(-len(s) + 1, len(t)):
            run = 0
            for i in range(len(s)):
                j = i + d
                if 0 <= j < len(t):
                    run = max(0, run + int(sig[s[i]][t[j]]))
                    best = max(best, run)
        assert orc.sw_affine(s, t, sig, 10_000, 1)[0] == best


def test_affine_traceback_is_optimal(orc):
    g = np.random.default_rng(35)
    sig = dpgen.blosum62()
    for _ in range(60):
        s = g.integers(0, 20, size=g.integers(0, 60)).astype(np.uint8)
        t = g.integers(0, 20, size=g.integers(0, 60)).astype(np.uint8)
        go, ge = int(g.integers(0, 12)), int(g.integers(1, 3))
        sc, ei, ej = orc.sw_affine(s, t, sig, go, ge)
        ops, co = orc.sw_affine_traceback(s, t, sig, go, ge)
        if sc == 0:
            assert ops == "" and co == (0, 0, 0, 0)
            continue
        assert (co[2], co[3]) == (ei, ej)
        assert co[2] - co[0] == sum(o in "MXD" for o in ops)
        assert co[3] - co[1] == sum(o in "MXI" for o in ops)
        assert all((o == "M") == (s[i] == t[j]) for o, i, j in _walk(ops, co))
        assert _affine_score(list(s), list(t), ops, co, sig, go, ge) == sc


def _walk(ops, co):
    i, j = co[0], co[1]
    for o in ops:
        if o in "MX":
            yield o, i, j
            i += 1; j += 1
        elif o == "D":
            i += 1
        else:
            j += 1


def test_affine_identical_sequences(orc):
    # BLOSUM62's diagonal is positive: aligning a sequence with itself scores the diagonal sum
    g = np.random.default_rng(36)
    sig = dpgen.blosum62()
    for _ in range(10):
        s = g.integers(0, 20, size=g.integers(1, 80)).astype(np.uint8)
        assert orc.sw_affine(s, s, sig, 11, 1)[0] == int(sum(int(sig[c][c]) for c in s))
