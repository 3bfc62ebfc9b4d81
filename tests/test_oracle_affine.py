"""Pins for the oracle's affine-gap Smith–Waterman (SURVEY.md §8(f) NEXT rank 1,
Gotoh; DESIGN.md R-SW-AFFINE / R-TB-SWA).

* brute force: max over every local alignment scored with gap(k) = go + k*ge;
* special case go = 0: a gap of length k costs k*ge, i.e. linear SW with g = ge;
* special case go -> large: only gap-free local alignments (best diagonal run);
* the traceback spells a local alignment whose affine score is the optimum and
  whose coordinates match the ops."""
import numpy as np
import pytest

import dpgen
from tests import brute


def _affine_score(s, t, ops, co, sigma, go, ge):
    i0, j0, i1, j1 = co
    return brute.score_alignment_affine(s[i0:i1], t[j0:j1], ops, lambda a, b: int(sigma[a][b]), go, ge)


def test_affine_brute_force_random(orc):
    """Score and end cell = the maximum over EVERY local alignment, lengths <= 8."""
    g = np.random.default_rng(31)
    for trial in range(60):
        asz = int(g.integers(2, 5))
        sig = g.integers(-4, 6, size=(asz, asz)).astype(np.int8)
        go, ge = int(g.integers(0, 6)), int(g.integers(1, 4))
        n, m = (8, 8) if trial < 4 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        s = g.integers(0, asz, size=n).astype(np.uint8)
        t = g.integers(0, asz, size=m).astype(np.uint8)
        sc, ei, ej = orc.sw_affine(s, t, sig, go, ge)
        best, end = brute.local_affine_best(list(s), list(t), lambda a, b: int(sig[a][b]), go, ge)
        assert (sc, (ei, ej)) == (best, end), (trial, s, t, go, ge)
        if trial < 15 and n <= 4 and m <= 4:   # the pure-Python enumerator agrees
            assert sc == brute.brute_local_affine(list(s), list(t), sig, go, ge)


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


# ----------------------------------------------------------------------------- canonical traceback (R-TB-SWA)
def _extend_first(prev, op):
    """Alternative reading: extend an open gap before closing it."""
    if prev == "D":
        return {"D": 0, "S": 1, "I": 2}[op]
    if prev == "I":
        return {"I": 0, "S": 1, "D": 2}[op]
    return {"S": 0, "D": 1, "I": 2}[op]


def _i_before_d(prev, op):
    """Alternative reading: in H prefer E (I) over F (D)."""
    if prev == "D":
        return {"S": 0, "I": 1, "D": 2}[op]
    return {"S": 0, "I": 1, "D": 2}[op]


def _golden_sigma(pairs, asz=5, other=-20):
    sig = np.full((asz, asz), other, dtype=np.int8)
    for (a, b), v in pairs.items():
        sig[a][b] = v
    return sig


# Hand-derived goldens, one per decision of R-TB-SWA that the other pins cannot see.
#  (a) gap open before extend. Codes A=0 w=1 x=2 y=3 z=4; sigma(A,A) = 5, sigma(x,z) = 3,
#      sigma(w,z) = 4, all else -3; go = ge = 1; s = w x y A, t = z A.
#      Local alignments scoring 6: x/z, y/-, A/A (3 - 2 + 5) and w/z, x/-, y/-, A/A (4 - 3 + 5);
#      A/A alone is 5. End cell (4,2) (A/A). H(3,1) = F(3,1) = max(F(2,1) - 1, H(2,1) - 2) with
#      H(2,1) = 3 (x/z) and F(2,1) = H(1,1) - 2 = 2: both give 1 -> the gap opens at row 3 ->
#      H(2,1) -> diagonal x/z -> H(1,0) = 0 stop: "XDM" from (1,0); extend-first -> "XDDM".
#  (b) F before E in H. Codes A=0 p=1 q=2 r=3 s=4; sigma(A,A) = sigma(p,r) = 10, all else -20;
#      go = ge = 1; s = p q A, t = r s A. Best 16 = p/r + a D and an I gap (-2 each) + A/A; end (3,3),
#      H(2,2) = 6 = F(2,2) (from H(1,2) = 8 - 2) = E(2,2) (from H(2,1) = 8 - 2), the diagonal
#      q/s = -20 is out: F first -> D, opened at H(1,2) = E(1,2) -> I, opened at H(1,1) -> X (p/r):
#      "XIDM" from (0,0); I-before-D -> "XDIM".
AFFINE_GOLDENS = [
    ([1, 2, 3, 0], [4, 0], _golden_sigma({(0, 0): 5, (2, 4): 3, (1, 4): 4}, other=-3), 1, 1,
     6, "XDM", (1, 0, 4, 2), {"extend_first": "XDDM"}),
    ([1, 2, 0], [3, 4, 0], _golden_sigma({(0, 0): 10, (1, 3): 10}), 1, 1,
     16, "XIDM", (0, 0, 3, 3), {"i_before_d": "XDIM"}),
]


@pytest.mark.parametrize("s,t,sig,go,ge,score,ops,co,variants", AFFINE_GOLDENS)
def test_affine_traceback_goldens(orc, s, t, sig, go, ge, score, ops, co, variants):
    sa, ta = np.array(s, np.uint8), np.array(t, np.uint8)
    assert orc.sw_affine(sa, ta, sig, go, ge)[0] == score
    assert orc.sw_affine_traceback(sa, ta, sig, go, ge) == (ops, co)
    sub = lambda a, b: int(sig[a][b])
    end = (co[2], co[3])
    assert brute.canonical_local_traceback(s, t, end, score, sub, go, ge, rank=brute.rank_affine(go),
                                           affine=True) == (ops, (co[0], co[1]))
    ranks = {"extend_first": _extend_first, "i_before_d": _i_before_d}
    for var, other in variants.items():
        got, _ = brute.canonical_local_traceback(s, t, end, score, sub, go, ge, rank=ranks[var], affine=True)
        assert got == other != ops


def test_affine_traceback_canonical_bruteforce(orc):
    """Oracle traceback == the smallest reversed op sequence, under R-TB-SWA's context order
    (tests/brute.rank_affine), among EVERY optimal local alignment ending at the end cell
    (lengths <= 8, small alphabets and scores so that ties are common)."""
    g = np.random.default_rng(37)
    for trial in range(120):
        asz = int(g.integers(2, 5))
        sig = g.integers(-3, 5, size=(asz, asz)).astype(np.int8)
        go, ge = int(g.integers(0, 4)), int(g.integers(1, 3))
        n, m = (8, 8) if trial < 4 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        s = list(g.integers(0, asz, size=n))
        t = list(g.integers(0, asz, size=m))
        sa, ta = np.array(s, np.uint8), np.array(t, np.uint8)
        sc, ei, ej = orc.sw_affine(sa, ta, sig, go, ge)
        ops, co = orc.sw_affine_traceback(sa, ta, sig, go, ge)
        if sc == 0:
            assert ops == "" and co == (0, 0, 0, 0)
            continue
        want, start = brute.canonical_local_traceback(s, t, (ei, ej), sc, lambda a, b: int(sig[a][b]), go, ge,
                                                      rank=brute.rank_affine(go), affine=True)
        assert (ops, (co[0], co[1])) == (want, start), (trial, s, t, go, ge)
