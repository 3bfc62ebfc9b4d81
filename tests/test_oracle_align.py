"""Pins for the oracle's edit distance (Fig.7) and Smith–Waterman (§6.1) functions.

Brute force over every (local) alignment for lengths <= 8, closed forms and
textbook special cases."""
import numpy as np
import pytest

import dpgen
from tests import brute

EN = dpgen.EN


def enc(s):
    return dpgen.encode(s, EN)


def test_edit_textbook(orc):
    # Levenshtein's textbook example (not in PAPER.md): kitten -> sitting = 3.
    assert orc.edit(enc("kitten"), enc("sitting")) == 3
    assert orc.edit(enc("flaw"), enc("lawn")) == 2


def test_edit_closed_forms(orc):
    g = np.random.default_rng(1)
    for _ in range(50):
        s = g.integers(0, 4, size=g.integers(0, 12)).astype(np.uint8)
        t = g.integers(0, 4, size=g.integers(0, 12)).astype(np.uint8)
        d = orc.edit(s, t)
        assert orc.edit(s, np.zeros(0, np.uint8)) == len(s)        # d(s, eps) = |s|
        assert orc.edit(np.zeros(0, np.uint8), t) == len(t)
        assert orc.edit(s, s) == 0
        assert d == orc.edit(t, s)                                 # symmetry
        assert abs(len(s) - len(t)) <= d <= max(len(s), len(t))
        u = g.integers(0, 4, size=g.integers(0, 8)).astype(np.uint8)
        assert d <= orc.edit(s, u) + orc.edit(u, t)                # triangle inequality


def test_edit_brute_force(orc):
    """d = the minimum over EVERY global alignment (lengths <= 8: up to D(8,8) = 265,729)."""
    g = np.random.default_rng(2)
    for k in range(60):
        n, m = (8, 8) if k < 4 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        s = g.integers(0, 3, size=n).astype(np.uint8)
        t = g.integers(0, 3, size=m).astype(np.uint8)
        assert orc.edit(s, t) == int(brute.global_alignment_costs(list(s), list(t)).min())
    for _ in range(10):   # the pure-Python enumerator agrees on small cases
        s = g.integers(0, 3, size=g.integers(0, 6)).astype(np.uint8)
        t = g.integers(0, 3, size=g.integers(0, 6)).astype(np.uint8)
        assert orc.edit(s, t) == brute.brute_edit(list(s), list(t))


def test_edit_traceback_canonical(orc):
    """Ops are an optimal alignment and the canonical one: the smallest reversed op
    sequence under diag < up(D) < left(I) among all optimal global alignments (lengths <= 8)."""
    g = np.random.default_rng(3)
    for k in range(50):
        n, m = (8, 8) if k < 3 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        s = list(g.integers(0, 3, size=n))
        t = list(g.integers(0, 3, size=m))
        ops = orc.edit_traceback(np.array(s, np.uint8), np.array(t, np.uint8))
        d = orc.edit(np.array(s, np.uint8), np.array(t, np.uint8))
        i = j = 0
        for o in ops:  # M/X labels agree with the residues
            if o in "MX":
                assert (o == "M") == (s[i] == t[j]); i += 1; j += 1
            elif o == "D":
                i += 1
            else:
                j += 1
        assert (i, j) == (n, m)
        want, _ = brute.canonical_local_traceback(s, t, (n, m), -d, lambda a, b: -int(a != b), 0, 1, whole=True)
        assert ops == want


def test_sw_brute_force_cells_and_end(orc):
    """Score and end cell equal the maximum over EVERY local alignment (lengths <= 8)."""
    g = np.random.default_rng(4)
    sig = dpgen.blosum62()
    sub = lambda a, b: int(sig[a][b])
    for k in range(40):
        n, m = (8, 8) if k < 4 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        alpha = 24 if k % 2 else 4    # small alphabets: recurring maxima, end-cell ties
        s = list(g.integers(0, alpha, size=n))
        t = list(g.integers(0, alpha, size=m))
        gap = int(g.integers(1, 6))
        _, best, (bi, bj) = brute.local_alignment_scores(s, t, sub, gap)
        sc, ei, ej = orc.sw(np.array(s, np.uint8), np.array(t, np.uint8), sig, gap)
        assert sc == best
        assert (ei, ej) == (bi, bj)
    for _ in range(5):   # the pure-Python enumerator agrees on small cases
        s = list(g.integers(0, 24, size=g.integers(0, 4)))
        t = list(g.integers(0, 24, size=g.integers(0, 4)))
        assert orc.sw(np.array(s, np.uint8), np.array(t, np.uint8), sig, 3)[0] == brute.brute_local_cells(s, t, sig, 3)[1]


def test_sw_traceback_canonical(orc):
    """The canonical local alignment (R-TB-SW): among every optimal local alignment ending at the
    end cell, the smallest reversed op sequence under diag < up < left with stopping first
    (lengths <= 8)."""
    g = np.random.default_rng(5)
    sig = dpgen.blosum62()
    sub = lambda a, b: int(sig[a][b])
    for k in range(60):
        n, m = (8, 8) if k < 4 else (int(g.integers(0, 9)), int(g.integers(0, 9)))
        s = list(g.integers(0, 6, size=n))
        t = list(g.integers(0, 6, size=m))
        gap = int(g.integers(1, 5))
        sc, ei, ej = orc.sw(np.array(s, np.uint8), np.array(t, np.uint8), sig, gap)
        ops, (si, sj, ei2, ej2) = orc.sw_traceback(np.array(s, np.uint8), np.array(t, np.uint8), sig, gap)
        assert (ei2, ej2) == ((ei, ej) if sc > 0 else (0, 0))
        if sc == 0:
            assert ops == ""
            continue
        assert brute.score_alignment(s[si:ei], t[sj:ej], ops.replace("M", "S").replace("X", "S"), sub, gap) == sc
        want, start = brute.canonical_local_traceback(s, t, (ei, ej), sc, sub, 0, gap)
        assert ops == want and (si, sj) == start


def test_sw_longest_common_substring(orc):
    """match=+1, mismatch=-inf-like, gap=inf-like reduces SW to longest common substring."""
    g = np.random.default_rng(6)
    sig = np.full((4, 4), -100, dtype=np.int8)
    np.fill_diagonal(sig, 1)
    for _ in range(40):
        s = g.integers(0, 4, size=g.integers(0, 14)).astype(np.uint8)
        t = g.integers(0, 4, size=g.integers(0, 14)).astype(np.uint8)
        lcs = 0
        for i in range(len(s)):
            for j in range(len(t)):
                k = 0
                while i + k < len(s) and j + k < len(t) and s[i + k] == t[j + k]:
                    k += 1
                lcs = max(lcs, k)
        assert orc.sw(s, t, sig, 100)[0] == lcs


def test_sw_bounds(orc):
    g = np.random.default_rng(7)
    sig = dpgen.blosum62()
    for _ in range(30):
        s = g.integers(0, 20, size=g.integers(1, 40)).astype(np.uint8)
        t = g.integers(0, 20, size=g.integers(1, 40)).astype(np.uint8)
        sc = orc.sw(s, t, sig, 4)[0]
        assert sc >= max(0, max(int(sig[a][b]) for a in s for b in t))
        assert sc <= 11 * min(len(s), len(t))
        assert sc == orc.sw(t, s, sig.T.copy(), 4)[0]  # transposition symmetry
        assert orc.sw(s, s, sig, 4)[0] == int(sum(int(sig[a][a]) for a in s))  # identity: diagonal is optimal
