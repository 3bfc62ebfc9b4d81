"""Pins for the oracle's Nussinov interval DP (textbook, ref [3] of PAPER.md L598).

Brute force over every secondary structure for n <= 12, closed cases and
invariants; the canonical traceback (DESIGN.md R-TB-NUSS) against
hand-derived goldens that separate each rule order and against its definition over
the enumerated structures."""
import numpy as np
import pytest

import dpgen
from tests import brute

PM = dpgen.rna_pair_mask()
PM_WC = dpgen.rna_pair_mask(gu=False)


def enc(s):
    return dpgen.encode(s, dpgen.RNA)


@pytest.mark.parametrize("h", [0, 1, 3])
def test_nussinov_brute_force(orc, h):
    g = np.random.default_rng(10 + h)
    for _ in range(40):
        n = int(g.integers(0, 13))
        x = g.integers(0, 4, size=n).astype(np.uint8)
        for pm in (PM, PM_WC):
            want, _ = brute.brute_nussinov(list(x), pm, h) if n else (0, 1)
            assert orc.nussinov(x, pm, h) == want


def test_nussinov_closed_cases(orc):
    assert orc.nussinov(enc("GGGGAAAACCCC"), PM, 3) == 4
    assert orc.nussinov_traceback(enc("GGGGAAAACCCC"), PM, 3) == (4, "((((....))))")
    assert orc.nussinov(enc("A" * 40), PM, 3) == 0             # poly-A: nothing pairs
    assert orc.nussinov(enc(""), PM, 3) == 0                   # n <= 1 -> 0
    assert orc.nussinov(enc("G"), PM, 3) == 0
    assert orc.nussinov(enc("GC"), PM, 0) == 1                 # h = 0: adjacent pair allowed
    assert orc.nussinov(enc("GC"), PM, 1) == 0
    assert orc.nussinov(enc("GAAAC"), PM, 3) == 1 and orc.nussinov(enc("GAAC"), PM, 3) == 0
    # (AU)^k with h = 0 pairs everything: k pairs
    assert orc.nussinov(enc("AU" * 10), PM, 0) == 10


def test_nussinov_invariants(orc):
    g = np.random.default_rng(11)
    for _ in range(60):
        n = int(g.integers(2, 60))
        x = g.integers(0, 4, size=n).astype(np.uint8)
        v = orc.nussinov(x, PM, 3)
        assert v == orc.nussinov(x[::-1].copy(), PM, 3)         # reversal (symmetric pair set)
        assert 0 <= v <= max(0, (n - 3) // 2)                   # each pair uses 2 bases, hairpins
        assert orc.nussinov(x, PM, 0) >= v >= orc.nussinov(x, PM, 5)   # monotone in h
        assert orc.nussinov(x, PM, 3) >= orc.nussinov(x, PM_WC, 3)     # more pairs allowed


def test_nussinov_traceback_valid_and_optimal(orc):
    g = np.random.default_rng(12)
    for _ in range(80):
        n = int(g.integers(0, 40))
        h = int(g.integers(0, 4))
        x = g.integers(0, 4, size=n).astype(np.uint8)
        sc, db = orc.nussinov_traceback(x, PM, h)
        assert sc == orc.nussinov(x, PM, h)
        pairs = brute.dotbracket_pairs(db)
        assert len(pairs) == sc
        for i, j in pairs:
            assert PM[x[i]][x[j]] and j - i - 1 >= h


def test_nussinov_traceback_canonical_small(orc):
    """Durbin order: i unpaired before j unpaired before pairing before splits (smallest k)."""
    # "GC" h=0 -> pair; "GCGC" h=0: gamma(1,3)=1 first -> i=0 unpaired, then (1,3)... -> ".(.)"? check by rule:
    # gamma(0,3)=2 > gamma(1,3)=1, gamma(0,2)=1 -> pair(0,3) G-C: gamma(1,2)+1 = 1+1 = 2 -> '(' at 0, ')' at 3,
    # then (1,2) C-G pairs -> "(())".
    assert orc.nussinov_traceback(enc("GCGC"), PM, 0) == (2, "(())")
    # "GCAGC" h=0: gamma(0,4)=2; gamma(1,4)= C A G C -> CG at (1,3)=1 ... =1 < 2; gamma(0,3)=GCAG: (0,1)+... =1 <2;
    # pair(0,4) G-C: gamma(1,3)+1 = 2 -> "(" 0 ")" 4, then (1,3) C..G: pair -> "((.))"
    assert orc.nussinov_traceback(enc("GCAGC"), PM, 0) == (2, "((.))")


# ----------------------------------------------------------------------------- canonical traceback (R-TB-NUSS)
# Hand-derived goldens, one per ordering decision of the Durbin-order reading (DESIGN.md R-TB-NUSS:
# (1) i unpaired, (2) j unpaired, (3) pair (i, j), (4) smallest split k). gamma(a, b) below is the
# maximum number of pairs on x[a..b]; pairs AU/UA/GC/CG/GU/UG.
TB_GOLDENS = [
    # (1) before (3): "AAU", h = 0. Pairable: (0,2) A-U, (1,2) A-U; gamma(0,2) = 1.
    #   (1) gamma(1,2) = 1 (A-U) = gamma(0,2) -> 0 unpaired, recurse on (1,2);
    #   on (1,2): (1) gamma(2,2) = 0, (2) gamma(1,1) = 0, (3) A-U with 2-1-1 = 0 >= h -> pair.
    #   Canonical ".()"; a pair-first rule would give "(.)".
    ("AAU", 0, 1, ".()", {"pair_first": "(.)"}),
    # (1) before (2): "AUA", h = 0. gamma(0,2) = 1. (1) gamma(1,2) = 1 (U-A) -> 0 unpaired, then (1,2)
    #   pairs -> ".()"; a j-first rule takes gamma(0,1) = 1 (A-U) -> 2 unpaired -> "().".
    ("AUA", 0, 1, ".()", {"j_first": "()."}),
    # (2) before (3): "GCC", h = 0. Pairable (0,1), (0,2) (G-C); gamma(0,2) = 1.
    #   (1) gamma(1,2) = 0 (C-C) fails; (2) gamma(0,1) = 1 -> 2 unpaired, then (0,1) pairs -> "().";
    #   a pair-first rule would pair (0,2) -> "(.)".
    ("GCC", 0, 1, "().", {"pair_first": "(.)"}),
    # smallest k in (4): "AUAUCG", h = 0, gamma(0,5) = 3 (e.g. (0,1) (2,3) (4,5)).
    #   (1) gamma(1,5) = 2 (UAUCG: (1,2) (4,5)); (2) gamma(0,4) = 2 (AUAUC); (3) A-G cannot pair;
    #   (4) k = 1: gamma(0,1) + gamma(2,5) = 1 + 2 = 3 (k = 2: 1 + 1, k = 3: 2 + 1 = 3, k = 4: 2 + 0),
    #   so the candidates are k in {1, 3}; the smallest is 1: (0,1) -> "()"; (2,5) "AUCG":
    #   (1) gamma(3,5) = 1, (2) gamma(2,4) = 1, (3) A-G no, (4) k = 3: 1 + 1 = 2 -> "()()".
    #   Canonical "()()()"; the largest k (3) gives (0,3) = "(())" (AUAU: (1), (2) fail, (3) A-U
    #   pairs around gamma(1,2) = 1) + "()" = "(())()".
    ("AUAUCG", 0, 3, "()()()", {"largest_k": "(())()"}),
    # hairpin h = 3 with a split: "GAAACGAAAC". Pairable with loops >= 3: (0,4) G-C and (5,9) G-C
    #   (4 - 0 - 1 = 3), and (0,9) G-C; gamma(0,9) = 2 with (0,4) (5,9).
    #   (1) gamma(1,9) = 1 ("AAACGAAAC": (5,9) only), (2) gamma(0,8) = 1, (3) pair (0,9) gives
    #   gamma(1,8) + 1 = 0 + 1 (C4-G5 are adjacent) = 1 < 2; (4) k = 4: gamma(0,4) + gamma(5,9) = 2
    #   (k = 1..3: 0 + 1, k = 5..8: 1 + 0) -> "(...)" + "(...)".
    ("GAAACGAAAC", 3, 2, "(...)(...)", {}),
]


@pytest.mark.parametrize("seq,h,score,db,variants", TB_GOLDENS)
def test_nussinov_traceback_goldens(orc, seq, h, score, db, variants):
    x = enc(seq)
    assert orc.nussinov_traceback(x, PM, h) == (score, db)
    assert brute.canonical_structure(list(x), PM, h) == db          # the enumeration-level definition
    for var, other in variants.items():                              # the golden separates the readings
        assert brute.canonical_structure(list(x), PM, h, variant=var) == other != db


def test_nussinov_traceback_canonical_bruteforce(orc):
    """Oracle traceback == the canonical structure defined over the enumeration of all secondary
    structures (tests/brute.canonical_structure), n <= 12, h in 0..3, both pair sets."""
    g = np.random.default_rng(13)
    differ = {"pair_first": 0, "j_first": 0, "largest_k": 0}
    for _ in range(160):
        n = int(g.integers(0, 13))
        h = int(g.integers(0, 4))
        pm = PM if g.random() < 0.7 else PM_WC
        x = g.integers(0, 4, size=n).astype(np.uint8)
        sc, db = orc.nussinov_traceback(x, pm, h)
        assert db == brute.canonical_structure(list(x), pm, h), (dpgen.decode(x, dpgen.RNA), h)
        for var in differ:
            differ[var] += brute.canonical_structure(list(x), pm, h, variant=var) != db
    # every alternative reading disagrees on some of these inputs, so this check can tell them apart
    assert all(v > 0 for v in differ.values()), differ
