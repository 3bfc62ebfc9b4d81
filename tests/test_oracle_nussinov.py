"""Pins for the oracle's Nussinov interval DP (textbook, ref [3] of PAPER.md L598).

Brute force over every secondary structure for n <= 12, closed cases and
invariants."""
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
        n = int(g.integers(0, 12 if h else 10))
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
