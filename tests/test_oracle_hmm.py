"""Pins for the oracle's HMM forward (Fig.11a) and Viterbi (max-variant, L463-L464).

Brute force over all S^T state paths, normalisation, closed forms
(SURVEY.md §8(c) C5, C6)."""
import itertools
import math

import numpy as np
import pytest

import dpgen
from tests import brute


def rand_hmm(g, S, K):
    return dpgen.hmm_params(g, S, K)


def test_forward_brute_force(orc):
    """log P(x) = log of the sum over EVERY state path (S <= 8, T <= 6: up to 262,144 paths)."""
    g = np.random.default_rng(20)
    for k in range(30):
        S, K, T = (8, 4, 6) if k < 3 else (int(g.integers(1, 7)), int(g.integers(2, 5)), int(g.integers(0, 7)))
        pi, A, E = rand_hmm(g, S, K)
        x = g.integers(0, K, size=T).astype(np.uint8)
        want = brute.brute_forward_np(list(x), pi, A, E)
        got = orc.forward(x, pi, A, E)
        assert abs(got - want) <= 1e-12 * max(1.0, abs(want))
        if S <= 3 and T <= 4:   # the pure-Python enumerator agrees
            assert abs(brute.brute_forward(list(x), pi, A, E) - want) <= 1e-12 * max(1.0, abs(want))


def test_forward_sums_to_one(orc):
    """sum over all x in Sigma^T of P(x) = 1 for stochastic pi, A, E."""
    g = np.random.default_rng(21)
    S, K, T = 3, 4, 5
    pi, A, E = rand_hmm(g, S, K)
    tot = 0.0
    for x in itertools.product(range(K), repeat=T):
        tot += math.exp(orc.forward(np.array(x, np.uint8), pi, A, E))
    assert abs(tot - 1.0) < 1e-12


def test_forward_closed_forms(orc):
    g = np.random.default_rng(22)
    # uniform emissions => log P(x) = -T log K, whatever pi and A are
    S, K, T = 7, 4, 300
    pi, A, _ = rand_hmm(g, S, K)
    E = np.full((S, K), 1.0 / K)
    x = g.integers(0, K, size=T).astype(np.uint8)
    assert abs(orc.forward(x, pi, A, E) - (-T * math.log(K))) < 1e-9
    # S = 1 => prod e(x_t)
    E1 = g.dirichlet(np.ones(K))[None, :]
    x = g.integers(0, K, size=50).astype(np.uint8)
    assert abs(orc.forward(x, np.ones(1), np.ones((1, 1)), E1) - float(np.sum(np.log(E1[0][x])))) < 1e-9
    # T = 1 => log sum_s pi_s e_s(x_1)
    pi, A, E = rand_hmm(g, 5, 3)
    assert abs(orc.forward(np.array([2], np.uint8), pi, A, E) - math.log(float(np.dot(pi, E[:, 2])))) < 1e-12
    # T = 0 => 0 (log 1)
    assert orc.forward(np.zeros(0, np.uint8), pi, A, E) == 0.0


def test_viterbi_brute_force_and_canonical_path(orc):
    """Score = max over all paths; path = the optimal path whose reversal is
    lexicographically smallest (final state lowest, then predecessors lowest)."""
    g = np.random.default_rng(23)
    for k in range(40):
        S, K, T = (8, 3, 6) if k < 3 else (int(g.integers(1, 7)), int(g.integers(2, 4)), int(g.integers(1, 7)))
        pi, A, E = rand_hmm(g, S, K)
        # coarse scores so that ties actually occur
        lpi, lA, lE = (np.rint(dpgen.millibits(v) / 997.0).astype(np.int32) for v in (pi, A, E))
        x = g.integers(0, K, size=T).astype(np.uint8)
        best, canon = brute.brute_viterbi_np(list(x), lpi, lA, lE)
        sc, path = orc.viterbi(x, lpi, lA, lE)
        assert sc == best
        assert brute.viterbi_path_score(list(x), list(path), lpi, lA, lE) == best
        assert tuple(int(v) for v in path) == canon
        if S <= 3 and T <= 4:   # the pure-Python enumerator agrees
            b2, paths = brute.brute_viterbi(list(x), lpi, lA, lE)
            assert b2 == best and min(paths, key=lambda p: tuple(reversed(p))) == canon


def test_viterbi_closed_forms(orc):
    g = np.random.default_rng(24)
    # all-equal scores: every path ties -> all zeros
    S, K, T = 5, 4, 20
    z = np.zeros(S, np.int32)
    sc, path = orc.viterbi(g.integers(0, K, size=T).astype(np.uint8), z, np.zeros((S, S), np.int32), np.zeros((S, K), np.int32))
    assert sc == 0 and not path.any()
    # identity-like A (huge self-loop cost 0, others very negative) and per-step argmax of emissions
    lA = np.full((S, S), -10**6, np.int32)
    np.fill_diagonal(lA, 0)
    lA[:] = 0
    lE = g.integers(-5000, 0, size=(S, K)).astype(np.int32)
    x = g.integers(0, K, size=T).astype(np.uint8)
    sc, path = orc.viterbi(x, z, lA, lE)
    assert sc == int(sum(lE[:, c].max() for c in x))          # free transitions: per-step best emission
    assert all(lE[path[t], x[t]] == lE[:, x[t]].max() for t in range(T))
    # S = 1
    sc, _ = orc.viterbi(x, np.array([-7], np.int32), np.array([[-3]], np.int32), np.array([[-1, -2, -4, -8]], np.int32))
    assert sc == -7 - 3 * (T - 1) + int(sum(np.array([-1, -2, -4, -8])[x]))
    # T = 0
    assert orc.viterbi(np.zeros(0, np.uint8), z, lA, lE)[0] == 0


def test_viterbi_below_forward(orc):
    """In probability space P(best path) <= P(x) (scores in micro-bits keep rounding tiny)."""
    g = np.random.default_rng(25)
    for _ in range(10):
        S, K, T = 6, 4, 30
        pi, A, E = rand_hmm(g, S, K)
        x = g.integers(0, K, size=T).astype(np.uint8)
        mu = [np.rint(np.log2(v) * 1e6).astype(np.int32) for v in (pi, A, E)]
        sc, _ = orc.viterbi(x, *mu)
        assert sc / 1e6 * math.log(2) <= orc.forward(x, pi, A, E) + 1e-6 * 2 * T
