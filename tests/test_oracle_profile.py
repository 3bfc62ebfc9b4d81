"""Pins for the oracle's HMM forward with silent states and the profile HMM written in the
paper's generic HMM extension (§6.3, §5.2
L448-L464; DESIGN.md R-PHMM).

* brute force: the sum over every state path emitting x, for random generic HMMs with silent
  states and for random profiles (walked from the profile's own description, not the generic
  encoding the oracle builds), T <= 5;
* normalisation: over a one-letter alphabet P(a^T) is the length distribution, sum_T = 1;
* closed forms: a pure match chain (P = prod e_Mj(x_j) when T = L, else 0), the all-delete
  path for the empty sequence;
* reduction: with only a silent begin (transitions pi) and a silent end reached from every
  state with probability 1, the silent-state forward equals the dense forward of Fig.11a."""
import math

import numpy as np
import pytest

import dpgen
from tests import brute


def rand_profile(g, L, K):
    return dpgen.profile_hmm_params(g, L, K)


def test_profile_brute_force(orc):
    g = np.random.default_rng(60)
    for k in range(40):
        L, K = int(g.integers(1, 4)), int(g.integers(1, 4))
        T = int(g.integers(0, 6))
        tr, eM, eI = rand_profile(g, L, K)
        if k % 3 == 0:   # flatter transitions: every path type matters
            tr = tr ** 0.3
            for j in range(L + 1):
                for f in range(3):
                    r = tr[j, 3 * f:3 * f + 3]
                    if j == 0 and f == 2 or r.sum() == 0:
                        tr[j, 3 * f:3 * f + 3] = 0
                        continue
                    if j == L:
                        r[2] = 0
                    tr[j, 3 * f:3 * f + 3] = r / r.sum()
        x = g.integers(0, K, size=T).astype(np.uint8)
        want = brute.brute_profile(list(x), tr, eM, eI)
        got = orc.profile_forward(x, tr, eM, eI)
        if want == -math.inf:
            assert got == -math.inf
        else:
            assert abs(got - want) <= 1e-11 * max(1.0, abs(want)), (k, L, K, T)


def random_silent_hmm(g, S, K):
    """A random generic HMM: state 0 = silent begin, S-1 = silent end, some silent states in
    between; silent -> silent transitions only go to higher indices (no silent cycle)."""
    silent = np.zeros(S, np.uint8)
    silent[0] = silent[-1] = 1
    for s in range(1, S - 1):
        silent[s] = g.random() < 0.4
    A = np.zeros((S, S))
    for p in range(S - 1):
        for s in range(1, S):
            if silent[p] and silent[s] and s <= p:
                continue
            if g.random() < 0.7:
                A[p, s] = g.random()
        if A[p].sum() == 0:
            A[p, S - 1] = 1.0
        A[p] /= A[p].sum()
    E = g.dirichlet(np.ones(K), size=S)
    return silent, A, E


def test_silent_forward_brute_force(orc):
    g = np.random.default_rng(61)
    for k in range(40):
        S, K, T = int(g.integers(3, 7)), int(g.integers(1, 4)), int(g.integers(0, 5))
        silent, A, E = random_silent_hmm(g, S, K)
        x = g.integers(0, K, size=T).astype(np.uint8)
        want = brute.brute_silent_hmm(list(x), silent, A, E, 0, S - 1)
        got = orc.silent_forward(x, silent, A, E, 0, S - 1)
        if want == -math.inf:
            assert got == -math.inf
        else:
            assert abs(got - want) <= 1e-11 * max(1.0, abs(want)), k


def test_silent_cycle_is_rejected(orc):
    silent = np.array([1, 1, 1, 1], np.uint8)
    A = np.zeros((4, 4))
    A[0, 1] = 1.0
    A[1, 2] = 0.5
    A[2, 1] = 0.5
    A[1, 3] = 0.5
    A[2, 3] = 0.5
    assert math.isnan(orc.silent_forward(np.zeros(0, np.uint8), silent, A, np.ones((4, 1)), 0, 3))


def test_profile_length_distribution_sums_to_one(orc):
    """Over a one-letter alphabet every emission is 1, so P(a^T) = P(length T); the lengths of
    a profile with insert self-loops < 1 have a geometric tail and sum to 1."""
    g = np.random.default_rng(62)
    for L in (1, 3, 7):
        tr, _, _ = rand_profile(g, L, 1)
        eM = np.ones((L + 1, 1))
        eI = np.ones((L + 1, 1))
        tot = sum(math.exp(orc.profile_forward(np.zeros(T, np.uint8), tr, eM, eI)) for T in range(0, 160))
        assert abs(tot - 1.0) < 1e-9, (L, tot)


def test_profile_closed_forms(orc):
    g = np.random.default_rng(63)
    L, K = 6, 4
    tr, eM, eI = rand_profile(g, L, K)
    # pure match chain: M_j -> M_{j+1} with probability 1
    chain = np.zeros_like(tr)
    chain[:, 0] = 1.0
    x = g.integers(0, K, size=L).astype(np.uint8)
    want = sum(math.log(eM[j + 1][x[j]]) for j in range(L))
    assert abs(orc.profile_forward(x, chain, eM, eI) - want) < 1e-12
    assert orc.profile_forward(x[:-1], chain, eM, eI) == -math.inf
    # the empty sequence only passes through the delete states
    want = math.log(tr[0][2]) + sum(math.log(tr[j][8]) for j in range(1, L)) + math.log(tr[L][6])
    assert abs(orc.profile_forward(np.zeros(0, np.uint8), tr, eM, eI) - want) < 1e-12


def test_silent_forward_reduces_to_dense_forward(orc):
    """Begin -> s with pi_s, s -> p with A, every s -> end with 1 (tau == 1, R-HMM-FWD): the
    silent-state forward is the dense forward of Fig.11a."""
    g = np.random.default_rng(64)
    for _ in range(10):
        S, K, T = int(g.integers(1, 9)), int(g.integers(2, 5)), int(g.integers(1, 40))
        pi, A, E = dpgen.hmm_params(g, S, K)
        N = S + 2
        G = np.zeros((N, N))
        G[0, 1:S + 1] = pi
        G[1:S + 1, 1:S + 1] = A
        # the end state is reached from every state; P(x) keeps sum_s F(s, T) (tau = 1)
        silent = np.zeros(N, np.uint8)
        silent[0] = silent[-1] = 1
        G[1:S + 1, N - 1] = 1.0
        EE = np.zeros((N, K))
        EE[1:S + 1] = E
        x = g.integers(0, K, size=T).astype(np.uint8)
        assert abs(orc.silent_forward(x, silent, G, EE, 0, N - 1) - orc.forward(x, pi, A, E)) < 1e-10
