"""Brute-force enumerators that pin the oracle (tests only; tiny inputs).

Each enumerates the OBJECTS the recurrence optimises over (alignments,
secondary structures, HMM state paths) and scores them directly, so it does
not share the recursion's decomposition: a dropped term, a wrong index or a
transposed operand in oracle/oracle.c shows up as a mismatch here.
"""
from __future__ import annotations

import itertools
import math
from functools import lru_cache


# ----------------------------------------------------------------------------- alignments
def all_global_alignments(n, m):
    """Every global alignment of lengths n and m as an op list over 'S' (substitute),
    'D' (consume s), 'I' (consume t). Count = Delannoy D(n, m)."""
    out = []

    def rec(i, j, ops):
        if i == n and j == m:
            out.append(tuple(ops))
            return
        if i < n and j < m:
            ops.append("S"); rec(i + 1, j + 1, ops); ops.pop()
        if i < n:
            ops.append("D"); rec(i + 1, j, ops); ops.pop()
        if j < m:
            ops.append("I"); rec(i, j + 1, ops); ops.pop()

    rec(0, 0, [])
    return out


def score_alignment(s, t, ops, sub, gap):
    i = j = 0
    tot = 0
    for o in ops:
        if o in "SMX":
            tot += sub(s[i], t[j]); i += 1; j += 1
        elif o == "D":
            tot -= gap; i += 1
        else:
            tot -= gap; j += 1
    assert i == len(s) and j == len(t)
    return tot


def brute_edit(s, t):
    """min over all global alignments of #mismatches + #indels."""
    best = None
    for ops in all_global_alignments(len(s), len(t)):
        c = 0
        i = j = 0
        for o in ops:
            if o == "S":
                c += s[i] != t[j]; i += 1; j += 1
            elif o == "D":
                c += 1; i += 1
            else:
                c += 1; j += 1
        best = c if best is None else min(best, c)
    return best


def brute_local_cells(s, t, sigma, gap):
    """H[i][j] = best score of any alignment of s[i0:i] with t[j0:j] (any i0<=i, j0<=j),
    empty alignment scoring 0. Returns (H, best, first row-major argmax (1-based))."""
    n, m = len(s), len(t)
    sub = lambda a, b: int(sigma[a][b])
    aligns = {}
    H = [[0] * (m + 1) for _ in range(n + 1)]
    for i in range(1, n + 1):
        for j in range(1, m + 1):
            best = 0
            for i0 in range(0, i + 1):
                for j0 in range(0, j + 1):
                    key = (i - i0, j - j0)
                    if key not in aligns:
                        aligns[key] = all_global_alignments(*key)
                    for ops in aligns[key]:
                        best = max(best, score_alignment(s[i0:i], t[j0:j], ops, sub, gap))
            H[i][j] = best
    best, bi, bj = 0, 0, 0
    for i in range(1, n + 1):
        for j in range(1, m + 1):
            if H[i][j] > best:
                best, bi, bj = H[i][j], i, j
    return H, best, (bi, bj)


def score_alignment_affine(s, t, ops, sub, go, ge):
    """Affine gap cost: every maximal run of k 'D' (or k 'I') ops costs go + k*ge; a
    D-run directly followed by an I-run is two gaps."""
    i = j = 0
    tot = 0
    prev = None
    for o in ops:
        if o in "SMX":
            tot += sub(s[i], t[j]); i += 1; j += 1
        else:
            if o != prev:
                tot -= go
            tot -= ge
            if o == "D":
                i += 1
            else:
                j += 1
        prev = o
    assert i == len(s) and j == len(t)
    return tot


def brute_local_affine(s, t, sigma, go, ge):
    """max over every local alignment (every pair of substrings, every global alignment
    of them) of the affine score; the empty alignment scores 0."""
    n, m = len(s), len(t)
    sub = lambda a, b: int(sigma[a][b])
    aligns = {}
    best = 0
    for i0 in range(n + 1):
        for i in range(i0, n + 1):
            for j0 in range(m + 1):
                for j in range(j0, m + 1):
                    key = (i - i0, j - j0)
                    if key not in aligns:
                        aligns[key] = all_global_alignments(*key)
                    for ops in aligns[key]:
                        best = max(best, score_alignment_affine(s[i0:i], t[j0:j], ops, sub, go, ge))
    return best


# ----------------------------------------------------------------------------- secondary structures
def all_structures(n, can_pair, h):
    """Every secondary structure (set of non-crossing pairs (i,j), i<j, j-i-1>=h,
    can_pair(i,j)) on positions 0..n-1, via the 'first base unpaired or paired with k'
    decomposition (not Nussinov's four cases)."""

    @lru_cache(maxsize=None)
    def rec(i, j):
        if i > j:
            return [frozenset()]
        res = list(rec(i + 1, j))  # i unpaired
        for k in range(i + h + 1, j + 1):
            if can_pair(i, k):
                for a in rec(i + 1, k - 1):
                    for b in rec(k + 1, j):
                        res.append(a | b | {(i, k)})
        return res

    return rec(0, n - 1)


def brute_nussinov(x, pair_mask, h):
    structs = all_structures(len(x), lambda i, j: bool(pair_mask[x[i]][x[j]]), h)
    return max(len(p) for p in structs), len(structs)


def dotbracket_pairs(db):
    st, pairs = [], []
    for k, c in enumerate(db):
        if c == "(":
            st.append(k)
        elif c == ")":
            assert st, "unbalanced"
            pairs.append((st.pop(), k))
        else:
            assert c == "."
    assert not st, "unbalanced"
    return sorted(pairs)


# ----------------------------------------------------------------------------- HMM paths
def brute_forward(x, pi, A, E):
    """log of sum over all S^T state paths of pi[q1] e[q1,x1] prod A[q_{t-1},q_t] e[q_t,x_t]."""
    S, T = len(pi), len(x)
    if T == 0:
        return 0.0
    tot = 0.0
    for path in itertools.product(range(S), repeat=T):
        p = pi[path[0]] * E[path[0]][x[0]]
        for k in range(1, T):
            p *= A[path[k - 1]][path[k]] * E[path[k]][x[k]]
        tot += p
    return math.log(tot) if tot > 0 else -math.inf


def brute_viterbi(x, lpi, lA, lE):
    """(max over all paths of the integer path score, lexicographically-last-position-first
    canonical path is NOT assumed: returns the score and the set of optimal paths)."""
    S, T = len(lpi), len(x)
    if T == 0:
        return 0, [()]
    best, arg = None, []
    for path in itertools.product(range(S), repeat=T):
        v = int(lpi[path[0]]) + int(lE[path[0]][x[0]])
        for k in range(1, T):
            v += int(lA[path[k - 1]][path[k]]) + int(lE[path[k]][x[k]])
        if best is None or v > best:
            best, arg = v, [path]
        elif v == best:
            arg.append(path)
    return best, arg


def viterbi_path_score(x, path, lpi, lA, lE):
    v = int(lpi[path[0]]) + int(lE[path[0]][x[0]])
    for k in range(1, len(x)):
        v += int(lA[path[k - 1]][path[k]]) + int(lE[path[k]][x[k]])
    return v
