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


# ----------------------------------------------------------------------------- canonical Nussinov structure
def canonical_structure(x, pair_mask, h, variant="durbin"):
    """The canonical optimal structure of DESIGN.md R-TB-NUSS, defined over ENUMERATED structures
    (no recursion values): on an interval (i, j) whose optimum is v,
      (1) if some optimal structure leaves i unpaired -> canonical(i+1, j);
      (2) else if some optimal structure leaves j unpaired -> canonical(i, j-1);
      (3) else if some optimal structure pairs (i, j) -> {(i,j)} + canonical(i+1, j-1);
      (4) else the smallest k such that some optimal structure has no pair crossing the cut
          k | k+1 -> canonical(i, k) + canonical(k+1, j).
    `variant` re-orders the rules ("pair_first": (3) before (1); "j_first": (2) before (1);
    "largest_k": the largest k in (4)) so tests can show the pins separate the readings."""
    n = len(x)
    can = lambda i, j: bool(pair_mask[x[i]][x[j]])

    @lru_cache(maxsize=None)
    def structs(i, j):
        if i > j:
            return (frozenset(),)
        res = list(structs(i + 1, j))
        for k in range(i + h + 1, j + 1):
            if can(i, k):
                for a in structs(i + 1, k - 1):
                    for b in structs(k + 1, j):
                        res.append(a | b | {(i, k)})
        return tuple(res)

    @lru_cache(maxsize=None)
    def canon(i, j):
        if j - i < 1:
            return frozenset()
        ss = structs(i, j)
        v = max(len(s) for s in ss)
        opt = [s for s in ss if len(s) == v]
        paired = lambda s, p: any(p in q for q in s)
        rules = []
        i_free = any(not paired(s, i) for s in opt)
        j_free = any(not paired(s, j) for s in opt)
        ij = any((i, j) in s for s in opt)
        rules = [("i", i_free), ("j", j_free), ("p", ij)]
        if variant == "pair_first":
            rules = [rules[2], rules[0], rules[1]]
        elif variant == "j_first":
            rules = [rules[1], rules[0], rules[2]]
        for name, ok in rules:
            if ok:
                if name == "i":
                    return canon(i + 1, j)
                if name == "j":
                    return canon(i, j - 1)
                return frozenset({(i, j)}) | canon(i + 1, j - 1)
        ks = [k for k in range(i + 1, j) if any(all(b <= k or a >= k + 1 for a, b in s) for s in opt)]
        k = max(ks) if variant == "largest_k" else min(ks)
        return canon(i, k) | canon(k + 1, j)

    pairs = canon(0, n - 1) if n > 1 else frozenset()
    db = ["."] * n
    for a, b in pairs:
        db[a], db[b] = "(", ")"
    return "".join(db)


# ----------------------------------------------------------------------------- vectorised enumerations (numpy)
def _np():
    import numpy as np
    return np


def local_alignment_scores(s, t, sub, gap):
    """Every local alignment enumerated explicitly (one array element per alignment): for each
    start cell (i0, j0) the scores of ALL paths to every cell (i, j) >= (i0, j0) are built by
    concatenating the path arrays of the three predecessor cells. Returns (H, best, first
    row-major argmax) with H[i][j] = max(0, max over alignments ending at (i, j))."""
    np = _np()
    n, m = len(s), len(t)
    H = np.zeros((n + 1, m + 1), dtype=np.int64)
    for i0 in range(n + 1):
        for j0 in range(m + 1):
            P = {(i0, j0): np.zeros(1, np.int64)}
            for i in range(i0, n + 1):
                for j in range(j0, m + 1):
                    if (i, j) == (i0, j0):
                        continue
                    parts = []
                    if i > i0 and j > j0:
                        parts.append(P[(i - 1, j - 1)] + sub(s[i - 1], t[j - 1]))
                    if i > i0:
                        parts.append(P[(i - 1, j)] - gap)
                    if j > j0:
                        parts.append(P[(i, j - 1)] - gap)
                    P[(i, j)] = np.concatenate(parts)
                    H[i, j] = max(H[i, j], int(P[(i, j)].max()))
    best, bi, bj = 0, 0, 0
    for i in range(1, n + 1):
        for j in range(1, m + 1):
            if H[i, j] > best:
                best, bi, bj = int(H[i, j]), i, j
    return H, best, (bi, bj)


def global_alignment_costs(s, t):
    """Edit costs of every global alignment (one element per alignment, Delannoy D(n, m))."""
    np = _np()
    n, m = len(s), len(t)
    P = {(0, 0): np.zeros(1, np.int64)}
    for i in range(n + 1):
        for j in range(m + 1):
            if (i, j) == (0, 0):
                continue
            parts = []
            if i and j:
                parts.append(P[(i - 1, j - 1)] + int(s[i - 1] != t[j - 1]))
            if i:
                parts.append(P[(i - 1, j)] + 1)
            if j:
                parts.append(P[(i, j - 1)] + 1)
            P[(i, j)] = np.concatenate(parts)
    return P[(n, m)]


_OPS = "SDI"  # reversed-op alphabet of the enumerations below: S = diagonal (M/X), D = up, I = left


def _rank_linear(prev, op):
    return {"S": 0, "D": 1, "I": 2}[op]


def rank_affine(go):
    """Context ranks of the affine traceback reading R-TB-SWA, written as a lexicographic order on
    the reversed op sequence: in H (start, or after a diagonal) diagonal < up (D) < left (I); after
    a D (inside a vertical gap) ending the gap here ranks before extending it, so with go > 0 the
    order is diagonal < I < D (a D right after a closed D-gap cannot be optimal); with go = 0 ending
    and extending give the same ops and the H order applies; after an I the H order applies
    (extending with I ranks last either way)."""
    def rank(prev, op):
        if prev == "D" and go > 0:
            return {"S": 0, "I": 1, "D": 2}[op]
        return {"S": 0, "D": 1, "I": 2}[op]
    return rank


def canonical_local_traceback(s, t, end, score, sub, go, ge, rank=_rank_linear, affine=False, whole=False):
    """Enumerate every local alignment ENDING at `end` backwards (one array element per
    alignment: score, key, last op); among those scoring `score`, return the op string (start ->
    end, 'M'/'X'/'D'/'I') and start cell of the one with the smallest key, where the key is the
    reversed op sequence under `rank` (shorter prefix first: stopping ranks before continuing).
    Linear gap: go = 0, ge = g. whole=True: only alignments starting at (0, 0) (global)."""
    np = _np()
    ei, ej = end
    L = ei + ej
    W = 4 ** np.arange(L, -1, -1, dtype=np.int64)  # digit weights, position 0 most significant
    # per cell: arrays (score, key, depth, last op code 0 none / 1 S / 2 D / 3 I)
    cells = {(ei, ej): (np.zeros(1, np.int64), np.zeros(1, np.int64), np.zeros(1, np.int64), np.zeros(1, np.int64))}
    best_key, best_start = None, None
    codes = {1: "S", 2: "D", 3: "I"}
    for i in range(ei, -1, -1):
        for j in range(ej, -1, -1):
            if (i, j) not in cells:
                continue
            sc, key, dep, last = cells.pop((i, j))
            hit = sc == score
            if hit.any() and (not whole or (i, j) == (0, 0)):
                k = int(key[hit].min())
                if best_key is None or k < best_key:
                    best_key, best_start = k, (i, j)
            for op, di, dj in (("S", 1, 1), ("D", 1, 0), ("I", 0, 1)):
                ni, nj = i - di, j - dj
                if ni < 0 or nj < 0:
                    continue
                if op == "S":
                    delta = np.full(len(sc), sub(s[i - 1], t[j - 1]), np.int64)
                elif affine:
                    same = last == {"D": 2, "I": 3}[op]
                    delta = np.where(same, -ge, -go - ge)
                else:
                    delta = np.full(len(sc), -ge, np.int64)
                r = np.array([_rank(rank, codes.get(int(p)), op) for p in range(4)], np.int64)
                nk = key + (r[last] + 1) * W[dep]
                code = {"S": 1, "D": 2, "I": 3}[op]
                new = (sc + delta, nk, dep + 1, np.full(len(sc), code, np.int64))
                if (ni, nj) in cells:
                    old = cells[(ni, nj)]
                    new = tuple(np.concatenate([a, b]) for a, b in zip(old, new))
                cells[(ni, nj)] = new
    # decode
    ops, k = [], best_key
    digits = []
    for p in range(L + 1):
        d = (k // int(W[p])) % 4
        if d == 0:
            break
        digits.append(int(d))
    # replay the ranks to recover the ops
    prev = None
    rev = []
    for d in digits:
        for op in "SDI":
            if _rank(rank, prev, op) + 1 == d:
                rev.append(op)
                prev = op
                break
    i, j = ei, ej
    out = []
    for op in rev:
        if op == "S":
            out.append("M" if s[i - 1] == t[j - 1] else "X")
            i, j = i - 1, j - 1
        elif op == "D":
            out.append("D")
            i -= 1
        else:
            out.append("I")
            j -= 1
    assert (i, j) == best_start
    return "".join(reversed(out)), best_start


def _rank(rank, prev, op):
    return rank(prev, op)


def all_paths(S, T):
    """Every state path of length T over S states, one row per path (S^T x T)."""
    np = _np()
    if T == 0:
        return np.zeros((1, 0), np.int64)
    return np.stack(np.meshgrid(*([np.arange(S)] * T), indexing="ij"), -1).reshape(-1, T)


def brute_forward_np(x, pi, A, E):
    """log of the sum over every state path of its probability (vectorised enumeration)."""
    np = _np()
    T = len(x)
    if T == 0:
        return 0.0
    P = all_paths(len(pi), T)
    x = np.asarray(x)
    p = np.asarray(pi)[P[:, 0]] * np.asarray(E)[P[:, 0], x[0]]
    for k in range(1, T):
        p = p * np.asarray(A)[P[:, k - 1], P[:, k]] * np.asarray(E)[P[:, k], x[k]]
    tot = float(p.sum())
    return math.log(tot) if tot > 0 else -math.inf


def brute_viterbi_np(x, lpi, lA, lE):
    """(best integer path score, canonical path = the optimal path whose reversal is
    lexicographically smallest), by enumerating every path."""
    np = _np()
    T = len(x)
    if T == 0:
        return 0, ()
    P = all_paths(len(lpi), T)
    x = np.asarray(x)
    v = np.asarray(lpi, np.int64)[P[:, 0]] + np.asarray(lE, np.int64)[P[:, 0], x[0]]
    for k in range(1, T):
        v = v + np.asarray(lA, np.int64)[P[:, k - 1], P[:, k]] + np.asarray(lE, np.int64)[P[:, k], x[k]]
    best = int(v.max())
    opt = P[v == best]
    order = np.lexsort(tuple(opt[:, k] for k in range(T)))  # last key = column T-1 is primary
    return best, tuple(int(c) for c in opt[order[0]])


def local_affine_best(s, t, sub, go, ge):
    """Max over EVERY local alignment of its affine score (a maximal run of k gap ops of one kind
    costs go + k*ge), enumerated per start cell as arrays (score, last op) per reachable cell;
    returns (best, first row-major end cell of a best alignment) — 0 and (0, 0) when empty wins."""
    np = _np()
    n, m = len(s), len(t)
    H = np.zeros((n + 1, m + 1), dtype=np.int64)
    for i0 in range(n + 1):
        for j0 in range(m + 1):
            P = {(i0, j0): (np.zeros(1, np.int64), np.zeros(1, np.int64))}
            for i in range(i0, n + 1):
                for j in range(j0, m + 1):
                    if (i, j) == (i0, j0):
                        continue
                    sc, lo = [], []
                    if i > i0 and j > j0:
                        a, l = P[(i - 1, j - 1)]
                        sc.append(a + sub(s[i - 1], t[j - 1])); lo.append(np.full(len(a), 1))
                    if i > i0:
                        a, l = P[(i - 1, j)]
                        sc.append(a - ge - np.where(l == 2, 0, go)); lo.append(np.full(len(a), 2))
                    if j > j0:
                        a, l = P[(i, j - 1)]
                        sc.append(a - ge - np.where(l == 3, 0, go)); lo.append(np.full(len(a), 3))
                    P[(i, j)] = (np.concatenate(sc), np.concatenate(lo))
                    H[i, j] = max(H[i, j], int(P[(i, j)][0].max()))
    best, bi, bj = 0, 0, 0
    for i in range(1, n + 1):
        for j in range(1, m + 1):
            if H[i, j] > best:
                best, bi, bj = int(H[i, j]), i, j
    return best, (bi, bj)


# ----------------------------------------------------------------------------- HMMs with silent states
def brute_silent_hmm(x, silent, A, E, begin, end):
    """log of the sum over EVERY state path begin -> ... -> end that emits exactly x (emitting
    states consume one symbol each, silent ones none), each path's probability the product of its
    transitions and emissions. Depth-first over (state, symbols emitted); silent cycles are not
    allowed (a path through a silent cycle would not terminate)."""
    T = len(x)
    S = len(silent)
    tot = 0.0
    stack = [(begin, 0, 1.0, 0)]
    while stack:
        s, i, p, depth = stack.pop()
        assert depth <= (T + 1) * S + 1, "silent cycle"
        if s == end and i == T:
            tot += p
            continue
        for t in range(S):
            a = A[s][t]
            if a <= 0:
                continue
            if silent[t]:
                stack.append((t, i, p * a, depth + 1))
            elif i < T:
                e = E[t][x[i]]
                if e > 0:
                    stack.append((t, i + 1, p * a * e, depth + 1))
    return math.log(tot) if tot > 0 else -math.inf


def brute_profile(x, trans, emit_m, emit_i):
    """log P(x) of a profile HMM by walking its states directly ((M,j), (I,j), (D,j); M_0 = begin,
    M_{L+1} = end) over every path that emits exactly x — written from the profile's own
    description, independent of any generic-HMM encoding."""
    L = len(trans) - 1
    T = len(x)
    tot = 0.0
    stack = [("M", 0, 0, 1.0)]
    while stack:
        k, j, i, p = stack.pop()
        if k == "M" and j == L + 1:
            if i == T:
                tot += p
            continue
        f = "MID".index(k)
        for t, (kt, jt) in enumerate((("M", j + 1), ("I", j), ("D", j + 1))):
            a = trans[j][3 * f + t]
            if a <= 0 or (kt == "D" and jt > L):
                continue
            if kt == "D" or (kt == "M" and jt == L + 1):
                stack.append((kt, jt, i, p * a))
            elif i < T:
                e = (emit_m if kt == "M" else emit_i)[jt][x[i]]
                if e > 0:
                    stack.append((kt, jt, i + 1, p * a * e))
    return math.log(tot) if tot > 0 else -math.inf
