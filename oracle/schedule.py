"""Schedule oracle — TEST INFRASTRUCTURE ONLY (see oracle/oracle.c header).

Brute force over EXPLICIT call graphs of small concrete instances, written
from PAPER.md §4.2–§4.8; shares nothing with the product's symbolic front-end
(paper_conf_pldi_carteylm12_b200/csrc/frontend.cpp), which reasons about
dependency *families*; this module instead enumerates every call and every
edge of the instance.

  * call graph G(C,E): every call site of every call is an edge, no branch
    analysis (§4.4);
  * schedule S_f = a1 x1 + ... + an xn with integer a (§4.2);
  * validity: S(c1) > S(c2) for every edge c1 -> c2 (eq.3), which
    implies the partition-ordering condition eq.(1) on the transitive closure;
  * goal: min_a (max_x S - min_x S) over the box 0 <= x_i < n_i (eq.4,
    L359-L369), coefficients bounded by 10 (L403-L404);
  * ties: the first solution in lexicographic order of a (DESIGN.md R-SCHED-TIE);
  * partitions are enumerated over the exact domain (Fig.9/10 L278-L282);
  * sliding window: max over edges of S(c1) - S(c2) when all call sites are
    uniform (§4.8), else None;
  * conditional schedules (§4.7): for each of the n! orders of the
    dimensions, the valid a minimising |a| dimension by dimension in that order
    ("the first lexicographical solution with respect to the permutation of
    dimensions", L398-L401; |a_i| per DESIGN.md R-SCHED-COND), then at run time
    the candidate with the smallest box range for the problem's extents.
"""
from __future__ import annotations

import itertools


def edges_of(domain, calls):
    dom = set(domain)
    out = []
    for c in domain:
        for d in calls(c):
            if d in dom:
                out.append((c, d))
    return out


def schedule_value(a, x):
    return sum(ai * xi for ai, xi in zip(a, x))


def is_valid(a, edges):
    return all(schedule_value(a, c1) > schedule_value(a, c2) for c1, c2 in edges)


def box_range(a, extents):
    """max_x S - min_x S over the box 0 <= x_i < n_i (eq.4)."""
    hi = sum(ai * (n - 1) if ai > 0 else 0 for ai, n in zip(a, extents))
    lo = sum(ai * (n - 1) if ai < 0 else 0 for ai, n in zip(a, extents))
    return hi - lo


def derive(domain, calls, extents, bound=10):
    """Returns dict(a, goal, p_lo, p_hi) or None when no valid schedule exists."""
    domain = list(domain)
    edges = edges_of(domain, calls)
    ndim = len(extents)
    best = None
    for a in itertools.product(range(-bound, bound + 1), repeat=ndim):
        if not is_valid(a, edges):
            continue
        g = box_range(a, extents)
        if best is None or g < best[1]:
            best = (a, g)
    if best is None:
        return None
    a = best[0]
    vals = [schedule_value(a, x) for x in domain]
    return {"a": tuple(a), "goal": best[1], "p_lo": min(vals), "p_hi": max(vals)}


def conditional(domain, calls, ndim, bound=10):
    """§4.7: distinct per-permutation solutions, in itertools.permutations order (identity first)."""
    edges = edges_of(list(domain), calls)
    valid = [a for a in itertools.product(range(-bound, bound + 1), repeat=ndim) if is_valid(a, edges)]
    out = []
    for perm in itertools.permutations(range(ndim)):
        if not valid:
            break
        a = min(valid, key=lambda v: (tuple(abs(v[i]) for i in perm), v))
        if a not in out:
            out.append(a)
    return out


def select(candidates, extents):
    """Run-time half of §4.7 (L384-L386): the candidate with the smallest box range (first on ties)."""
    return min(range(len(candidates)), key=lambda k: (box_range(candidates[k], extents), k))


def partitions(domain, a):
    """Partition p -> sorted cells with S(x) = p, over the exact domain."""
    parts = {}
    for x in domain:
        parts.setdefault(schedule_value(a, x), []).append(x)
    return {p: sorted(v) for p, v in sorted(parts.items())}


def window(domain, calls, a, uniform=True):
    if not uniform:
        return None
    edges = edges_of(list(domain), calls)
    return max((schedule_value(a, c1) - schedule_value(a, c2) for c1, c2 in edges), default=0)


def transitive_closure(domain, calls):
    domain = list(domain)
    idx = {c: k for k, c in enumerate(domain)}
    succ = [set() for _ in domain]
    for c1, c2 in edges_of(domain, calls):
        succ[idx[c1]].add(idx[c2])
    reach = []
    for k in range(len(domain)):
        seen, stack = set(), list(succ[k])
        while stack:
            v = stack.pop()
            if v in seen:
                continue
            seen.add(v)
            stack.extend(succ[v])
        reach.append(seen)
    return domain, idx, reach


def independent_partitions(domain, calls, a):
    """eq.(2): S(c1) == S(c2) implies no call path between c1 and c2; and eq.(1)."""
    domain, idx, reach = transitive_closure(domain, calls)
    for c1 in domain:
        for k2 in reach[idx[c1]]:
            c2 = domain[k2]
            if schedule_value(a, c1) <= schedule_value(a, c2):
                return False
    return True


# ---------------------------------------------------------------- concrete instances
def edit_instance(n, m):
    """d(i,j) on 0..n x 0..m with calls (i-1,j), (i,j-1), (i-1,j-1) (Fig.1/Fig.7)."""
    dom = [(i, j) for i in range(n + 1) for j in range(m + 1)]
    return dom, (lambda c: [(c[0] - 1, c[1]), (c[0], c[1] - 1), (c[0] - 1, c[1] - 1)]), (n + 1, m + 1)


def profile_instance(L, T, position_major=True):
    """Profile-HMM forward (§6.3) on cells (j, i), j = 0..L positions, i = 0..T: the cell holds
    M, I, D of position j; M calls (j-1, i-1), I calls (j, i-1), the silent D calls (j-1, i) (all
    three states of the called cell). position_major=False: the generic §5.2 reading over a flat
    state axis s = 3 j + type where `t.start` may be ANY state (L466-L472) and a silent state
    reads the same index: every state calls every state at i-1 (emitting) and at i (silent)."""
    if position_major:
        dom = [(j, i) for j in range(L + 1) for i in range(T + 1)]
        return dom, (lambda c: [(c[0] - 1, c[1] - 1), (c[0], c[1] - 1), (c[0] - 1, c[1])]), (L + 1, T + 1)
    S = 3 * (L + 1)
    dom = [(s, i) for s in range(S) for i in range(T + 1)]

    def calls(c):
        s, i = c
        same = [(q, i) for q in range(S) if q != s] if s % 3 == 2 else []   # silent delete states
        return [(q, i - 1) for q in range(S)] + same

    return dom, calls, (S, T + 1)


def diagonal_instance(nx, ny):
    """f(x,y) = ... f(x-1,y-1) ... (§4.7)."""
    dom = [(x, y) for x in range(nx) for y in range(ny)]
    return dom, (lambda c: [(c[0] - 1, c[1] - 1)]), (nx, ny)


def nussinov_instance(n):
    """gamma(i,j), 0 <= i <= j < n: calls (i+1,j), (i,j-1), (i+1,j-1), (i,k), (k+1,j) for i<k<j."""
    dom = [(i, j) for i in range(n) for j in range(i, n)]

    def calls(c):
        i, j = c
        out = [(i + 1, j), (i, j - 1), (i + 1, j - 1)]
        for k in range(i + 1, j):
            out += [(i, k), (k + 1, j)]
        return out

    return dom, calls, (n, n)


def hmm_instance(S, T):
    """F(s,i), s in 0..S-1, i in 0..T: sum over t in s.transitionsto of F(t.start, i-1) (Fig.11b)."""
    dom = [(s, i) for s in range(S) for i in range(T + 1)]
    return dom, (lambda c: [(p, c[1] - 1) for p in range(S)]), (S, T + 1)


def fib_instance(n):
    dom = [(x,) for x in range(n + 1)]
    return dom, (lambda c: [(c[0] - 1,), (c[0] - 2,)]), (n + 1,)


def cyclic_instance(n):
    dom = [(x,) for x in range(n)]
    return dom, (lambda c: [(c[0] - 1,), (c[0] + 1,)]), (n,)
