"""Pins for the oracle's diagonal-only recurrence (oracle.lcsubstr; the §4.7
example f(x, y) = ... f(x-1, y-1) ..., L386-L388, instantiated as the longest
common substring, DESIGN.md R-DIAG): brute force over all substring pairs,
the standard library's longest matching block, closed forms."""
import difflib
import random

import numpy as np

import oracle


def brute(s, t):
    best = 0
    for i in range(len(s) + 1):
        for k in range(best + 1, len(s) - i + 1):
            u = s[i:i + k]
            if any(t[j:j + k] == u for j in range(len(t) - k + 1)):
                best = k
    return best


def test_bruteforce_tiny():
    rnd = random.Random(4701)
    for _ in range(600):
        k = rnd.randint(1, 4)
        s = [rnd.randrange(k) for _ in range(rnd.randint(0, 9))]
        t = [rnd.randrange(k) for _ in range(rnd.randint(0, 9))]
        assert oracle.lcsubstr(s, t) == brute(s, t), (s, t)


def test_difflib_longest_block():
    """SequenceMatcher.find_longest_match (autojunk off) is the longest common substring."""
    rnd = np.random.default_rng(4702)
    for _ in range(60):
        s = rnd.integers(0, 4, rnd.integers(1, 300)).astype(np.uint8)
        t = rnd.integers(0, 4, rnd.integers(1, 300)).astype(np.uint8)
        m = difflib.SequenceMatcher(None, s.tolist(), t.tolist(), autojunk=False)
        assert oracle.lcsubstr(s, t) == m.find_longest_match(0, len(s), 0, len(t)).size


def test_closed_forms():
    rnd = np.random.default_rng(4703)
    for n in (1, 7, 64, 513):
        s = rnd.integers(0, 4, n).astype(np.uint8)
        assert oracle.lcsubstr(s, s) == n                      # a string against itself
        assert oracle.lcsubstr(s, []) == 0 and oracle.lcsubstr([], s) == 0
        assert oracle.lcsubstr(s, s + 4) == 0                  # disjoint alphabets
        t = rnd.integers(0, 4, n + 5).astype(np.uint8)
        assert oracle.lcsubstr(s, t) == oracle.lcsubstr(t, s)  # symmetric
        u = s[n // 3: n // 3 + max(1, n // 4)]
        assert oracle.lcsubstr(s, u) == len(u)                 # a substring of s
