"""Host-side tests of the product (no GPU): the C-ABI library loads and exports
every symbol include/dp.h declares, and its symbolic schedule front-end
(dp_schedule_derive) agrees with the brute-force schedule oracle on explicit
call graphs and with the paper's worked examples."""
import json
import os
import re

import pytest

from oracle import schedule as sch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLD = json.load(open(os.path.join(ROOT, "tests", "golden", "schedule_pins.json")))


@pytest.fixture(scope="module")
def dp():
    from paper_conf_pldi_carteylm12_b200 import _build
    _build.build()
    import paper_conf_pldi_carteylm12_b200 as dp
    dp.lib()
    return dp


def test_exports_match_header(dp):
    hdr = open(os.path.join(ROOT, "include", "dp.h")).read()
    declared = set(re.findall(r"\b(dp_[a-z_]+)\s*\(", hdr))
    assert declared == set(dp.EXPORTS)
    L = dp.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert L.dp_abi_version() == 4
    for code in range(8):
        assert L.dp_status_string(code)


def U(*off):
    return (off, None, 0, 0)


def test_edit_and_sw_schedule(dp):
    for n, m in [(2, 2), (256, 256), (5, 9)]:
        r = dp.schedule_derive((n + 1, m + 1), [U(-1, 0), U(0, -1), U(-1, -1)])
        assert list(r["a"]) == GOLD["edit_schedule"]["a"]
        assert (r["p_lo"], r["p_hi"]) == (0, n + m)
        assert r["window"] == 2
        dom, calls, ext = sch.edit_instance(min(n, 5), min(m, 5))
        o = sch.derive(dom, calls, ext)
        assert o["a"] == r["a"]
    assert dp.schedule_derive((3, 3), [U(-1, 0), U(0, -1), U(-1, -1)])["p_hi"] + 1 == 5   # Fig.3


def test_user_schedule_verification(dp):
    deps = [U(-1, 0), U(0, -1), U(-1, -1)]
    r = dp.schedule_derive((5, 5), deps, user_coeff=(2, 1))          # valid, more partitions (L168-L170)
    assert r["a"] == (2, 1) and r["p_hi"] == 12
    with pytest.raises(dp.DPError) as e:
        dp.schedule_derive((5, 5), deps, user_coeff=(1, -1))
    assert e.value.code == 2


@pytest.mark.parametrize("nx,ny", [(3, 5), (5, 3), (4, 4), (7, 2)])
def test_diagonal_only_matches_oracle(dp, nx, ny):
    r = dp.schedule_derive((nx, ny), [U(-1, -1)])
    dom, calls, ext = sch.diagonal_instance(nx, ny)
    assert r["a"] == sch.derive(dom, calls, ext)["a"]
    want = GOLD["diagonal_only"]["nx_lt_ny"] if nx < ny else GOLD["diagonal_only"]["nx_gt_ny"]
    assert list(r["a"]) == want


@pytest.mark.parametrize("n", [3, 6, 64, 8192])
def test_nussinov_schedule(dp, n):
    deps = [U(1, 0), U(0, -1), U(1, -1), ((0, 0), 1, -(n - 1), -1), ((0, 0), 0, 1, n - 1)]
    r = dp.schedule_derive((n, n), deps, triangular=True)
    assert r["a"] == (-1, 1)
    assert (r["p_lo"], r["p_hi"]) == (0, n - 1)     # n partitions over the triangle
    assert r["window"] == -1                        # ranged descent: no sliding window (§4.8)
    if n <= 6:
        dom, calls, ext = sch.nussinov_instance(n)
        o = sch.derive(dom, calls, ext)
        assert o["a"] == r["a"] and (o["p_lo"], o["p_hi"]) == (r["p_lo"], r["p_hi"])


@pytest.mark.parametrize("S,T", [(4, 5), (64, 1000)])
def test_hmm_schedule(dp, S, T):
    r = dp.schedule_derive((S, T + 1), [((0, -1), 0, -(S - 1), S - 1)])
    assert list(r["a"]) == GOLD["hmm_forward"]["a"]
    assert r["window"] == 1 and (r["p_lo"], r["p_hi"]) == (0, T)
    if S * T < 40:
        dom, calls, ext = sch.hmm_instance(S, T)
        assert sch.derive(dom, calls, ext)["a"] == r["a"]


def test_fibonacci_and_cyclic(dp):
    r = dp.schedule_derive((9,), [U(-1), U(-2)])
    assert r["a"] == (1,) and r["window"] == 2
    with pytest.raises(dp.DPError) as e:
        dp.schedule_derive((5,), [U(-1), U(1)])
    assert e.value.code == 2


def test_random_families_match_bruteforce(dp):
    """Random uniform dependency sets in 2-D: symbolic criteria == explicit call graph."""
    import random
    rnd = random.Random(7)
    for _ in range(40):
        deps = set()
        while len(deps) < rnd.randint(1, 3):
            d = (rnd.randint(-2, 1), rnd.randint(-2, 1))
            if d != (0, 0):
                deps.add(d)
        nx, ny = rnd.randint(2, 5), rnd.randint(2, 5)
        dom = [(x, y) for x in range(nx) for y in range(ny)]
        calls = lambda c, deps=tuple(deps): [(c[0] + a, c[1] + b) for a, b in deps]
        o = sch.derive(dom, calls, (nx, ny))
        # the call graph only contains in-domain edges; keep cases where every family has an edge
        if any(not any((x + a, y + b) in set(dom) for x, y in dom) for a, b in deps):
            continue
        try:
            r = dp.schedule_derive((nx, ny), [U(a, b) for a, b in deps])
        except dp.DPError as e:
            assert e.code == 2 and o is None
            continue
        assert o is not None and r["a"] == o["a"], (deps, nx, ny, r, o)


def test_bad_arguments(dp):
    with pytest.raises(dp.DPError) as e:
        dp.schedule_derive((0, 3), [U(-1, 0)])
    assert e.value.code == 1


# ---------------------------------------------------------------- §4.7 conditional schedules
def test_conditional_diagonal_only(dp):
    """§4.7: f(x-1, y-1) -> candidates (0,1), (1,0); S = x when nx < ny."""
    g = GOLD["diagonal_only"]
    cands = dp.schedule_conditional(2, [U(-1, -1)])
    dom, calls, ext = sch.diagonal_instance(5, 6)
    assert cands == sch.conditional(dom, calls, 2)
    assert sorted(cands) == sorted([tuple(g["nx_lt_ny"]), tuple(g["nx_gt_ny"])])
    assert cands[dp.schedule_select(cands, (4, 9))] == tuple(g["nx_lt_ny"])
    assert cands[dp.schedule_select(cands, (9, 4))] == tuple(g["nx_gt_ny"])
    for a in g["valid_never_minimal"]:
        assert tuple(a) not in cands
        assert dp.schedule_derive((5, 6), [U(-1, -1)], user_coeff=tuple(a))["a"] == tuple(a)  # valid (L326)


def test_conditional_case_studies_single(dp):
    """The case studies' recurrences have one candidate each, equal to dp_schedule_derive's."""
    nuss = [U(1, 0), U(0, -1), U(1, -1), ((0, 0), 1, -63, -1), ((0, 0), 0, 1, 63)]
    for nd, deps, ext in [(2, [U(-1, 0), U(0, -1), U(-1, -1)], (257, 257)),
                          (2, [((-63, -1), 0, 0, 126)], (64, 1001)),
                          (2, nuss, (64, 64))]:
        cands = dp.schedule_conditional(nd, deps)
        assert cands == [dp.schedule_derive(ext, deps)["a"]]
    with pytest.raises(dp.DPError) as e:
        dp.schedule_conditional(1, [U(-1), U(1)])
    assert e.value.code == 2


@pytest.mark.parametrize("seed", range(12))
def test_conditional_matches_bruteforce(dp, seed):
    """Random uniform dependency sets in 2-D and 3-D: the symbolic front-end's candidates
    equal the brute force over the explicit call graph of a concrete instance, and each
    is dp_schedule_derive's choice for extents skewed in its permutation's order."""
    import itertools
    import random
    rnd = random.Random(seed)
    nd = 2 if seed < 6 else 3
    B = 3
    offs = []
    while len(offs) < rnd.randint(1, 3):
        o = tuple(rnd.randint(-2, 1) for _ in range(nd))
        if any(o) and o not in offs:
            offs.append(o)
    deps = [U(*o) for o in offs]
    side = 4 if nd == 3 else 6
    dom = list(itertools.product(range(side), repeat=nd))

    def calls(c):
        return [tuple(ci + oi for ci, oi in zip(c, o)) for o in offs]

    want = sch.conditional(dom, calls, nd, bound=B)
    if not want:
        with pytest.raises(dp.DPError):
            dp.schedule_conditional(nd, deps, coeff_bound=B)
        return
    got = dp.schedule_conditional(nd, deps, coeff_bound=B)
    assert got == want
    for perm in itertools.permutations(range(nd)):
        ext = [0] * nd
        for rank, d in enumerate(perm):
            ext[d] = [10 ** 6, 10 ** 4, 10 ** 2][rank]
        a = dp.schedule_derive(tuple(ext), deps, coeff_bound=B)["a"]
        assert a in got
        assert got[dp.schedule_select(got, tuple(ext))] == a


def test_profile_schedule_depends_on_state_order():
    """"the ordering of the model elements may be important ... different
    orderings may permit or restrict the available schedules". A profile HMM's silent deletes read
    the same index: with the generic `transitionsto` reading ("t.start varies over any state",
    L466-L472) that is a ranged family over all states at offset 0 in i, cyclic -> no schedule;
    with the states in position-major order the families are uniform, (-1,-1), (0,-1), (-1,0),
    and the schedule is the anti-diagonal (1,1)."""
    import paper_conf_pldi_carteylm12_b200 as dp
    S = 3 * 10 + 3
    with pytest.raises(dp.DPError) as e:
        dp.schedule_derive((S, 50), [((0, -1), 0, -(S - 1), S - 1), ((0, 0), 0, -(S - 1), S - 1)])
    assert e.value.code == 2
    r = dp.schedule_derive((11, 50), [((-1, -1), None, 0, 0), ((0, -1), None, 0, 0), ((-1, 0), None, 0, 0)])
    assert r["a"] == (1, 1) and r["window"] == 2
