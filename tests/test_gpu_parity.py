"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by
element on seeded inputs. Integer scores and tracebacks bit-exact; forward
log-likelihoods within relative 1e-5 of log P (north_star; DESIGN.md §2
"Tolerances"), the achieved error printed in nats."""
import concurrent.futures
import hashlib
import json
import os

import numpy as np
import pytest

import dpgen

pytestmark = pytest.mark.gpu
THREADS = os.cpu_count() or 4


@pytest.fixture(scope="module")
def dp():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_pldi_carteylm12_b200 import _build
    _build.build()
    import paper_conf_pldi_carteylm12_b200 as dp
    return dp


def cuda(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def host(t):
    return t.cpu().numpy()


def rand_batch(g, n, lo, hi, k):
    seqs = [g.integers(0, k, size=int(g.integers(lo, hi + 1))).astype(np.uint8) for _ in range(n)]
    return seqs, dpgen.pack(seqs)


# ----------------------------------------------------------------------------- alignment
def run_align(dp, kind, a_seqs, b_seqs, sigma=None, gap=0, asz=26, tb=True, go=0, ge=0):
    a_cat, a_off = dpgen.pack(a_seqs)
    b_cat, b_off = dpgen.pack(b_seqs)
    la = max((len(s) for s in a_seqs), default=0)
    lb = max((len(s) for s in b_seqs), default=0)
    plan = dp.Plan(kind, max(la, 1), max(lb, 1), sigma=sigma, gap=gap, alphabet_size=asz, want_traceback=tb,
                   gap_open=go, gap_extend=ge)
    A = (cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off))
    sc = plan.solve_batch(*A, max_len_a=la, max_len_b=lb)
    res = {"scores": host(sc)}
    if tb:
        out, ln, co = plan.traceback(0, len(a_seqs), la + lb + 1)
        res["ops"] = [bytes(host(out[q, :int(l)])).decode() for q, l in enumerate(host(ln))]
        res["coords"] = host(co)
    plan.close()
    return res


def test_edit_random_ragged(dp, orc):
    g = np.random.default_rng(100)
    a, _ = rand_batch(g, 300, 0, 150, 26)
    b, _ = rand_batch(g, 300, 0, 150, 26)
    a += [np.zeros(0, np.uint8), dpgen.encode("kitten", dpgen.EN)]
    b += [dpgen.encode("abc", dpgen.EN), dpgen.encode("sitting", dpgen.EN)]
    r = run_align(dp, dp.EDIT, a, b)
    for q in range(len(a)):
        assert r["scores"][q] == orc.edit(a[q], b[q]), q
        assert r["ops"][q] == orc.edit_traceback(a[q], b[q]), q


@pytest.mark.parametrize("maxlen", [40, 300, 700])
def test_sw_random_ragged(dp, orc, maxlen):
    """Lengths span several lane tiles, strips (> 256 rows) and ragged tails."""
    g = np.random.default_rng(101 + maxlen)
    sig = dpgen.blosum62()
    n = 200
    a, _ = rand_batch(g, n, 0, maxlen, 24)
    b, _ = rand_batch(g, n, 0, maxlen, 24)
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24)
    for q in range(n):
        sc, ei, ej = orc.sw(a[q], b[q], sig, 4)
        assert r["scores"][q] == sc, q
        if q % 4 == 0:
            ops, co = orc.sw_traceback(a[q], b[q], sig, 4)
            assert r["ops"][q] == ops, q
            assert tuple(r["coords"][q]) == co, q


def test_sw_int32_kernel_path(dp, orc, monkeypatch):
    """The general int32 kernel (used when s16x2 could overflow) on the same cases."""
    monkeypatch.setenv("DP_FORCE_INT32", "1")
    g = np.random.default_rng(104)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 60, 0, 300, 24)
    b, _ = rand_batch(g, 60, 0, 300, 24)
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24)
    for q in range(60):
        assert r["scores"][q] == orc.sw(a[q], b[q], sig, 4)[0], q
        ops, co = orc.sw_traceback(a[q], b[q], sig, 4)
        assert r["ops"][q] == ops and tuple(r["coords"][q]) == co, q


def test_sw_s16_guard_crosses_to_int32(dp, orc):
    """a plan whose score bound does not fit the s16x2 keys takes the int32
    kernels automatically (no environment override). Identical high-scoring sequences make the
    real scores exceed the s16 traceback keys (4 x score > 32767) and, score-only, exceed int16."""
    g = np.random.default_rng(107)
    asz = 8
    sig = np.full((asz, asz), -2, np.int8)
    np.fill_diagonal(sig, 60)
    a = [g.integers(0, asz, size=int(l)).astype(np.uint8) for l in (200, 150, 260, 40)]
    b = [x.copy() for x in a]
    b[1][70] = (b[1][70] + 1) % asz
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=5, asz=asz)
    assert r["scores"][0] == 60 * 200 > 7900
    for q in range(4):
        sc, _, _ = orc.sw(a[q], b[q], sig, 5)
        ops, co = orc.sw_traceback(a[q], b[q], sig, 5)
        assert r["scores"][q] == sc and r["ops"][q] == ops and tuple(r["coords"][q]) == co, q
    sig2 = np.full((asz, asz), -2, np.int8)
    np.fill_diagonal(sig2, 127)
    a2 = [g.integers(0, asz, size=300).astype(np.uint8)]
    r2 = run_align(dp, dp.SW_LINEAR, a2, [a2[0].copy()], sigma=sig2, gap=5, asz=asz, tb=False)
    assert r2["scores"][0] == 127 * 300 == orc.sw(a2[0], a2[0], sig2, 5)[0] > 32767


def _sw_check_all(orc, r, a, b, sig, gap):
    for q in range(len(a)):
        sc, _, _ = orc.sw(a[q], b[q], sig, gap)
        ops, co = orc.sw_traceback(a[q], b[q], sig, gap)
        assert r["scores"][q] == sc and r["ops"][q] == ops and tuple(r["coords"][q]) == co, q


def test_sw_inter_short_pairs(dp, orc):
    """SURVEY §8(f) NEXT 1 (inter-task, one pair per thread): a batch whose
    pairs all have max(|a|, |b|) <= 64 runs k_sw_inter. Lengths 0..64 cover every column bucket,
    empty sides, the 64-column maximum and ragged warps (3001 pairs: a partial last warp)."""
    g = np.random.default_rng(120)
    sig = dpgen.blosum62()
    n = 3001
    a, _ = rand_batch(g, n, 0, 64, 20)
    b, _ = rand_batch(g, n, 0, 64, 20)
    a[0], b[0] = a[0][:0], b[0][:5]          # empty a
    a[1], b[1] = a[1][:64], b[1][:0]         # empty b
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24)
    _sw_check_all(orc, r, a, b, sig, 4)


def test_sw_inter_ties_and_gap_one(dp, orc):
    """Low-entropy alphabet (frequent ties: end-cell and direction tie-breaks), gap 1 (the
    smallest gap the inter-task kernel's sentinel-column argument allows), self-alignments."""
    g = np.random.default_rng(121)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 500, 1, 64, 3)
    b, _ = rand_batch(g, 500, 1, 64, 3)
    b[:40] = [x.copy() for x in a[:40]]
    for gap in (1, 4):
        r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=gap, asz=24)
        _sw_check_all(orc, r, a, b, sig, gap)


def test_sw_inter_matches_intra(dp, orc, monkeypatch):
    """The hybrid's two kernels agree on the same short batch: the inter-task path (default) and
    the intra-task warp kernel (DP_SW_INTRA=1) give identical scores, ops and coordinates, and
    launch different kernels (launch counts differ)."""
    g = np.random.default_rng(122)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 700, 1, 64, 20)
    b, _ = rand_batch(g, 700, 1, 64, 20)
    r1 = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24)
    monkeypatch.setenv("DP_SW_INTRA", "1")
    r2 = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24)
    assert (r1["scores"] == r2["scores"]).all()
    assert r1["ops"] == r2["ops"] and (r1["coords"] == r2["coords"]).all()
    for q in range(0, 700, 7):
        assert r1["scores"][q] == orc.sw(a[q], b[q], sig, 4)[0]


def test_sw_inter_score_only_and_host_path(dp, orc):
    """Score-only plan (no code retention) and the host entry point (chunked H2D / solve /
    traceback / D2H) on a short batch larger than one host chunk."""
    g = np.random.default_rng(123)
    sig = dpgen.blosum62()
    n = 40000
    a, (a_cat, a_off) = rand_batch(g, n, 0, 64, 20)
    b, (b_cat, b_off) = rand_batch(g, n, 0, 64, 20)
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24, tb=False)
    want = orc.sw_batch(a_cat, a_off, b_cat, b_off, sig, 4, threads=THREADS)
    assert (r["scores"] == want).all()
    with dp.Plan(dp.SW_LINEAR, 64, 64, sigma=sig, gap=4, want_traceback=True) as p:
        sc, tb, tl, co = p.solve_batch_host(a_cat, a_off, b_cat, b_off, tb_stride=129)
    assert (sc == want).all()
    for q in range(0, n, 97):
        ops, c = orc.sw_traceback(a[q], b[q], sig, 4)
        assert bytes(tb[q, :tl[q]]).decode() == ops and tuple(co[q]) == c, q


def test_sw_packed_odd_batch_and_ties(dp, orc):
    """Odd batch (last warp half empty), mismatched pair lengths in one warp, and
    a low-entropy alphabet that makes ties frequent (end cell / traceback tie-breaks)."""
    g = np.random.default_rng(105)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 77, 1, 260, 3)
    b, _ = rand_batch(g, 77, 1, 90, 3)
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=2, asz=24)
    for q in range(77):
        sc, ei, ej = orc.sw(a[q], b[q], sig, 2)
        ops, co = orc.sw_traceback(a[q], b[q], sig, 2)
        assert r["scores"][q] == sc and r["ops"][q] == ops and tuple(r["coords"][q]) == co, q


def test_sw_long_columns_multiwindow_search(dp, orc):
    """|b| > 993 (more than 32 checkpoint slabs: the end-cell search probes several slab
    windows), several strips of rows, and a 3-letter alphabet so that the maximum recurs in
    several slabs (the candidate list of one window is walked slab by slab)."""
    g = np.random.default_rng(106)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 24, 150, 600, 3)
    b, _ = rand_batch(g, 24, 1000, 1600, 3)
    a[0], b[0] = np.zeros(700, np.uint8), np.zeros(1500, np.uint8)   # one long run: ties everywhere
    r = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=3, asz=24)
    for q in range(24):
        sc, ei, ej = orc.sw(a[q], b[q], sig, 3)
        ops, co = orc.sw_traceback(a[q], b[q], sig, 3)
        assert r["scores"][q] == sc and r["ops"][q] == ops and tuple(r["coords"][q]) == co, q


@pytest.mark.parametrize("maxlen,go,ge", [(40, 11, 1), (300, 11, 1), (300, 3, 2), (600, 0, 4)])
def test_sw_affine_random_ragged(dp, orc, maxlen, go, ge):
    """Affine gaps (NEXT rank 1): ragged lengths across lane tiles and strips; scores
    and canonical three-table tracebacks bit-exact."""
    g = np.random.default_rng(110 + maxlen + go)
    sig = dpgen.blosum62()
    n = 120
    a, _ = rand_batch(g, n, 0, maxlen, 24)
    b, _ = rand_batch(g, n, 0, maxlen, 24)
    a += [np.arange(20, dtype=np.uint8)]
    b += [np.concatenate([np.arange(10), [5, 5, 5], np.arange(10, 20)]).astype(np.uint8)]  # one long gap
    r = run_align(dp, dp.SW_AFFINE, a, b, sigma=sig, asz=24, go=go, ge=ge)
    for q in range(len(a)):
        sc, _, _ = orc.sw_affine(a[q], b[q], sig, go, ge)
        assert r["scores"][q] == sc, q
        if q % 3 == 0 or q == len(a) - 1:
            ops, co = orc.sw_affine_traceback(a[q], b[q], sig, go, ge)
            assert r["ops"][q] == ops, q
            assert tuple(r["coords"][q]) == co, q


def test_sw_affine_int32_kernel_path(dp, orc, monkeypatch):
    """The int32 affine kernel (used when the s16x2 keys could overflow) on ragged cases."""
    monkeypatch.setenv("DP_FORCE_INT32", "1")
    g = np.random.default_rng(121)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 60, 0, 300, 24)
    b, _ = rand_batch(g, 60, 0, 300, 24)
    r = run_align(dp, dp.SW_AFFINE, a, b, sigma=sig, asz=24, go=11, ge=1)
    for q in range(60):
        assert r["scores"][q] == orc.sw_affine(a[q], b[q], sig, 11, 1)[0], q
        ops, co = orc.sw_affine_traceback(a[q], b[q], sig, 11, 1)
        assert r["ops"][q] == ops and tuple(r["coords"][q]) == co, q


def test_sw_affine_packed_variants(dp, orc):
    """The packed s16x2 affine kernel: chosen for BLOSUM62-range scores (odd batch: the last warp
    carries one problem), score-only equal to traceback mode, tie-heavy inputs (a 2-letter
    alphabet, repeats, identical pairs); a sigma whose keys 4 sigma + 3 leave int8 falls back to
    the int32 kernel, bit-exact as well."""
    g = np.random.default_rng(122)
    n = 81
    a = [g.integers(0, 2, size=int(g.integers(0, 90))).astype(np.uint8) for _ in range(n)]
    b = [g.integers(0, 2, size=int(g.integers(0, 90))).astype(np.uint8) for _ in range(n)]
    a += [np.array([0, 1] * 20, np.uint8), np.zeros(30, np.uint8)]
    b += [np.array([0, 1] * 20, np.uint8), np.zeros(25, np.uint8)]
    a_cat, a_off = dpgen.pack(a)
    b_cat, b_off = dpgen.pack(b)
    A = (cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off))
    m = len(a)
    for sig, go, ge, want in ((np.array([[2, -1], [-1, 2]], np.int8), 2, 1, "k_affine16"),
                              (np.array([[3, -3], [-3, 3]], np.int8), 0, 2, "k_affine16"),
                              (np.array([[40, -9], [-9, 40]], np.int8), 5, 1, "k_align_affine")):
        with dp.Plan(dp.SW_AFFINE, 90, 90, sigma=sig, alphabet_size=2, want_traceback=True, gap_open=go,
                     gap_extend=ge) as p:
            sc = host(p.solve_batch(*A, max_len_a=90, max_len_b=90))
            assert p.last_variant == want
            out, ln, co = p.traceback(0, m, 181)
            out, ln, co = host(out), host(ln), host(co)
        with dp.Plan(dp.SW_AFFINE, 90, 90, sigma=sig, alphabet_size=2, want_traceback=False, gap_open=go,
                     gap_extend=ge) as p:
            sc0 = host(p.solve_batch(*A, max_len_a=90, max_len_b=90))
        assert (sc0 == sc).all()
        for q in range(m):
            assert sc[q] == orc.sw_affine(a[q], b[q], sig, go, ge)[0], (want, q)
            ops, c = orc.sw_affine_traceback(a[q], b[q], sig, go, ge)
            assert bytes(out[q, :ln[q]]).decode() == ops and tuple(co[q]) == c, (want, q)


def test_sw_affine_packed_guard_boundaries(dp, orc):
    """SURVEY §8(c) C7 for the packed affine kernel: the plan checks 4 sigma_max min(|a|,|b|) + 3
    <= 32000 (keys 4 v + code in int16) and 4 sigma + 4 (go + ge) + 2 in int8 (the profile holds the
    opening-shifted diagonal term); one residue under / over each bound picks k_affine16 /
    k_align_affine, both bit-exact on identical (high-scoring) and random pairs."""
    sig = dpgen.blosum62()
    g = np.random.default_rng(123)
    for L, go, ge, want in ((727, 11, 1, "k_affine16"), (728, 11, 1, "k_align_affine"),
                            (200, 19, 1, "k_affine16"), (200, 20, 1, "k_align_affine")):
        x = g.integers(0, 20, size=L).astype(np.uint8)
        y = g.integers(0, 20, size=L).astype(np.uint8)
        a, b = [x, x, y], [x.copy(), y, x]
        r = run_align(dp, dp.SW_AFFINE, a, b, sigma=sig, asz=24, go=go, ge=ge)
        with dp.Plan(dp.SW_AFFINE, L, L, sigma=sig, alphabet_size=24, want_traceback=True, gap_open=go,
                     gap_extend=ge) as p:
            a_cat, a_off = dpgen.pack(a)
            b_cat, b_off = dpgen.pack(b)
            p.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=L, max_len_b=L)
            assert p.last_variant == want, (L, go, want)
        for q in range(3):
            assert r["scores"][q] == orc.sw_affine(a[q], b[q], sig, go, ge)[0], (L, go, q)
            ops, co = orc.sw_affine_traceback(a[q], b[q], sig, go, ge)
            assert r["ops"][q] == ops and tuple(r["coords"][q]) == co, (L, go, q)


def test_sw_affine_config2_sampled(dp, orc):
    """BASELINE config 2's pairs with affine gaps (open 11, extend 1) at full size,
    in the bench's launch configuration; sampled pairs against the oracle."""
    n = 100_000
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n, 256, first=0)
    sig = dpgen.blosum62()
    plan = dp.Plan(dp.SW_AFFINE, 256, 256, sigma=sig, alphabet_size=24, want_traceback=True, gap_open=11,
                   gap_extend=1)
    sc = host(plan.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=256, max_len_b=256))
    out, ln, co = plan.traceback(0, n, 513)
    idx = np.random.default_rng(111).choice(n, 40, replace=False)
    out, ln, co = host(out), host(ln), host(co)
    for q in idx:
        a = a_cat[a_off[q]:a_off[q + 1]]
        b = b_cat[b_off[q]:b_off[q + 1]]
        ops, c = orc.sw_affine_traceback(a, b, sig, 11, 1)
        assert sc[q] == orc.sw_affine(a, b, sig, 11, 1)[0], q
        assert bytes(out[q, :ln[q]]).decode() == ops and tuple(co[q]) == c, q
    plan.close()


def test_sw_score_only_matches_traceback_mode(dp):
    g = np.random.default_rng(102)
    sig = dpgen.blosum62()
    a, _ = rand_batch(g, 64, 1, 256, 20)
    b, _ = rand_batch(g, 64, 1, 256, 20)
    r1 = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24, tb=False)
    r2 = run_align(dp, dp.SW_LINEAR, a, b, sigma=sig, gap=4, asz=24, tb=True)
    assert (r1["scores"] == r2["scores"]).all()


def test_sw_config2_full_size_sampled(dp, orc):
    """BASELINE config 2 at full size (100k x 256, the bench launch), sampled against the oracle."""
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs()
    sig = dpgen.blosum62()
    plan = dp.Plan(dp.SW_LINEAR, 256, 256, sigma=sig, gap=dpgen.SW_GAP, want_traceback=True)
    A = (cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off))
    sc = host(plan.solve_batch(*A, max_len_a=256, max_len_b=256))
    n = len(a_off) - 1
    ids = np.random.default_rng(103).choice(n, size=150, replace=False)
    ids = np.concatenate([ids, [0, n - 1]])
    out, ln, co = plan.traceback(0, n, 513)
    out, ln, co = host(out), host(ln), host(co)
    for q in ids:
        s, t = a_cat[a_off[q]:a_off[q + 1]], b_cat[b_off[q]:b_off[q + 1]]
        assert sc[q] == orc.sw(s, t, sig, dpgen.SW_GAP)[0]
        ops, c = orc.sw_traceback(s, t, sig, dpgen.SW_GAP)
        assert bytes(out[q, :ln[q]]).decode() == ops
        assert tuple(co[q]) == c
    assert sc.min() >= 0 and sc.max() <= 11 * 256
    plan.close()


def test_align_degenerate(dp, orc):
    sig = dpgen.blosum62()
    e = np.zeros(0, np.uint8)
    x = dpgen.encode("ARND", dpgen.PROTEIN)
    r = run_align(dp, dp.SW_LINEAR, [e, x, e], [x, e, e], sigma=sig, gap=4, asz=24)
    assert list(r["scores"]) == [0, 0, 0] and r["ops"] == ["", "", ""]
    r = run_align(dp, dp.EDIT, [e, x, e], [x, e, e], asz=24)
    assert list(r["scores"]) == [4, 4, 0]
    assert r["ops"] == ["IIII", "DDDD", ""]


# ----------------------------------------------------------------------------- Nussinov
def run_nuss(dp, seqs, h=3, pm=None, tb=True):
    pm = dpgen.rna_pair_mask() if pm is None else pm
    cat, off = dpgen.pack(seqs)
    ml = max((len(s) for s in seqs), default=1)
    plan = dp.Plan(dp.NUSSINOV, max(ml, 1), pair_mask=pm, min_hairpin=h, want_traceback=tb)
    sc = host(plan.solve_batch(cuda(cat), cuda(off), max_len_a=ml))
    res = {"scores": sc}
    if tb:
        out, ln, _ = plan.traceback(0, len(seqs), max(ml, 1), coords=False)
        res["db"] = [bytes(host(out[q, :int(l)])).decode() for q, l in enumerate(host(ln))]
    plan.close()
    return res


def test_nussinov_config1(dp, orc):
    x = dpgen.config1_rna64()
    r = run_nuss(dp, [x])
    assert r["scores"][0] == orc.nussinov(x, dpgen.rna_pair_mask(), 3)
    assert r["db"][0] == orc.nussinov_traceback(x, dpgen.rna_pair_mask(), 3)[1]


@pytest.mark.parametrize("h", [0, 3])
def test_nussinov_random_smem(dp, orc, h):
    g = np.random.default_rng(110 + h)
    seqs, _ = rand_batch(g, 120, 0, 200, 4)
    seqs += [dpgen.encode("GGGGAAAACCCC", dpgen.RNA), dpgen.encode("A" * 50, dpgen.RNA)]
    pm = dpgen.rna_pair_mask(gu=(h == 3))
    r = run_nuss(dp, seqs, h=h, pm=pm)
    for q, x in enumerate(seqs):
        sc, db = orc.nussinov_traceback(x, pm, h)
        assert r["scores"][q] == sc, q
        assert r["db"][q] == db, q


@pytest.mark.parametrize("h", [0, 1, 3])
def test_nussinov_small_kernel_edges(dp, orc, h):
    """k_nuss_small (one CTA per problem, table in shared memory; a few problems of <= 128 nt):
    lengths at the 8-wide chunk edges and the 128 maximum, empty and 1-nt problems, hairpins 0
    (the d = 1 pair term), 1 and 3, poly-A (score 0) and a fully pairing hairpin."""
    g = np.random.default_rng(170 + h)
    lens = [0, 1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 63, 64, 65, 100, 127, 128]
    seqs = [g.integers(0, 4, size=l).astype(np.uint8) for l in lens]
    seqs += [dpgen.encode("A" * 90, dpgen.RNA), dpgen.encode("GGGGGGGGAAAACCCCCCCC", dpgen.RNA)]
    pm = dpgen.rna_pair_mask(gu=(h != 0))
    r = run_nuss(dp, seqs, h=h, pm=pm)
    for q, x in enumerate(seqs):
        assert (r["scores"][q], r["db"][q]) == orc.nussinov_traceback(x, pm, h), (q, len(x))
    r1 = run_nuss(dp, [seqs[-4]], h=h, pm=pm)  # a single problem (config 1's launch)
    assert (r1["scores"][0], r1["db"][0]) == orc.nussinov_traceback(seqs[-4], pm, h)


@pytest.mark.parametrize("lens", [[129, 160, 300, 512, 33, 0, 1], [513, 700, 1000, 1024, 640]])
def test_nussinov_cluster_path(dp, orc, lens, monkeypatch):
    """a few mid-length problems, one thread-block cluster each with the
    table in distributed shared memory (tile-diagonals separated by cluster barriers); lengths
    around tile multiples, the cluster sizes' capacity edges (512 / 1024), empty and 1-nt
    problems in the same batch. Bit-exact scores and canonical dot-brackets against the oracle
    and against the batch kernel (DP_NUSS_NO_CLUSTER=1) on the same batch."""
    g = np.random.default_rng(180 + len(lens))
    seqs = [g.integers(0, 4, size=l).astype(np.uint8) for l in lens]
    r = run_nuss(dp, seqs)
    pm = dpgen.rna_pair_mask()
    with concurrent.futures.ThreadPoolExecutor(THREADS) as ex:
        want = list(ex.map(lambda x: orc.nussinov_traceback(x, pm, 3), seqs))
    for q, x in enumerate(seqs):
        assert (r["scores"][q], r["db"][q]) == want[q], (q, len(x))
    monkeypatch.setenv("DP_NUSS_NO_CLUSTER", "1")
    r2 = run_nuss(dp, seqs)
    assert list(r2["scores"]) == list(r["scores"]) and r2["db"] == r["db"]


@pytest.mark.parametrize("lens", [[128, 127, 5], [129, 128, 5], [1024, 700], [1025]])
def test_nussinov_dispatch_boundaries(dp, orc, lens):
    """The plan's Nussinov variants meet at 128 / 129 nt (one small CTA per problem vs a cluster
    per problem) and 1024 / 1025 nt (a cluster per problem vs the whole grid for one problem):
    batches on either side of each boundary, with and without tracebacks, bit-exact."""
    g = np.random.default_rng(190 + sum(lens))
    seqs = [g.integers(0, 4, size=l).astype(np.uint8) for l in lens]
    pm = dpgen.rna_pair_mask()
    with concurrent.futures.ThreadPoolExecutor(THREADS) as ex:
        want = list(ex.map(lambda x: orc.nussinov_traceback(x, pm, 3), seqs))
    r = run_nuss(dp, seqs)
    for q, x in enumerate(seqs):
        assert (r["scores"][q], r["db"][q]) == want[q], (q, len(x))
    r0 = run_nuss(dp, seqs, tb=False)
    assert [int(v) for v in r0["scores"]] == [w[0] for w in want]


def test_nussinov_cell_level_path(dp, orc, monkeypatch):
    """The cell-level CTA kernels (shared-memory table; L2 table above 340) on the same cases."""
    monkeypatch.setenv("DP_NUSS_CELL", "1")
    g = np.random.default_rng(113)
    seqs, _ = rand_batch(g, 40, 0, 420, 4)
    r = run_nuss(dp, seqs)
    pm = dpgen.rna_pair_mask()
    for q, x in enumerate(seqs):
        sc, db = orc.nussinov_traceback(x, pm, 3)
        assert r["scores"][q] == sc and r["db"][q] == db, q


def test_nussinov_tiled_ragged(dp, orc):
    """Tiled batch kernel: lengths around tile multiples (31, 32, 33, 64, 65 ...)."""
    g = np.random.default_rng(114)
    lens = [129, 130, 159, 160, 161, 191, 192, 193, 255, 256, 257, 300, 2, 1, 0, 31, 32, 33]
    seqs = [g.integers(0, 4, size=l).astype(np.uint8) for l in lens]
    r = run_nuss(dp, seqs)
    pm = dpgen.rna_pair_mask()
    for q, x in enumerate(seqs):
        sc, db = orc.nussinov_traceback(x, pm, 3)
        assert r["scores"][q] == sc and r["db"][q] == db, (q, len(x))


def test_nussinov_global_scratch_path(dp, orc):
    """Lengths above the shared-memory limit use the L2-resident table."""
    g = np.random.default_rng(112)
    seqs, _ = rand_batch(g, 6, 341, 512, 4)
    r = run_nuss(dp, seqs)
    pm = dpgen.rna_pair_mask()
    for q, x in enumerate(seqs):
        sc, db = orc.nussinov_traceback(x, pm, 3)
        assert r["scores"][q] == sc and r["db"][q] == db, q


def test_nussinov_grid_sweep(dp, orc):
    """A single large table swept by the whole grid (config 4's path) at n = 1500."""
    x = dpgen.random_seq(dpgen.rng(5, extra=9), 1500, 4)
    r = run_nuss(dp, [x])
    sc, db = orc.nussinov_traceback(x, dpgen.rna_pair_mask(), 3)
    assert r["scores"][0] == sc and r["db"][0] == db


def test_nussinov_config4_golden(dp):
    """BASELINE config 4 (n = 8192, the grid-wide sweep, the bench's launch) bit-exact against the
    oracle's verdict committed in tests/golden/config4.json (written by
    scripts/make_golden_config4.py, which calls only oracle/): score and dot-bracket."""
    from tests import brute
    with open(os.path.join(os.path.dirname(__file__), "golden", "config4.json")) as f:
        gold = json.load(f)
    x = dpgen.config4_rna8192()
    assert hashlib.sha256(x.tobytes()).hexdigest() == gold["input_sha256"]
    r = run_nuss(dp, [x])
    assert r["scores"][0] == gold["score"]
    assert hashlib.sha256(r["db"][0].encode()).hexdigest() == gold["dotbracket_sha256"]
    assert r["db"][0] == gold["dotbracket"]
    pairs = brute.dotbracket_pairs(r["db"][0])
    assert len(pairs) == gold["score"]


def test_nussinov_config5_sampled(dp, orc):
    """BASELINE config 5 at full size (1M RNAs, U[128, 512]) in the bench's launch (scores and
    tracebacks of the whole batch in one solve); scores and canonical dot-brackets of a seeded
    sample (ids spread over the batch plus the first and last) bit-exact against the oracle."""
    cat, off = dpgen.config5_rna_batch()
    n = len(off) - 1
    lens = np.diff(off)
    ml = int(lens.max())
    pm = dpgen.rna_pair_mask()
    plan = dp.Plan(dp.NUSSINOV, ml, pair_mask=pm, min_hairpin=3, want_traceback=True)
    sc = host(plan.solve_batch(cuda(cat), cuda(off), max_len_a=ml))
    out, ln, _ = plan.traceback(0, n, 512, coords=False)
    out, ln = host(out), host(ln)
    plan.close()
    ids = np.concatenate([[0, n - 1], np.sort(np.random.default_rng(141).choice(n, 62, replace=False))])
    ids = np.concatenate([ids, [int(np.argmax(lens)), int(np.argmin(lens))]])

    def one(q):
        return orc.nussinov_traceback(cat[off[q]:off[q + 1]], pm, 3)

    with concurrent.futures.ThreadPoolExecutor(THREADS) as ex:
        want = list(ex.map(one, ids))
    for q, (wsc, wdb) in zip(ids, want):
        assert sc[q] == wsc, q
        assert ln[q] == lens[q] and bytes(out[q, :ln[q]]).decode() == wdb, q
    # scores of a larger seeded subset (oracle, scores only)
    sub = dpgen.config5_sample_ids(k=400)
    scat, soff = dpgen.config5_rna_batch(ids=sub)
    assert (sc[sub] == orc.nussinov_batch(scat, soff, pm, 3, threads=THREADS)).all()


def test_nussinov_batch_sampled_small(dp, orc):
    ids = dpgen.config5_sample_ids(k=400)
    cat, off = dpgen.config5_rna_batch(ids=ids)
    seqs = [cat[off[q]:off[q + 1]] for q in range(len(ids))]
    r = run_nuss(dp, seqs, tb=True)
    for q in range(0, len(ids), 20):
        assert (r["scores"][q], r["db"][q]) == orc.nussinov_traceback(seqs[q], dpgen.rna_pair_mask(), 3), q
    want = orc.nussinov_batch(cat, off, dpgen.rna_pair_mask(), 3, threads=THREADS)
    assert (r["scores"] == want).all()


# ----------------------------------------------------------------------------- HMM
def hmm_case(g, S, n, tlo, thi):
    pi, A, E = dpgen.hmm_params(g, S, 4)
    pi32, A32, E32 = (v.astype(np.float32) for v in (pi, A, E))
    seqs = [dpgen.sample_hmm(g, pi, A, E, 1, int(g.integers(tlo, thi + 1)))[0] for _ in range(n)]
    return pi32, A32, E32, seqs


def forward_errors(ll, want, label, capsys):
    """Achieved error of log P: max |delta| in nats and max relative; printed into the test log
    (the north_star bar is relative 1e-5 of log P, DESIGN.md §2 "Tolerances")."""
    ll, want = np.asarray(ll, np.float64), np.asarray(want, np.float64)
    d = np.abs(ll - want)
    rel = d / np.maximum(np.abs(want), 1e-30)
    with capsys.disabled():
        print(f"\n[forward {label}] n={len(d)} max |dlogP| = {d.max():.3e} nats, max rel = {rel.max():.3e}")
    return d, rel


@pytest.mark.parametrize("S", [1, 5, 64])
def test_forward_random(dp, orc, S, capsys):
    g = np.random.default_rng(120 + S)
    pi, A, E, seqs = hmm_case(g, S, 60, 0, 300)
    cat, off = dpgen.pack(seqs)
    plan = dp.Plan(dp.HMM_FORWARD, max(len(s) for s in seqs), pi=pi, A=A, E=E)
    ll = host(plan.solve_batch(cuda(cat), cuda(off)))
    want = orc.forward_batch(cat, off, pi.astype(np.float64), A.astype(np.float64), E.astype(np.float64),
                             threads=THREADS)
    live = np.array([len(x) > 0 for x in seqs])
    assert (ll[~live] == 0.0).all()
    dl, rel = forward_errors(ll[live], want[live], f"tcgen05 S={S}", capsys)
    assert rel.max() <= 1e-5


@pytest.mark.parametrize("S", [5, 64])
def test_forward_simt_path(dp, orc, S, monkeypatch, capsys):
    """The SIMT forward kernel (used when the tensor-core path is disabled)."""
    monkeypatch.setenv("DP_HMM_SIMT", "1")
    g = np.random.default_rng(125 + S)
    pi, A, E, seqs = hmm_case(g, S, 40, 0, 300)
    cat, off = dpgen.pack(seqs)
    plan = dp.Plan(dp.HMM_FORWARD, max(len(s) for s in seqs), pi=pi, A=A, E=E)
    ll = host(plan.solve_batch(cuda(cat), cuda(off)))
    want = orc.forward_batch(cat, off, pi.astype(np.float64), A.astype(np.float64), E.astype(np.float64),
                             threads=THREADS)
    dl, rel = forward_errors(ll, want, f"SIMT S={S}", capsys)
    assert rel.max() <= 1e-5


@pytest.mark.parametrize("S", [1, 7, 64])
def test_viterbi_random(dp, orc, S):
    g = np.random.default_rng(130 + S)
    pi, A, E, seqs = hmm_case(g, S, 60, 0, 300)
    lpi, lA, lE = dpgen.millibits(pi), dpgen.millibits(A), dpgen.millibits(E)
    cat, off = dpgen.pack(seqs)
    ml = max(len(s) for s in seqs)
    plan = dp.Plan(dp.HMM_VITERBI, ml, lpi=lpi, lA=lA, lE=lE, want_traceback=True)
    sc = host(plan.solve_batch(cuda(cat), cuda(off)))
    assert plan.last_variant == "k_viterbi16"  # Dirichlet(1) scores fit the 16-bit guard
    out, ln, _ = plan.traceback(0, len(seqs), max(ml, 1), coords=False)
    out, ln = host(out), host(ln)
    for q, x in enumerate(seqs):
        v, path = orc.viterbi(x, lpi, lA, lE)
        assert sc[q] == v, q
        assert ln[q] == len(x) and (out[q, :len(x)] == path).all(), q


def _viterbi_check(dp, orc, lpi, lA, lE, seqs, variant, tb=True):
    cat, off = dpgen.pack(seqs)
    ml = max(max(len(s) for s in seqs), 1)
    plan = dp.Plan(dp.HMM_VITERBI, ml, lpi=lpi, lA=lA, lE=lE, want_traceback=tb)
    sc = host(plan.solve_batch(cuda(cat), cuda(off)))
    assert plan.last_variant == variant
    if tb:
        out, ln, _ = plan.traceback(0, len(seqs), ml, coords=False)
        out, ln = host(out), host(ln)
    for q, x in enumerate(seqs):
        v, path = orc.viterbi(x, lpi, lA, lE)
        assert sc[q] == v, q
        if tb:
            assert ln[q] == len(x) and (out[q, :len(x)] == path).all(), q


@pytest.mark.parametrize("case", ["int32_forced", "guard_fails", "saturating", "ties", "odd_ragged", "score_only"])
def test_viterbi_variants(dp, orc, case, monkeypatch):
    """The s16x2 Viterbi's guard (hmm_vit16.cu: A' <= 16383 exact, saturating emission add when
    A' + E'' > 32768) and the int32 kernel it falls back to, each bit-exact against the oracle."""
    g = np.random.default_rng(150 + len(case))
    S = 64 if case != "odd_ragged" else 23
    pi, A, E = dpgen.hmm_params(g, S, 4)
    lpi, lA, lE = dpgen.millibits(pi), dpgen.millibits(A), dpgen.millibits(E)
    seqs = [dpgen.sample_hmm(g, pi, A, E, 1, int(g.integers(0, 200)))[0] for _ in range(21)]
    variant = "k_viterbi16"
    if case == "int32_forced":
        monkeypatch.setenv("DP_FORCE_INT32", "1")
        variant = "k_viterbi"
    elif case == "guard_fails":      # one transition at the p = 0 floor: A' = 100000-ish > 16383
        lA = lA.copy()
        lA[3, 5] = dpgen.MILLIBIT_FLOOR
        variant = "k_viterbi"
    elif case == "saturating":       # A' within the guard, emissions down to 2^-24: A' + E'' > 32768
        lA = np.maximum(lA, lA.max(axis=0, keepdims=True) - 12000).astype(np.int32)
        lE = lE.copy()
        lE[::3, 1] = -24000
        cr = lA.max(axis=0)
        ep = lE + cr[:, None]
        assert (cr - lA.min(axis=0)).max() + (ep.max(axis=0) - ep.min(axis=0)).max() > 32768
    elif case == "ties":             # uniform transitions and emissions: every predecessor ties
        lpi = np.full(S, -6000, np.int32)
        lA = np.full((S, S), -6000, np.int32)
        lE = np.full((S, 4), -2000, np.int32)
    elif case == "odd_ragged":       # S = 23 (inactive lanes), odd n, T = 0 and T = 1 rows
        seqs[0] = seqs[0][:0]
        seqs[7] = seqs[7][:1]
        seqs.append(seqs[4][:1])
    _viterbi_check(dp, orc, lpi, lA, lE, seqs, variant, tb=(case != "score_only"))


def test_hmm_config3_sampled(dp, orc, capsys):
    """BASELINE config 3 at full size (10k x 1000, S = 64), sampled against the oracle."""
    d = dpgen.config3_hmm()
    seqs = d["seqs"]
    n, T = seqs.shape
    off = np.arange(n + 1, dtype=np.int64) * T
    cat = seqs.reshape(-1)
    pf = dp.Plan(dp.HMM_FORWARD, T, pi=d["pi"], A=d["A"], E=d["E"])
    ll = host(pf.solve_batch(cuda(cat), cuda(off), max_len_a=T))
    pv = dp.Plan(dp.HMM_VITERBI, T, lpi=d["lpi"], lA=d["lA"], lE=d["lE"], want_traceback=True)
    vs = host(pv.solve_batch(cuda(cat), cuda(off), max_len_a=T))
    assert pv.last_variant == "k_viterbi16"
    out, ln, _ = pv.traceback(0, n, T, coords=False)
    out = host(out)
    ids = np.random.default_rng(140).choice(n, size=24, replace=False)
    sub_off = np.arange(len(ids) + 1, dtype=np.int64) * T
    sub = seqs[ids].reshape(-1)
    want = orc.forward_batch(sub, sub_off, *(d[k].astype(np.float64) for k in ("pi", "A", "E")), threads=THREADS)
    dl, rel = forward_errors(ll[ids], want, "config 3 (S=64, T=1000)", capsys)
    assert rel.max() <= 1e-5
    for k, q in enumerate(ids):
        v, path = orc.viterbi(seqs[q], d["lpi"], d["lA"], d["lE"])
        assert vs[q] == v and (out[q] == path).all()


# ----------------------------------------------------------------------------- boundary
def test_errors_and_empty(dp):
    import torch
    sig = dpgen.blosum62()
    plan = dp.Plan(dp.SW_LINEAR, 16, 16, sigma=sig, gap=4)
    z = torch.zeros(1, dtype=torch.int64, device="cuda")
    e = torch.zeros(0, dtype=torch.uint8, device="cuda")
    out = plan.solve_batch(e, z, e, z, max_len_a=0, max_len_b=0)
    assert out.numel() == 0
    a = cuda(np.zeros(20, np.uint8))
    off = cuda(np.array([0, 20], np.int64))
    with pytest.raises(dp.DPError) as ex:
        plan.solve_batch(a, off, a, off, max_len_a=20, max_len_b=20)
    assert ex.value.code == 4   # DP_E_TOO_LARGE
    with pytest.raises(dp.DPError) as ex:
        plan.traceback(0, 1, 64)
    assert ex.value.code == 7   # DP_E_NO_TRACEBACK
    with pytest.raises(dp.DPError) as ex:
        dp.Plan(dp.HMM_FORWARD, 10, pi=np.ones(2, np.float32), A=np.ones((2, 2), np.float32),
                E=np.ones((2, 4), np.float32), want_traceback=True)
    assert ex.value.code == 3   # forward has no traceback
    with pytest.raises(dp.DPError) as ex:
        dp.Plan(dp.SW_LINEAR, 16, 16, sigma=sig, gap=4, user_coeff=(1, -1))
    assert ex.value.code == 2   # user schedule violates eq.(3)
    plan.close()


def test_dp_solve_single_problem(dp, orc):
    """dp_solve (one problem, device buffers): each kind against the oracle, and many calls on
    two streams in flight at once (the per-call offset slots must not be shared)."""
    import torch
    sig = dpgen.blosum62()
    g = np.random.default_rng(151)
    pairs = [(g.integers(0, 20, int(g.integers(1, 300))).astype(np.uint8),
              g.integers(0, 20, int(g.integers(1, 300))).astype(np.uint8)) for _ in range(40)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    with dp.Plan(dp.SW_LINEAR, 300, 300, sigma=sig, gap=4) as p:
        outs = []
        for k, (a, b) in enumerate(pairs):
            st = streams[k % 2]
            with torch.cuda.stream(st):
                ta, tb = cuda(a), cuda(b)
                outs.append((p.solve(ta, tb, stream=st), ta, tb))
        torch.cuda.synchronize()
        for (o, _, _), (a, b) in zip(outs, pairs):
            assert int(o[0]) == orc.sw(a, b, sig, 4)[0]
    # retained state belongs to the plan's most recent solve: traceback after dp_solve
    a, b = pairs[-1]
    with dp.Plan(dp.SW_LINEAR, 300, 300, sigma=sig, gap=4, want_traceback=True) as p:
        p.solve(cuda(a), cuda(b))
        out, ln, co = p.traceback(0, 1, 600)
        ops, c = orc.sw_traceback(a, b, sig, 4)
        assert bytes(host(out[0, :int(ln[0])])).decode() == ops and tuple(host(co[0])) == c
    x = dpgen.config1_rna64()
    with dp.Plan(dp.NUSSINOV, 64, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
        assert int(p.solve(cuda(x))[0]) == orc.nussinov(x, dpgen.rna_pair_mask(), 3)
    s, t = dpgen.encode("kitten", dpgen.EN), dpgen.encode("sitting", dpgen.EN)
    with dp.Plan(dp.EDIT, 6, 7, alphabet_size=26) as p:
        assert int(p.solve(cuda(s), cuda(t))[0]) == 3
    with pytest.raises(dp.DPError) as ex:
        with dp.Plan(dp.EDIT, 6, 7, alphabet_size=26) as p:
            p.solve(cuda(np.zeros(9, np.uint8)), cuda(t))
    assert ex.value.code == 4


def test_plan_rejects_what_the_kernels_cannot_run(dp):
    """Plan creation checks the kernels' shared-memory needs against the device limit
    (DP_E_TOO_LARGE at dp_plan_create, not DP_E_CUDA at solve time)."""
    sig = dpgen.blosum62()
    for kind, kw in ((dp.SW_AFFINE, dict(gap_open=11, gap_extend=1)), (dp.EDIT, {})):
        with pytest.raises(dp.DPError) as ex:
            dp.Plan(kind, 200_000, 200_000, sigma=sig if kind == dp.SW_AFFINE else None, alphabet_size=24,
                    want_traceback=False, **kw)
        assert ex.value.code == 4


def test_host_entry_point(dp, orc):
    """dp_solve_batch_host (H2D + solve + traceback + D2H) equals the device path."""
    g = np.random.default_rng(150)
    sig = dpgen.blosum62()
    a, (a_cat, a_off) = rand_batch(g, 50, 1, 256, 20)
    b, (b_cat, b_off) = rand_batch(g, 50, 1, 256, 20)
    plan = dp.Plan(dp.SW_LINEAR, 256, 256, sigma=sig, gap=4, want_traceback=True)
    sc, tb, tbl, tbc = plan.solve_batch_host(a_cat, a_off, b_cat, b_off, tb_stride=512)
    for q in range(50):
        s0, _, _ = orc.sw(a[q], b[q], sig, 4)
        ops, co = orc.sw_traceback(a[q], b[q], sig, 4)
        assert sc[q] == s0 and bytes(tb[q, :tbl[q]]).decode() == ops and tuple(tbc[q]) == co
    plan.close()


def test_host_entry_point_chunked(dp, orc):
    """A batch large enough for several chunks (packed SW alternates two compute streams and two
    retained-state buffers): the host path equals the device path everywhere and the oracle on a
    sample spread over the chunks."""
    import torch
    n = 70_000
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n)
    sig = dpgen.blosum62()
    plan = dp.Plan(dp.SW_LINEAR, 256, 256, sigma=sig, gap=dpgen.SW_GAP, want_traceback=True)
    sc, tb, tbl, tbc = plan.solve_batch_host(a_cat, a_off, b_cat, b_off, tb_stride=513)
    dsc = host(plan.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=256, max_len_b=256))
    out, ln, co = plan.traceback(0, n, 513)
    torch.cuda.synchronize()
    assert (sc == dsc).all()
    assert (tbl == host(ln)).all() and (tbc == host(co)).all()
    used = np.arange(513)[None, :] < tbl[:, None]  # bytes past a row's length are unspecified
    assert (tb[used] == host(out)[used]).all()
    for q in range(0, n, 1750):
        x, y = a_cat[a_off[q]:a_off[q + 1]], b_cat[b_off[q]:b_off[q + 1]]
        ops, c = orc.sw_traceback(x, y, sig, dpgen.SW_GAP)
        assert sc[q] == orc.sw(x, y, sig, dpgen.SW_GAP)[0] and bytes(tb[q, :tbl[q]]).decode() == ops
    plan.close()


def test_host_entry_point_affine_chunked(dp, orc):
    """The packed affine kernel through the host entry point in several chunks of odd size (a
    chunk's last warp carries one problem): equal to the device path everywhere, the oracle on a
    sample spread over the chunks."""
    import torch
    n = 40_001
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(n)
    sig = dpgen.blosum62()
    plan = dp.Plan(dp.SW_AFFINE, 256, 256, sigma=sig, alphabet_size=24, want_traceback=True, gap_open=11,
                   gap_extend=1)
    sc, tb, tbl, tbc = plan.solve_batch_host(a_cat, a_off, b_cat, b_off, tb_stride=513)
    dsc = host(plan.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=256, max_len_b=256))
    assert plan.last_variant == "k_affine16"
    out, ln, co = plan.traceback(0, n, 513)
    torch.cuda.synchronize()
    assert (sc == dsc).all()
    assert (tbl == host(ln)).all() and (tbc == host(co)).all()
    used = np.arange(513)[None, :] < tbl[:, None]
    assert (tb[used] == host(out)[used]).all()
    for q in list(range(0, n, 2500)) + [n - 1]:
        x, y = a_cat[a_off[q]:a_off[q + 1]], b_cat[b_off[q]:b_off[q + 1]]
        ops, c = orc.sw_affine_traceback(x, y, sig, 11, 1)
        assert sc[q] == orc.sw_affine(x, y, sig, 11, 1)[0] and bytes(tb[q, :tbl[q]]).decode() == ops, q
    plan.close()


def test_host_entry_point_viterbi_chunked(dp, orc):
    """The s16x2 Viterbi through the host entry point on a batch big enough for three chunks:
    scores and paths equal to the device path, the oracle on a sample spread over the chunks; an
    odd batch so a chunk's last warp carries one sequence."""
    import torch
    h = dpgen.config3_hmm(n_seqs=70_001, T=100)
    cat, off = dpgen.pack(h["seqs"])
    n = len(off) - 1
    plan = dp.Plan(dp.HMM_VITERBI, 100, lpi=h["lpi"], lA=h["lA"], lE=h["lE"], want_traceback=True)
    sc, tb, tbl, _ = plan.solve_batch_host(cat, off, tb_stride=100)
    dsc = host(plan.solve_batch(cuda(cat), cuda(off)))
    assert plan.last_variant == "k_viterbi16"
    out, ln, _ = plan.traceback(0, n, 100, coords=False)
    torch.cuda.synchronize()
    out, ln = host(out), host(ln)
    assert (sc == dsc).all() and (tbl == ln).all() and (tb == out).all()
    for q in list(range(0, n, 5000)) + [n - 1]:
        v, path = orc.viterbi(h["seqs"][q], h["lpi"], h["lA"], h["lE"])
        assert sc[q] == v and (tb[q] == path).all(), q
    plan.close()


# ----------------------------------------------------------------------------- §4.7 diagonal-only
def run_diag(dp, a_seqs, b_seqs, **kw):
    a_cat, a_off = dpgen.pack(a_seqs)
    b_cat, b_off = dpgen.pack(b_seqs)
    la = max((len(s) for s in a_seqs), default=0)
    lb = max((len(s) for s in b_seqs), default=0)
    with dp.Plan(dp.DIAG_LCS, max(la, 1), max(lb, 1), **kw) as plan:
        return host(plan.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=la, max_len_b=lb))


@pytest.mark.parametrize("force,asz", [(None, 0), ("0", 0), ("1", 0), (None, 4), ("0", 4), ("1", 4)])
def test_diag_mixed_shapes(dp, orc, monkeypatch, force, asz):
    """Ragged tall and wide pairs, empty sides, length 1: bit-exact against the oracle under the
    run-time schedule choice and under each candidate forced (the result cannot depend on it),
    with the alphabet unknown (one cell per register) and given (asz = 4: two per register)."""
    if force is not None:
        monkeypatch.setenv("DP_DIAG_FORCE", force)
    g = np.random.default_rng(800)
    a = [g.integers(0, 4, int(g.integers(0, 700))).astype(np.uint8) for _ in range(150)]
    b = [g.integers(0, 4, int(g.integers(0, 700))).astype(np.uint8) for _ in range(150)]
    a[:4] = [np.zeros(0, np.uint8), np.ones(1, np.uint8), a[2], np.arange(300, dtype=np.uint8) % 4]
    b[:4] = [b[0], np.zeros(0, np.uint8), a[2].copy(), np.arange(5, 900, dtype=np.uint8) % 4]
    a[5], b[5] = np.full(257, 2, np.uint8), np.full(33, 2, np.uint8)   # a run: the answer is 33
    a[6], b[6] = g.integers(0, 4, 60).astype(np.uint8), g.integers(0, 4, 4500).astype(np.uint8)  # > 4096: smem path
    a[7], b[7] = g.integers(0, 2, 5000).astype(np.uint8), g.integers(0, 2, 3000).astype(np.uint8)
    got = run_diag(dp, a, b, alphabet_size=asz)
    want = np.array([orc.lcsubstr(x, y) for x, y in zip(a, b)])
    assert (got == want).all()
    assert got[5] == 33


def test_diag_workload_sampled(dp, orc):
    """The bench workload's distribution (log-uniform 32..4096 per side), first 120 pairs."""
    a_cat, a_off, b_cat, b_off = dpgen.diag_pairs(120)
    la, lb = int(np.diff(a_off).max()), int(np.diff(b_off).max())
    want = orc.lcsubstr_batch(a_cat, a_off, b_cat, b_off, threads=THREADS)
    for asz in (0, 4):
        with dp.Plan(dp.DIAG_LCS, la, lb, alphabet_size=asz) as plan:
            got = host(plan.solve_batch(cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off), max_len_a=la,
                                        max_len_b=lb))
        assert (got == want).all(), asz


def test_diag_plan_schedules(dp):
    """§4.7: the plan accepts a user schedule only if it is one of the conditional candidates
    (L326, L386-L388); no traceback is retained for this kind."""
    with dp.Plan(dp.DIAG_LCS, 100, 50) as p:
        assert p.schedule()["a"] in ((0, 1), (1, 0))
    for uc in ((1, 0), (0, 1)):
        with dp.Plan(dp.DIAG_LCS, 100, 50, user_coeff=uc) as p:
            assert p.schedule()["a"] == uc
    for uc, code in (((2, 1), 3), ((1, -1), 2)):      # valid but never minimal / invalid
        with pytest.raises(dp.DPError) as e:
            dp.Plan(dp.DIAG_LCS, 100, 50, user_coeff=uc)
        assert e.value.code == code
    with pytest.raises(dp.DPError) as e:
        dp.Plan(dp.DIAG_LCS, 100, 50, want_traceback=True)
    assert e.value.code == 3


# ----------------------------------------------------------------------------- profile HMM (NEXT 3)
@pytest.mark.parametrize("L,maxT", [(1, 12), (7, 40), (100, 160), (256, 300), (300, 420), (700, 800)])
def test_profile_forward_random(dp, orc, L, maxT, capsys):
    """Profile-HMM forward: random profiles (one strip, several strips of 256 rows, ragged last
    strip), sequences sampled from the model plus random ones, empty and length-1 sequences;
    log P within relative 1e-5 of the oracle's generic silent-state forward (fp64)."""
    g = np.random.default_rng(900 + L)
    K = 20
    tr, eM, eI = dpgen.profile_hmm_params(g, L, K)
    tr32, eM32, eI32 = (v.astype(np.float32) for v in (tr, eM, eI))
    seqs = dpgen.sample_profile(g, tr, eM, eI, 24, max_len=maxT)
    seqs += [g.integers(0, K, size=int(g.integers(0, maxT + 1))).astype(np.uint8) for _ in range(6)]
    seqs += [np.zeros(0, np.uint8), np.zeros(1, np.uint8)]
    cat, off = dpgen.pack(seqs)
    ml = max(len(s) for s in seqs)
    with dp.Plan(dp.PROFILE_FORWARD, ml, trans=tr32, emit_m=eM32, emit_i=eI32) as p:
        assert p.schedule()["a"] == (1, 1)
        ll = host(p.solve_batch(cuda(cat), cuda(off), max_len_a=ml))
    want = orc.profile_forward_batch(cat, off, L, tr32.astype(np.float64), eM32.astype(np.float64),
                                     eI32.astype(np.float64), threads=THREADS)
    fin = np.isfinite(want)
    assert (np.isfinite(ll) == fin).all()
    dl, rel = forward_errors(ll[fin], want[fin], f"profile L={L}", capsys)
    assert rel.max() <= 1e-5


def test_profile_workload_sampled(dp, orc, capsys):
    """The bench workload (L = 256, 13,355 sequences sampled from the profile) at full size in the
    bench's launch; a seeded sample against the oracle."""
    d = dpgen.profile_hmm_workload()
    cat, off = d["cat"], d["off"]
    ml = int(np.diff(off).max())
    with dp.Plan(dp.PROFILE_FORWARD, ml, **d["model"]) as p:
        ll = host(p.solve_batch(cuda(cat), cuda(off), max_len_a=ml))
    ids = np.sort(np.random.default_rng(901).choice(len(off) - 1, 48, replace=False))
    sub_cat, sub_off = dpgen.pack([cat[off[q]:off[q + 1]] for q in ids])
    want = orc.profile_forward_batch(sub_cat, sub_off, d["L"], **d["model64"], threads=THREADS)
    dl, rel = forward_errors(ll[ids], want, "profile workload (L=256)", capsys)
    assert rel.max() <= 1e-5
    assert np.isfinite(ll).all()


@pytest.mark.parametrize("count", [5, 120, 600])
def test_nussinov_short_batches(dp, orc, count):
    """Short sequences (lengths 0..128, the cell-level and tiled paths' boundary region), a few and
    many problems per batch, both hairpins; scores and canonical dot-brackets bit-exact."""
    g = np.random.default_rng(160 + count)
    for h, pm in ((3, dpgen.rna_pair_mask()), (0, dpgen.rna_pair_mask(gu=False))):
        seqs, _ = rand_batch(g, count, 0, 128, 4)
        seqs[0] = g.integers(0, 4, size=128).astype(np.uint8)
        r = run_nuss(dp, seqs, h=h, pm=pm)
        for q, x in enumerate(seqs):
            if count > 120 and q % 7:
                continue
            assert (r["scores"][q], r["db"][q]) == orc.nussinov_traceback(x, pm, h), (q, len(x))


# ----------------------------------------------------------------------------- determinism
def test_repeat_determinism(dp):
    """Race detection by repetition (compute-sanitizer is closed on this GPU pool): the
    warp-synchronous kernels with shared-memory hand-offs and the mbarrier-pipelined tcgen05
    forward give bit-identical outputs when the same plan runs the same batch again, at sizes that
    fill the GPU (several waves, both halves of every packed register, multi-strip columns)."""
    import torch
    sig = dpgen.blosum62()
    a_cat, a_off, b_cat, b_off = dpgen.config2_protein_pairs(20_001)
    A = (cuda(a_cat), cuda(a_off), cuda(b_cat), cuda(b_off))

    def used(out, ln):  # bytes past a row's length are unspecified (dp.h): zero them
        mask = torch.arange(out.shape[1], device=out.device)[None, :] < ln[:, None].long()
        return torch.where(mask, out, torch.zeros_like(out))

    def twice(plan, fn):
        r1 = fn(plan)
        torch.cuda.synchronize()
        r2 = fn(plan)
        torch.cuda.synchronize()
        for k, (x, y) in enumerate(zip(r1, r2)):
            assert torch.equal(x, y), k

    def align(p):
        sc = p.solve_batch(*A, max_len_a=256, max_len_b=256).clone()
        out, ln, co = p.traceback(0, 20_001, 513)
        return sc, used(out, ln), ln.clone(), co.clone()

    with dp.Plan(dp.SW_LINEAR, 256, 256, sigma=sig, gap=dpgen.SW_GAP, want_traceback=True) as p:
        twice(p, align)
        assert p.last_variant == "k_sw16"
    with dp.Plan(dp.SW_AFFINE, 256, 256, sigma=sig, alphabet_size=24, want_traceback=True, gap_open=11,
                 gap_extend=1) as p:
        twice(p, align)
        assert p.last_variant == "k_affine16"
    h = dpgen.config3_hmm(n_seqs=2_000, T=400)
    cat, off = dpgen.pack(h["seqs"])
    X = (cuda(cat), cuda(off))
    with dp.Plan(dp.HMM_FORWARD, 400, pi=h["pi"], A=h["A"], E=h["E"]) as p:
        twice(p, lambda q: (q.solve_batch(*X).clone(),))
    with dp.Plan(dp.HMM_VITERBI, 400, lpi=h["lpi"], lA=h["lA"], lE=h["lE"], want_traceback=True) as p:
        def vit(q):
            sc = q.solve_batch(*X).clone()
            out, ln, _ = q.traceback(0, 2_000, 400, coords=False)
            return sc, used(out, ln), ln.clone()
        twice(p, vit)
        assert p.last_variant == "k_viterbi16"
    rna = dpgen.config5_rna_batch(n_seqs=3_000)
    R = (cuda(rna[0]), cuda(rna[1]))
    with dp.Plan(dp.NUSSINOV, 512, pair_mask=dpgen.rna_pair_mask(), min_hairpin=3, want_traceback=True) as p:
        def nuss(q):
            sc = q.solve_batch(*R, max_len_a=512).clone()
            out, ln, _ = q.traceback(0, 3_000, 512, coords=False)
            return sc, used(out, ln), ln.clone()
        twice(p, nuss)
