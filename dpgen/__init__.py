"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NONE of the method's arithmetic (no recursion, no schedule,
no scoring). It only draws sequences and model parameters and writes down the
fixed scoring tables the workloads name, so both sides of every parity check
see byte-identical problem definitions (task ③: "only the seeded input
generators serve both, from a module of their own").

Workload recipe (SURVEY.md §8(d) D1–D5; DESIGN.md §2 "Inputs"):
  * master seed 20120611 + config index, numpy PCG64;
  * RNA  : bases i.i.d. uniform over ACGU (codes 0..3);
  * protein: residues i.i.d. uniform over the 20 standard amino acids (codes 0..19
    in the BLOSUM62 order ARNDCQEGHILKMFPSTWYV; BZX* = 20..23 exist in the table);
  * HMM  : S=64 states, DNA alphabet (ACGT), rows of A, E and pi ~ Dirichlet(1),
    sequences sampled from the model itself;
  * Viterbi log-scores: int32 milli-bits round(1000*log2 p), computed once here.
"""
from __future__ import annotations

import numpy as np

MASTER_SEED = 20120611

RNA = "ACGU"
DNA = "ACGT"
PROTEIN = "ARNDCQEGHILKMFPSTWYVBZX*"
EN = "abcdefghijklmnopqrstuvwxyz"  # Fig.7's `en` alphabet, used by the edit-distance mode

# NCBI BLOSUM62 in the order of PROTEIN (a published constant; scoring input of
# the substitution-matrix extension, §5.1; matrix named by
# the decisions register SURVEY.md App. B).
_B62_ROWS = """
 4 -1 -2 -2  0 -1 -1  0 -2 -1 -1 -1 -1 -2 -1  1  0 -3 -2  0 -2 -1  0 -4
-1  5  0 -2 -3  1  0 -2  0 -3 -2  2 -1 -3 -2 -1 -1 -3 -2 -3 -1  0 -1 -4
-2  0  6  1 -3  0  0  0  1 -3 -3  0 -2 -3 -2  1  0 -4 -2 -3  3  0 -1 -4
-2 -2  1  6 -3  0  2 -1 -1 -3 -4 -1 -3 -3 -1  0 -1 -4 -3 -3  4  1 -1 -4
 0 -3 -3 -3  9 -3 -4 -3 -3 -1 -1 -3 -1 -2 -3 -1 -1 -2 -2 -1 -3 -3 -2 -4
-1  1  0  0 -3  5  2 -2  0 -3 -2  1  0 -3 -1  0 -1 -2 -1 -2  0  3 -1 -4
-1  0  0  2 -4  2  5 -2  0 -3 -3  1 -2 -3 -1  0 -1 -3 -2 -2  1  4 -1 -4
 0 -2  0 -1 -3 -2 -2  6 -2 -4 -4 -2 -3 -3 -2  0 -2 -2 -3 -3 -1 -2 -1 -4
-2  0  1 -1 -3  0  0 -2  8 -3 -3 -1 -2 -1 -2 -1 -2 -2  2 -3  0  0 -1 -4
-1 -3 -3 -3 -1 -3 -3 -4 -3  4  2 -3  1  0 -3 -2 -1 -3 -1  3 -3 -3 -1 -4
-1 -2 -3 -4 -1 -2 -3 -4 -3  2  4 -2  2  0 -3 -2 -1 -2 -1  1 -4 -3 -1 -4
-1  2  0 -1 -3  1  1 -2 -1 -3 -2  5 -1 -3 -1  0 -1 -3 -2 -2  0  1 -1 -4
-1 -1 -2 -3 -1  0 -2 -3 -2  1  2 -1  5  0 -2 -1 -1 -1 -1  1 -3 -1 -1 -4
-2 -3 -3 -3 -2 -3 -3 -3 -1  0  0 -3  0  6 -4 -2 -2  1  3 -1 -3 -3 -1 -4
-1 -2 -2 -1 -3 -1 -1 -2 -2 -3 -3 -1 -2 -4  7 -1 -1 -4 -3 -2 -2 -1 -2 -4
 1 -1  1  0 -1  0  0  0 -1 -2 -2  0 -1 -2 -1  4  1 -3 -2 -2  0  0  0 -4
 0 -1  0 -1 -1 -1 -1 -2 -2 -1 -1 -1 -1 -2 -1  1  5 -2 -2  0 -1 -1  0 -4
-3 -3 -4 -4 -2 -2 -3 -2 -2 -3 -2 -3 -1  1 -4 -3 -2 11  2 -3 -4 -3 -2 -4
-2 -2 -2 -3 -2 -1 -2 -3  2 -1 -1 -2 -1  3 -3 -2 -2  2  7 -1 -3 -2 -1 -4
 0 -3 -3 -3 -1 -2 -2 -3 -3  3  1 -2  1 -1 -2 -2  0 -3 -1  4 -3 -2 -1 -4
-2 -1  3  4 -3  0  1 -1  0 -3 -4  0 -3 -3 -2  0 -1 -4 -3 -3  4  1 -1 -4
-1  0  0  1 -3  3  4 -2  0 -3 -3  1 -1 -3 -1  0 -1 -3 -2 -2  1  4 -1 -4
 0 -1 -1 -1 -2 -1 -1 -1 -1 -1 -1 -1 -1 -1 -2  0  0 -2 -1 -1 -1 -1 -1 -4
-4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4 -4  1
"""

SW_GAP = 4          # linear gap penalty g (BLOSUM62's '*' score)
SW_GAP_OPEN, SW_GAP_EXTEND = 11, 1  # affine SW (NEXT rank 1): gap of length k costs 11 + k (NCBI BLOSUM62 default)
NUSS_HAIRPIN = 3    # minimum hairpin loop h
HMM_STATES = 64
MILLIBIT_FLOOR = -100000  # score used for p == 0 (2^-100); Dirichlet(1) draws never hit it in practice


def rng(config_index: int, extra: int = 0) -> np.random.Generator:
    """numpy PCG64 seeded with 20120611 + config index (+ extra sub-stream)."""
    return np.random.Generator(np.random.PCG64(MASTER_SEED + config_index + 1000003 * extra))


def blosum62() -> np.ndarray:
    m = np.array([int(v) for v in _B62_ROWS.split()], dtype=np.int8).reshape(24, 24)
    return m


def rna_pair_mask(gu: bool = True) -> np.ndarray:
    """4x4 uint8 mask over ACGU: 1 where the two bases may pair (WC + optional GU wobble)."""
    m = np.zeros((4, 4), dtype=np.uint8)
    for a, b in ("AU", "UA", "GC", "CG") + (("GU", "UG") if gu else ()):
        m[RNA.index(a), RNA.index(b)] = 1
    return m


def encode(s: str, alphabet: str) -> np.ndarray:
    return np.frombuffer(bytes(alphabet.index(c) for c in s), dtype=np.uint8).copy()


def decode(codes, alphabet: str) -> str:
    return "".join(alphabet[int(c)] for c in codes)


def random_seq(g: np.random.Generator, n: int, k: int) -> np.ndarray:
    return g.integers(0, k, size=n, dtype=np.uint8)


def pack(seqs) -> tuple[np.ndarray, np.ndarray]:
    """Concatenate uint8 sequences; returns (cat, offsets[n+1] int64)."""
    lens = np.array([len(s) for s in seqs], dtype=np.int64)
    off = np.zeros(len(seqs) + 1, dtype=np.int64)
    np.cumsum(lens, out=off[1:])
    cat = np.concatenate([np.asarray(s, dtype=np.uint8) for s in seqs]) if len(seqs) else np.zeros(0, np.uint8)
    return cat, off


def unpack(cat: np.ndarray, off: np.ndarray, i: int) -> np.ndarray:
    return cat[off[i]:off[i + 1]]


# ----------------------------------------------------------------------------- configs
def config1_rna64() -> np.ndarray:
    """D1: one 64-nt RNA, seed 20120611+1."""
    return random_seq(rng(1), 64, 4)


def config2_protein_pairs(n_pairs: int = 100_000, length: int = 256, first: int = 0):
    """D2: n_pairs protein pairs of the given length, seed 20120611+2.

    Returns (a_cat, a_off, b_cat, b_off): pairs [first, first + n_pairs) of the
    stream drawn for first + n_pairs pairs (all a rows, then all b rows). The a
    sequences are prefix-consistent across totals, the b sequences are NOT: a
    shard of a larger batch must be sliced from that batch (bench.py does)."""
    g = rng(2)
    total = first + n_pairs
    a = g.integers(0, 20, size=(total, length), dtype=np.uint8)
    b = g.integers(0, 20, size=(total, length), dtype=np.uint8)
    a = a[first:]
    b = b[first:]
    off = np.arange(n_pairs + 1, dtype=np.int64) * length
    return a.reshape(-1).copy(), off, b.reshape(-1).copy(), off.copy()


def diag_pairs(n_pairs: int = 20_000, lo: int = 32, hi: int = 4096, first: int = 0):
    """Mixed-shape batch for the diagonal-only recurrence (§4.7 example):
    DNA pairs (codes 0..3) whose lengths |a|, |b| are drawn independently and log-uniformly
    from [lo, hi], so about half the pairs are taller than wide; seed 20120611+8.
    Returns (a_cat, a_off, b_cat, b_off); `first` skips that many pairs of the stream."""
    g = rng(8)
    total = first + n_pairs
    la = np.exp(g.uniform(np.log(lo), np.log(hi + 1), total)).astype(np.int64).clip(lo, hi)
    lb = np.exp(g.uniform(np.log(lo), np.log(hi + 1), total)).astype(np.int64).clip(lo, hi)
    a = g.integers(0, 4, int(la.sum()), dtype=np.uint8)
    b = g.integers(0, 4, int(lb.sum()), dtype=np.uint8)
    ao = np.concatenate([[0], np.cumsum(la)]).astype(np.int64)
    bo = np.concatenate([[0], np.cumsum(lb)]).astype(np.int64)
    a, b = a[ao[first]:], b[bo[first]:]
    ao, bo = ao[first:] - ao[first], bo[first:] - bo[first]
    return a.copy(), ao, b.copy(), bo


def short_protein_pairs(n_pairs: int = 1_000_000, lo: int = 8, hi: int = 64, first: int = 0):
    """Short-pair batch for the inter-task kernel (the hybrid's short side;
    PAPER.md §6.1): protein pairs whose lengths |a|, |b| are i.i.d. uniform integers in
    [lo, hi], residues i.i.d. uniform over the 20 standard amino acids; seed 20120611+11.
    Returns (a_cat, a_off, b_cat, b_off); `first` skips that many pairs of the stream."""
    g = rng(11)
    total = first + n_pairs
    la = g.integers(lo, hi + 1, total, dtype=np.int64)
    lb = g.integers(lo, hi + 1, total, dtype=np.int64)
    a = g.integers(0, 20, int(la.sum()), dtype=np.uint8)
    b = g.integers(0, 20, int(lb.sum()), dtype=np.uint8)
    ao = np.concatenate([[0], np.cumsum(la)]).astype(np.int64)
    bo = np.concatenate([[0], np.cumsum(lb)]).astype(np.int64)
    a, b = a[ao[first]:], b[bo[first]:]
    ao, bo = ao[first:] - ao[first], bo[first:] - bo[first]
    return a.copy(), ao, b.copy(), bo


def hmm_params(g: np.random.Generator, S: int = HMM_STATES, K: int = 4):
    """Rows of pi (1xS), A (SxS), E (SxK) ~ Dirichlet(1), float64."""
    pi = g.dirichlet(np.ones(S))
    A = g.dirichlet(np.ones(S), size=S)
    E = g.dirichlet(np.ones(K), size=S)
    return pi, A, E


def sample_hmm(g: np.random.Generator, pi, A, E, n: int, T: int) -> np.ndarray:
    """n sequences of length T drawn from the HMM (states by pi then A, symbols by E)."""
    S = len(pi)
    cA = np.cumsum(A, axis=1)
    cE = np.cumsum(E, axis=1)
    cpi = np.cumsum(pi)
    out = np.empty((n, T), dtype=np.uint8)
    if T == 0 or n == 0:
        return out
    st = np.minimum(np.searchsorted(cpi, g.random(n), side="right"), S - 1)
    for t in range(T):
        u = g.random(n)
        sym = (cE[st] <= u[:, None]).sum(axis=1)
        out[:, t] = np.minimum(sym, E.shape[1] - 1)
        u = g.random(n)
        st = np.minimum((cA[st] <= u[:, None]).sum(axis=1), S - 1)
    return out


def millibits(p) -> np.ndarray:
    """int32 round(1000*log2 p); p == 0 -> MILLIBIT_FLOOR. Computed once, here only."""
    p = np.asarray(p, dtype=np.float64)
    with np.errstate(divide="ignore"):
        v = np.where(p > 0, np.rint(1000.0 * np.log2(np.where(p > 0, p, 1.0))), MILLIBIT_FLOOR)
    return np.maximum(v, MILLIBIT_FLOOR).astype(np.int32)


def config3_hmm(n_seqs: int = 10_000, T: int = 1000, S: int = HMM_STATES):
    """D3: 64-state dense HMM over DNA, params seed +3, sequences seed +4.

    Returns dict with fp32 probabilities (pi, A, E) — the values both sides use —
    their int32 milli-bit scores (lpi, lA, lE), and sequences (n_seqs x T uint8)."""
    pi, A, E = hmm_params(rng(3), S, 4)
    pi32, A32, E32 = (x.astype(np.float32) for x in (pi, A, E))
    seqs = sample_hmm(rng(4), pi, A, E, n_seqs, T)
    return {
        "pi": pi32, "A": A32, "E": E32,
        "lpi": millibits(pi32), "lA": millibits(A32), "lE": millibits(E32),
        "seqs": seqs, "S": S, "K": 4,
    }


def config4_rna8192(n: int = 8192) -> np.ndarray:
    """D4: one RNA of length n (8192), seed 20120611+5."""
    return random_seq(rng(5), n, 4)


def mid_rna_batch(n_seqs: int = 16, lo: int = 482, hi: int = 1024):
    """Mid-length Nussinov batch (n between the batch kernel's and the
    grid kernel's regimes): n_seqs RNAs, lengths i.i.d. uniform integers in [lo, hi], bases
    i.i.d. uniform over ACGU; seed 20120611+12. Returns (cat, off)."""
    g = rng(12)
    lens = g.integers(lo, hi + 1, n_seqs, dtype=np.int64)
    return pack([random_seq(g, int(l), 4) for l in lens])


def config5_lengths(n_seqs: int = 1_000_000, lo: int = 128, hi: int = 512) -> np.ndarray:
    return rng(6).integers(lo, hi + 1, size=n_seqs, dtype=np.int64)


def config5_rna_batch(n_seqs: int = 1_000_000, lo: int = 128, hi: int = 512, ids=None):
    """D5: RNAs with lengths i.i.d. uniform in [lo, hi], bases i.i.d. ACGU, seed +6.

    Sequence i's bases come from its own sub-stream (seed +6, extra=i+1) so any
    subset `ids` is generated without drawing the whole million."""
    lens = config5_lengths(n_seqs, lo, hi)
    if ids is None:
        g = rng(6, extra=1)
        cat = g.integers(0, 4, size=int(lens.sum()), dtype=np.uint8)
        off = np.zeros(n_seqs + 1, dtype=np.int64)
        np.cumsum(lens, out=off[1:])
        return cat, off
    seqs = []
    full_off = np.zeros(n_seqs + 1, dtype=np.int64)
    np.cumsum(lens, out=full_off[1:])
    g = rng(6, extra=1)
    # regenerate the full stream lazily in chunks only up to the largest id needed
    need = int(full_off[max(ids) + 1])
    cat = g.integers(0, 4, size=need, dtype=np.uint8)
    for i in ids:
        seqs.append(cat[full_off[i]:full_off[i + 1]])
    return pack(seqs)


def config5_sample_ids(n_seqs: int = 1_000_000, k: int = 10_000) -> np.ndarray:
    """The fixed 1% subset (seed +7) used for the on-box oracle timing."""
    return np.sort(rng(7).choice(n_seqs, size=k, replace=False))


# ----------------------------------------------------------------------------- profile HMM
# Transition slots of position j (0..L): from state X_j, X in (M, I, D) (M_0 is the begin state B,
# D_0 does not exist), to (M_{j+1}, I_j, D_{j+1}) (M_{L+1} is the end state E, D_{L+1} does not
# exist). tr[j][3 * from + to], from/to order (M, I, D) / (M_{j+1}, I_j, D_{j+1}).
PROFILE_FROM = ("M", "I", "D")
PROFILE_TO = ("M+1", "I", "D+1")


def profile_hmm_params(g: np.random.Generator, L: int, K: int = 20):
    """A Plan7-like profile HMM of L match positions (Durbin et al. ch. 5, the paper's ref [3];
    PAPER.md §6.3), all nine transitions per position (M/I/D -> M/I/D):
      tr : (L+1) x 9 float64, rows from M ~ Dir(90, 5, 5), from I ~ Dir(60, 35, 5),
           from D ~ Dir(65, 5, 30); D_0 does not exist (its row is 0); at j = L the "to D_{L+1}"
           slot is 0 and each row is renormalised over (E, I_L);
      eM : (L+1) x K match emissions ~ Dir(0.4) (row 0 unused, zeros);
      eI : (L+1) x K insert emissions ~ Dir(20) (close to background)."""
    tr = np.zeros((L + 1, 9))
    for j in range(L + 1):
        tr[j, 0:3] = g.dirichlet([90, 5, 5])
        tr[j, 3:6] = g.dirichlet([60, 35, 5])
        tr[j, 6:9] = g.dirichlet([65, 5, 30]) if j > 0 else 0.0
        if j == L:
            for f in range(3):
                row = tr[j, 3 * f:3 * f + 3].copy()
                row[2] = 0.0
                tr[j, 3 * f:3 * f + 3] = row / row.sum() if row.sum() > 0 else 0.0
    eM = np.zeros((L + 1, K))
    eM[1:] = g.dirichlet(np.full(K, 0.4), size=L)
    eI = g.dirichlet(np.full(K, 20.0), size=L + 1)
    return tr, eM, eI


def sample_profile(g: np.random.Generator, tr, eM, eI, n: int, max_len: int = 1 << 30):
    """n sequences emitted by walking the profile from B to E (M and I states emit)."""
    L = tr.shape[0] - 1
    K = eM.shape[1]
    cM, cI = np.cumsum(eM, axis=1), np.cumsum(eI, axis=1)
    out = []
    while len(out) < n:
        st, j, seq = 0, 0, []   # st: 0 = M (M_0 = B), 1 = I, 2 = D; at position j
        while True:
            row = tr[j, 3 * st:3 * st + 3]
            to = min(int(np.searchsorted(np.cumsum(row), g.random(), side="right")), 2)
            if to == 1:
                st = 1
                seq.append(min(int(np.searchsorted(cI[j], g.random(), side="right")), K - 1))
            else:
                j += 1
                st = 0 if to == 0 else 2
                if j == L + 1:
                    break
                if st == 0:
                    seq.append(min(int(np.searchsorted(cM[j], g.random(), side="right")), K - 1))
            if len(seq) > max_len:
                break
        if len(seq) <= max_len:
            out.append(np.array(seq, dtype=np.uint8))
    return out


def profile_hmm_workload(n_seqs: int = 13_355, L: int = 256, K: int = 20):
    """NEXT 3 workload: one L = 256 position protein profile (params seed +9), n sequences sampled
    from it (seed +10; 13,355 = the database size of the paper's Fig.15). Both sides get the
    float32 parameters (the oracle widens them to float64)."""
    tr, eM, eI = profile_hmm_params(rng(9), L, K)
    tr32, eM32, eI32 = (x.astype(np.float32) for x in (tr, eM, eI))
    seqs = sample_profile(rng(10), tr, eM, eI, n_seqs, max_len=1023)
    cat, off = pack(seqs)
    return {"L": L, "K": K, "cat": cat, "off": off,
            "model": {"trans": tr32, "emit_m": eM32, "emit_i": eI32},
            "model64": {"trans": tr32.astype(np.float64), "emit_m": eM32.astype(np.float64),
                        "emit_i": eI32.astype(np.float64)}}
