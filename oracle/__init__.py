"""CPU oracle — TEST INFRASTRUCTURE ONLY.

Plain, slow, obviously-correct evaluation of the hot path's recurrences
(oracle/oracle.c, memoised recursions in int64 / fp64) and of the schedule
analysis (oracle/schedule.py, brute force over explicit call graphs).

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
`--impl reference` leg may import this package. The product
(paper_conf_pldi_carteylm12_b200) never imports it and shares no code with it.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

i64 = ctypes.c_int64
u8p = np.ctypeslib.ndpointer(dtype=np.uint8, flags="C_CONTIGUOUS")
i8p = np.ctypeslib.ndpointer(dtype=np.int8, flags="C_CONTIGUOUS")
i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
i64p = np.ctypeslib.ndpointer(dtype=np.int64, flags="C_CONTIGUOUS")
f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")


def build(force: bool = False) -> str:
    """Compile oracle.c with plain gcc -O2 (building the checker is not using it)."""
    with _lock:
        if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
            tmp = _LIB + f".{os.getpid()}.tmp"
            subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
            os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.orc_edit.restype = i64
        L.orc_edit.argtypes = [u8p, i64, u8p, i64]
        L.orc_edit_traceback.restype = i64
        L.orc_edit_traceback.argtypes = [u8p, i64, u8p, i64, u8p]
        L.orc_sw.restype = i64
        L.orc_sw.argtypes = [u8p, i64, u8p, i64, i8p, ctypes.c_int, i64, ctypes.POINTER(i64), ctypes.POINTER(i64)]
        L.orc_sw_traceback.restype = i64
        L.orc_sw_traceback.argtypes = [u8p, i64, u8p, i64, i8p, ctypes.c_int, i64, u8p, i64p]
        L.orc_sw_affine.restype = i64
        L.orc_sw_affine.argtypes = [u8p, i64, u8p, i64, i8p, ctypes.c_int, i64, i64, ctypes.POINTER(i64),
                                    ctypes.POINTER(i64)]
        L.orc_sw_affine_traceback.restype = i64
        L.orc_sw_affine_traceback.argtypes = [u8p, i64, u8p, i64, i8p, ctypes.c_int, i64, i64, u8p, i64p]
        L.orc_sw_affine_batch.restype = None
        L.orc_sw_affine_batch.argtypes = [i64, i64, u8p, i64p, u8p, i64p, i8p, ctypes.c_int, i64, i64, i64p]
        L.orc_sw_affine_traceback_batch.restype = None
        L.orc_sw_affine_traceback_batch.argtypes = [i64, i64, u8p, i64p, u8p, i64p, i8p, ctypes.c_int, i64, i64,
                                                    u8p, i64, i64p]
        L.orc_nussinov.restype = i64
        L.orc_lcsubstr.restype = i64
        L.orc_lcsubstr.argtypes = [u8p, i64, u8p, i64]
        L.orc_lcsubstr_batch.argtypes = [i64, i64, u8p, i64p, u8p, i64p, i64p]
        L.orc_nussinov.argtypes = [u8p, i64, u8p, ctypes.c_int]
        L.orc_nussinov_traceback.restype = i64
        L.orc_nussinov_traceback.argtypes = [u8p, i64, u8p, ctypes.c_int, u8p]
        L.orc_forward.restype = ctypes.c_double
        L.orc_forward.argtypes = [u8p, i64, ctypes.c_int, ctypes.c_int, f64p, f64p, f64p]
        L.orc_silent_forward.restype = ctypes.c_double
        L.orc_silent_forward.argtypes = [u8p, i64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, u8p, f64p,
                                         f64p]
        L.orc_silent_forward_batch.restype = None
        L.orc_silent_forward_batch.argtypes = [i64, i64, u8p, i64p, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                               ctypes.c_int, u8p, f64p, f64p, f64p]
        L.orc_viterbi.restype = i64
        L.orc_viterbi.argtypes = [u8p, i64, ctypes.c_int, ctypes.c_int, i32p, i32p, i32p, u8p]
        L.orc_sw_batch.restype = None
        L.orc_sw_batch.argtypes = [i64, i64, u8p, i64p, u8p, i64p, i8p, ctypes.c_int, i64, i64p]
        L.orc_sw_traceback_batch.restype = None
        L.orc_sw_traceback_batch.argtypes = [i64, i64, u8p, i64p, u8p, i64p, i8p, ctypes.c_int, i64, u8p, i64, i64p]
        L.orc_nussinov_batch.restype = None
        L.orc_nussinov_batch.argtypes = [i64, i64, u8p, i64p, u8p, ctypes.c_int, i64p]
        L.orc_forward_batch.restype = None
        L.orc_forward_batch.argtypes = [i64, i64, u8p, i64p, ctypes.c_int, ctypes.c_int, f64p, f64p, f64p, f64p]
        L.orc_viterbi_batch.restype = None
        L.orc_viterbi_batch.argtypes = [i64, i64, u8p, i64p, ctypes.c_int, ctypes.c_int, i32p, i32p, i32p, i64p]
        _lib = L
    return _lib


def _u8(x):
    return np.ascontiguousarray(np.asarray(x, dtype=np.uint8))


# ----------------------------------------------------------------------------- single problems
def edit(s, t) -> int:
    s, t = _u8(s), _u8(t)
    return int(lib().orc_edit(s, len(s), t, len(t)))


def edit_traceback(s, t) -> str:
    s, t = _u8(s), _u8(t)
    buf = np.zeros(len(s) + len(t) + 1, dtype=np.uint8)
    n = lib().orc_edit_traceback(s, len(s), t, len(t), buf)
    return bytes(buf[:n]).decode()


def sw(s, t, sigma, g) -> tuple[int, int, int]:
    """Returns (score, end_i, end_j) (end = first max cell in row-major order, 1-based)."""
    s, t = _u8(s), _u8(t)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    ei, ej = i64(0), i64(0)
    sc = lib().orc_sw(s, len(s), t, len(t), sig, sig.shape[0], int(g), ctypes.byref(ei), ctypes.byref(ej))
    return int(sc), int(ei.value), int(ej.value)


def sw_traceback(s, t, sigma, g) -> tuple[str, tuple[int, int, int, int]]:
    """Returns (ops, (start_i, start_j, end_i, end_j)); cells are 1-based DP indices,
    the alignment covers s[start_i:end_i], t[start_j:end_j]."""
    s, t = _u8(s), _u8(t)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    buf = np.zeros(len(s) + len(t) + 1, dtype=np.uint8)
    co = np.zeros(4, dtype=np.int64)
    n = lib().orc_sw_traceback(s, len(s), t, len(t), sig, sig.shape[0], int(g), buf, co)
    return bytes(buf[:n]).decode(), tuple(int(v) for v in co)


def sw_affine(s, t, sigma, go, ge) -> tuple[int, int, int]:
    """Affine-gap SW (gap of length k costs go + k*ge): (score, end_i, end_j)."""
    s, t = _u8(s), _u8(t)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    ei, ej = i64(0), i64(0)
    sc = lib().orc_sw_affine(s, len(s), t, len(t), sig, sig.shape[0], int(go), int(ge), ctypes.byref(ei),
                             ctypes.byref(ej))
    return int(sc), int(ei.value), int(ej.value)


def sw_affine_traceback(s, t, sigma, go, ge) -> tuple[str, tuple[int, int, int, int]]:
    s, t = _u8(s), _u8(t)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    buf = np.zeros(len(s) + len(t) + 1, dtype=np.uint8)
    co = np.zeros(4, dtype=np.int64)
    n = lib().orc_sw_affine_traceback(s, len(s), t, len(t), sig, sig.shape[0], int(go), int(ge), buf, co)
    return bytes(buf[:n]).decode(), tuple(int(v) for v in co)


def sw_affine_batch(a_cat, a_off, b_cat, b_off, sigma, go, ge, threads=1) -> np.ndarray:
    n = len(a_off) - 1
    out = np.zeros(n, dtype=np.int64)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    a_cat, b_cat = _u8(a_cat), _u8(b_cat)
    a_off, b_off = np.ascontiguousarray(a_off, np.int64), np.ascontiguousarray(b_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_sw_affine_batch(f, c, a_cat, a_off, b_cat, b_off, sig, sig.shape[0],
                                                        int(go), int(ge), out), threads)
    return out


def sw_affine_traceback_batch(a_cat, a_off, b_cat, b_off, sigma, go, ge, stride, threads=1):
    n = len(a_off) - 1
    ops = np.zeros((n, stride), dtype=np.uint8)
    lens = np.zeros(n, dtype=np.int64)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    a_cat, b_cat = _u8(a_cat), _u8(b_cat)
    a_off, b_off = np.ascontiguousarray(a_off, np.int64), np.ascontiguousarray(b_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_sw_affine_traceback_batch(f, c, a_cat, a_off, b_cat, b_off, sig,
                                                                  sig.shape[0], int(go), int(ge), ops.reshape(-1),
                                                                  stride, lens), threads)
    return ops, lens


def lcsubstr(s, t) -> int:
    """Diagonal-only recurrence of §4.7 (L386-L388) as the longest common substring."""
    s, t = _u8(s), _u8(t)
    return int(lib().orc_lcsubstr(s, len(s), t, len(t)))


def nussinov(x, pair_mask, h) -> int:
    x = _u8(x)
    return int(lib().orc_nussinov(x, len(x), _u8(pair_mask).reshape(-1).copy(), int(h)))


def nussinov_traceback(x, pair_mask, h) -> tuple[int, str]:
    x = _u8(x)
    buf = np.zeros(max(len(x), 1), dtype=np.uint8)
    sc = lib().orc_nussinov_traceback(x, len(x), _u8(pair_mask).reshape(-1).copy(), int(h), buf)
    return int(sc), bytes(buf[:len(x)]).decode()


def forward(x, pi, A, E) -> float:
    """log P(x) (natural log), fp64."""
    x = _u8(x)
    pi = np.ascontiguousarray(pi, dtype=np.float64)
    A = np.ascontiguousarray(A, dtype=np.float64)
    E = np.ascontiguousarray(E, dtype=np.float64)
    return float(lib().orc_forward(x, len(x), len(pi), E.shape[1], pi, A, E))


def silent_forward(x, silent, A, E, begin, end) -> float:
    """log P(x) (natural log, fp64) of a generic HMM with silent states (§5.2; DESIGN.md R-PHMM)."""
    x = _u8(x)
    sil = _u8(silent)
    A = np.ascontiguousarray(A, dtype=np.float64)
    E = np.ascontiguousarray(E, dtype=np.float64)
    return float(lib().orc_silent_forward(x, len(x), len(sil), E.shape[1], int(begin), int(end), sil, A, E))


def profile_as_hmm(trans, emit_m, emit_i):
    """The profile HMM of L positions written as a generic HMM in the paper's extension (§5.2:
    states, transitions, emissions, silent states), so its forward is §5.2's forward. State
    order: B = M_0, then for j = 1..L: M_j, I_{j-1}, D_j; then I_L, then E (= M_{L+1}) — a
    position-major total order (the paper's "arbitrary total order", L453-L455).
    trans[j][3 f + t]: from (M_j, I_j, D_j)[f] to (M_{j+1}, I_j, D_{j+1})[t]."""
    trans = np.asarray(trans, np.float64)
    eM, eI = np.asarray(emit_m, np.float64), np.asarray(emit_i, np.float64)
    L = trans.shape[0] - 1
    K = eM.shape[1]
    idx = {("M", 0): 0}
    for j in range(1, L + 1):
        idx[("M", j)] = len(idx)
        idx[("I", j - 1)] = len(idx)
        idx[("D", j)] = len(idx)
    idx[("I", L)] = len(idx)
    idx[("M", L + 1)] = len(idx)       # E
    S = len(idx)
    A = np.zeros((S, S))
    E = np.zeros((S, K))
    silent = np.zeros(S, np.uint8)
    for (k, j), s in idx.items():
        if k == "D" or (k == "M" and j in (0, L + 1)):
            silent[s] = 1
        elif k == "M":
            E[s] = eM[j]
        else:
            E[s] = eI[j]
    for j in range(L + 1):
        for f, kf in enumerate("MID"):
            src = idx.get((kf, j))
            if src is None:
                continue
            for t, dst in enumerate((("M", j + 1), ("I", j), ("D", j + 1))):
                p = trans[j][3 * f + t]
                if p > 0 and dst in idx:
                    A[src, idx[dst]] += p
    return silent, A, E, idx[("M", 0)], idx[("M", L + 1)]


def profile_forward(x, trans, emit_m, emit_i) -> float:
    """log P(x) of the profile HMM, via the generic silent-state forward."""
    silent, A, E, b, e = profile_as_hmm(trans, emit_m, emit_i)
    return silent_forward(x, silent, A, E, b, e)


def profile_forward_batch(cat, off, L, trans, emit_m, emit_i, threads=1) -> np.ndarray:
    silent, A, E, b, e = profile_as_hmm(trans, emit_m, emit_i)
    n = len(off) - 1
    out = np.zeros(n, dtype=np.float64)
    cat, off = _u8(cat), np.ascontiguousarray(off, np.int64)
    A = np.ascontiguousarray(A)
    E = np.ascontiguousarray(E)
    _parallel(n, lambda f, c: lib().orc_silent_forward_batch(f, c, cat, off, len(silent), E.shape[1], int(b), int(e),
                                                             silent, A, E, out), threads)
    return out


def viterbi(x, lpi, lA, lE) -> tuple[int, np.ndarray]:
    x = _u8(x)
    lpi = np.ascontiguousarray(lpi, dtype=np.int32)
    lA = np.ascontiguousarray(lA, dtype=np.int32)
    lE = np.ascontiguousarray(lE, dtype=np.int32)
    path = np.zeros(max(len(x), 1), dtype=np.uint8)
    sc = lib().orc_viterbi(x, len(x), len(lpi), lE.shape[1], lpi, lA, lE, path)
    return int(sc), path[:len(x)].copy()


# ----------------------------------------------------------------------------- batches (threaded)
def _parallel(total, fn, threads):
    threads = max(1, min(threads, total)) if total else 1
    if total == 0:
        return
    chunk = (total + threads - 1) // threads
    ts = []
    for k in range(threads):
        f, c = k * chunk, min(chunk, total - k * chunk)
        if c <= 0:
            break
        t = threading.Thread(target=fn, args=(f, c))
        t.start()
        ts.append(t)
    for t in ts:
        t.join()


def sw_batch(a_cat, a_off, b_cat, b_off, sigma, g, threads=1) -> np.ndarray:
    n = len(a_off) - 1
    out = np.zeros(n, dtype=np.int64)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    a_cat, b_cat = _u8(a_cat), _u8(b_cat)
    a_off, b_off = np.ascontiguousarray(a_off, np.int64), np.ascontiguousarray(b_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_sw_batch(f, c, a_cat, a_off, b_cat, b_off, sig, sig.shape[0], int(g), out), threads)
    return out


def sw_traceback_batch(a_cat, a_off, b_cat, b_off, sigma, g, stride, threads=1):
    """Canonical tracebacks of a batch (ops, lengths); each problem's score is recomputed inside."""
    n = len(a_off) - 1
    ops = np.zeros((n, stride), dtype=np.uint8)
    lens = np.zeros(n, dtype=np.int64)
    sig = np.ascontiguousarray(sigma, dtype=np.int8)
    a_cat, b_cat = _u8(a_cat), _u8(b_cat)
    a_off, b_off = np.ascontiguousarray(a_off, np.int64), np.ascontiguousarray(b_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_sw_traceback_batch(f, c, a_cat, a_off, b_cat, b_off, sig, sig.shape[0],
                                                           int(g), ops.reshape(-1), stride, lens), threads)
    return ops, lens


def lcsubstr_batch(a_cat, a_off, b_cat, b_off, threads=1) -> np.ndarray:
    """Diagonal-only recurrence (§4.7 example; longest common substring) over a packed batch."""
    n = len(a_off) - 1
    out = np.zeros(n, dtype=np.int64)
    a_cat, b_cat = _u8(a_cat), _u8(b_cat)
    a_off, b_off = np.ascontiguousarray(a_off, np.int64), np.ascontiguousarray(b_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_lcsubstr_batch(f, c, a_cat, a_off, b_cat, b_off, out), threads)
    return out


def nussinov_batch(x_cat, x_off, pair_mask, h, threads=1) -> np.ndarray:
    n = len(x_off) - 1
    out = np.zeros(n, dtype=np.int64)
    pm = _u8(pair_mask).reshape(-1).copy()
    x_cat, x_off = _u8(x_cat), np.ascontiguousarray(x_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_nussinov_batch(f, c, x_cat, x_off, pm, int(h), out), threads)
    return out


def forward_batch(x_cat, x_off, pi, A, E, threads=1) -> np.ndarray:
    n = len(x_off) - 1
    out = np.zeros(n, dtype=np.float64)
    pi = np.ascontiguousarray(pi, dtype=np.float64)
    A = np.ascontiguousarray(A, dtype=np.float64)
    E = np.ascontiguousarray(E, dtype=np.float64)
    x_cat, x_off = _u8(x_cat), np.ascontiguousarray(x_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_forward_batch(f, c, x_cat, x_off, len(pi), E.shape[1], pi, A, E, out), threads)
    return out


def viterbi_batch(x_cat, x_off, lpi, lA, lE, threads=1) -> np.ndarray:
    n = len(x_off) - 1
    out = np.zeros(n, dtype=np.int64)
    lpi = np.ascontiguousarray(lpi, dtype=np.int32)
    lA = np.ascontiguousarray(lA, dtype=np.int32)
    lE = np.ascontiguousarray(lE, dtype=np.int32)
    x_cat, x_off = _u8(x_cat), np.ascontiguousarray(x_off, np.int64)
    _parallel(n, lambda f, c: lib().orc_viterbi_batch(f, c, x_cat, x_off, len(lpi), lE.shape[1], lpi, lA, lE, out), threads)
    return out
