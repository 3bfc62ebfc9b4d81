"""B200-native hyperplane DP (Cartey, Lyngsø & de Moor, PLDI 2012): thin Python
binding over the C ABI in include/dp.h (libdp.so, built in-tree for sm_100a).

Argument marshalling only: every step of the path runs in the library's CUDA
kernels. PyTorch supplies device memory and streams. There is no CPU
fallback: importing the binding without the built library raises.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("DP_LIB") or os.path.join(_PKG, "libdp.so")  # DP_LIB: experiment builds only

EDIT, SW_LINEAR, NUSSINOV, HMM_FORWARD, HMM_VITERBI, SW_AFFINE, DIAG_LCS, PROFILE_FORWARD = range(8)
KIND_NAMES = {EDIT: "edit", SW_LINEAR: "sw_linear", NUSSINOV: "nussinov", HMM_FORWARD: "hmm_forward",
              HMM_VITERBI: "hmm_viterbi", SW_AFFINE: "sw_affine", DIAG_LCS: "diag_lcs",
              PROFILE_FORWARD: "profile_forward"}
FLOAT_KINDS = (HMM_FORWARD, PROFILE_FORWARD)
STATUS = {0: "DP_OK", 1: "DP_E_INVALID", 2: "DP_E_NO_SCHEDULE", 3: "DP_E_UNSUPPORTED", 4: "DP_E_TOO_LARGE",
          5: "DP_E_NOMEM", 6: "DP_E_CUDA", 7: "DP_E_NO_TRACEBACK"}
MAX_DIM = 4
DEBUG = os.environ.get("DP_DEBUG", "0") == "1"


class DPError(RuntimeError):
    def __init__(self, code, where):
        self.code = code
        super().__init__(f"{where}: {STATUS.get(code, code)} ({lib().dp_status_string(code).decode()})")


class Dep(ctypes.Structure):
    _fields_ = [("offset", ctypes.c_int32 * MAX_DIM), ("ranged_axis", ctypes.c_int32),
                ("lo", ctypes.c_int64), ("hi", ctypes.c_int64)]


class Desc(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_uint32), ("kind", ctypes.c_int32),
        ("max_len_a", ctypes.c_int64), ("max_len_b", ctypes.c_int64),
        ("alphabet_size", ctypes.c_int32), ("sigma", ctypes.c_void_p), ("gap", ctypes.c_int32),
        ("pair_mask", ctypes.c_void_p), ("min_hairpin", ctypes.c_int32),
        ("n_states", ctypes.c_int32), ("pi", ctypes.c_void_p), ("A", ctypes.c_void_p), ("E", ctypes.c_void_p),
        ("lpi", ctypes.c_void_p), ("lA", ctypes.c_void_p), ("lE", ctypes.c_void_p),
        ("coeff_bound", ctypes.c_int32), ("user_coeff", ctypes.c_void_p), ("want_traceback", ctypes.c_int32),
        ("gap_open", ctypes.c_int32), ("gap_extend", ctypes.c_int32),
        ("n_positions", ctypes.c_int32), ("ptrans", ctypes.c_void_p), ("pemit_m", ctypes.c_void_p),
        ("pemit_i", ctypes.c_void_p),
    ]


_lib = None


def lib():
    """Loads libdp.so; raises if it was not built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_pldi_carteylm12_b200._build` "
                              "(or __graft_entry__.build()); there is no CPU fallback")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
        L.dp_abi_version.restype = ctypes.c_int
        L.dp_status_string.restype = ctypes.c_char_p
        L.dp_status_string.argtypes = [ctypes.c_int]
        L.dp_schedule_derive.restype = ctypes.c_int
        L.dp_schedule_derive.argtypes = [ctypes.c_int, ctypes.POINTER(i64), ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(Dep), ctypes.c_int, ctypes.POINTER(i32),
                                         ctypes.POINTER(i32), ctypes.POINTER(i64), ctypes.POINTER(i64),
                                         ctypes.POINTER(i32)]
        L.dp_schedule_conditional.restype = ctypes.c_int
        L.dp_schedule_conditional.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.POINTER(Dep), ctypes.c_int,
                                              ctypes.c_int, ctypes.POINTER(i32), ctypes.POINTER(ctypes.c_int)]
        L.dp_schedule_select.restype = ctypes.c_int
        L.dp_schedule_select.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.POINTER(i32), ctypes.POINTER(i64)]
        L.dp_plan_create.restype = ctypes.c_int
        L.dp_plan_create.argtypes = [ctypes.POINTER(Desc), ctypes.POINTER(vp)]
        L.dp_plan_destroy.restype = None
        L.dp_plan_destroy.argtypes = [vp]
        L.dp_plan_get_schedule.restype = ctypes.c_int
        L.dp_plan_get_schedule.argtypes = [vp, ctypes.POINTER(i32), ctypes.POINTER(ctypes.c_int),
                                           ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i32)]
        L.dp_plan_launch_count.restype = i64
        L.dp_plan_launch_count.argtypes = [vp]
        L.dp_plan_last_variant.restype = ctypes.c_char_p
        L.dp_plan_last_variant.argtypes = [vp]
        L.dp_solve_batch.restype = ctypes.c_int
        L.dp_solve_batch.argtypes = [vp, i64, vp, vp, vp, vp, i64, i64, vp, vp]
        L.dp_solve.restype = ctypes.c_int
        L.dp_solve.argtypes = [vp, vp, i64, vp, i64, vp, vp]
        L.dp_solve_batch_host.restype = ctypes.c_int
        L.dp_solve_batch_host.argtypes = [vp, i64, vp, vp, vp, vp, vp, vp, i64, vp, vp, vp]
        L.dp_traceback.restype = ctypes.c_int
        L.dp_traceback.argtypes = [vp, i64, i64, vp, i64, vp, vp, vp]
        _lib = L
    return _lib


EXPORTS = ["dp_abi_version", "dp_status_string", "dp_schedule_derive", "dp_schedule_conditional",
           "dp_schedule_select", "dp_plan_create", "dp_plan_destroy",
           "dp_plan_get_schedule", "dp_solve_batch", "dp_solve", "dp_solve_batch_host", "dp_traceback",
           "dp_plan_launch_count", "dp_plan_last_variant"]


def _check(code, where):
    if code != 0:
        raise DPError(code, where)


def schedule_derive(extent, deps, triangular=False, coeff_bound=10, user_coeff=None):
    """Front-end (A1–A4). deps: list of (offset tuple, ranged_axis or None, lo, hi).
    Returns dict(a, p_lo, p_hi, window); raises DPError (DP_E_NO_SCHEDULE) when infeasible."""
    nd = len(extent)
    ext = (ctypes.c_int64 * nd)(*extent)
    arr = (Dep * max(1, len(deps)))()
    for k, (off, axis, lo, hi) in enumerate(deps):
        for i, v in enumerate(off):
            arr[k].offset[i] = int(v)
        arr[k].ranged_axis = -1 if axis is None else int(axis)
        arr[k].lo, arr[k].hi = int(lo), int(hi)
    out = (ctypes.c_int32 * MAX_DIM)()
    lo, hi, w = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
    uc = (ctypes.c_int32 * nd)(*user_coeff) if user_coeff is not None else None
    _check(lib().dp_schedule_derive(nd, ext, int(bool(triangular)), len(deps), arr, int(coeff_bound), uc, out,
                                    ctypes.byref(lo), ctypes.byref(hi), ctypes.byref(w)), "dp_schedule_derive")
    return {"a": tuple(out[i] for i in range(nd)), "p_lo": lo.value, "p_hi": hi.value, "window": w.value}


def _deps_array(deps):
    arr = (Dep * max(1, len(deps)))()
    for k, (off, axis, lo, hi) in enumerate(deps):
        for i, v in enumerate(off):
            arr[k].offset[i] = int(v)
        arr[k].ranged_axis = -1 if axis is None else int(axis)
        arr[k].lo, arr[k].hi = int(lo), int(hi)
    return arr


def schedule_conditional(ndim, deps, coeff_bound=10):
    """§4.7 candidates (dp_schedule_conditional): list of coefficient tuples, identity order
    first; raises DPError (DP_E_NO_SCHEDULE) when infeasible."""
    out = (ctypes.c_int32 * (24 * MAX_DIM))()
    cnt = ctypes.c_int()
    _check(lib().dp_schedule_conditional(int(ndim), len(deps), _deps_array(deps), int(coeff_bound), 24, out,
                                         ctypes.byref(cnt)), "dp_schedule_conditional")
    return [tuple(out[c * ndim + i] for i in range(ndim)) for c in range(cnt.value)]


def schedule_select(candidates, extent):
    """Index of the candidate with the smallest box range for these extents (dp_schedule_select)."""
    nd = len(extent)
    flat = (ctypes.c_int32 * (len(candidates) * nd))(*[int(v) for a in candidates for v in a])
    k = lib().dp_schedule_select(nd, len(candidates), flat, (ctypes.c_int64 * nd)(*extent))
    if k < 0:
        raise DPError(1, "dp_schedule_select")
    return k


def _ptr(t):
    if t is None:
        return None
    if isinstance(t, np.ndarray):
        return t.ctypes.data
    return t.data_ptr()


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


class Plan:
    """A plan for one recurrence kind (dp_plan_create). Keeps host copies alive."""

    def __init__(self, kind, max_len_a, max_len_b=0, *, sigma=None, gap=0, alphabet_size=0, pair_mask=None,
                 min_hairpin=0, pi=None, A=None, E=None, lpi=None, lA=None, lE=None, want_traceback=False,
                 coeff_bound=0, user_coeff=None, gap_open=0, gap_extend=0, trans=None, emit_m=None, emit_i=None):
        self.kind = kind
        self._keep = []
        d = Desc()
        d.struct_size = ctypes.sizeof(Desc)
        d.kind = kind
        d.max_len_a, d.max_len_b = int(max_len_a), int(max_len_b)
        d.alphabet_size = int(alphabet_size)
        d.gap = int(gap)
        d.gap_open, d.gap_extend = int(gap_open), int(gap_extend)
        d.min_hairpin = int(min_hairpin)
        d.want_traceback = int(bool(want_traceback))
        d.coeff_bound = int(coeff_bound)

        def keep(arr, dtype):
            if arr is None:
                return None
            a = np.ascontiguousarray(arr, dtype=dtype)
            self._keep.append(a)
            return a.ctypes.data

        if sigma is not None:
            sig = np.ascontiguousarray(sigma, dtype=np.int8)
            d.alphabet_size = sig.shape[0] if not alphabet_size else alphabet_size
            d.sigma = keep(sig, np.int8)
        d.pair_mask = keep(None if pair_mask is None else np.asarray(pair_mask).reshape(-1), np.uint8)
        if pi is not None or lpi is not None:
            d.n_states = len(pi if pi is not None else lpi)
            EE = E if E is not None else lE
            d.alphabet_size = np.asarray(EE).shape[1]
        d.pi, d.A, d.E = keep(pi, np.float32), keep(A, np.float32), keep(E, np.float32)
        d.lpi, d.lA, d.lE = keep(lpi, np.int32), keep(lA, np.int32), keep(lE, np.int32)
        d.user_coeff = keep(user_coeff, np.int32)
        if trans is not None:  # profile HMM: (L+1) x 9 transitions, (L+1) x K emissions
            d.n_positions = np.asarray(trans).shape[0] - 1
            d.alphabet_size = np.asarray(emit_m).shape[1]
            d.ptrans = keep(np.asarray(trans).reshape(-1), np.float32)
            d.pemit_m = keep(np.asarray(emit_m).reshape(-1), np.float32)
            d.pemit_i = keep(np.asarray(emit_i).reshape(-1), np.float32)
        self.alphabet_size = d.alphabet_size
        self.max_len_a, self.max_len_b = int(max_len_a), int(max_len_b)
        self.want_traceback = bool(want_traceback)
        self.n_states = d.n_states
        h = ctypes.c_void_p()
        _check(lib().dp_plan_create(ctypes.byref(d), ctypes.byref(h)), "dp_plan_create")
        self._h = h

    def close(self):
        if getattr(self, "_h", None):
            lib().dp_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    @property
    def launches(self):
        return int(lib().dp_plan_launch_count(self._h))

    @property
    def last_variant(self):
        """The kernel family the last solve ran (dp_plan_last_variant)."""
        return lib().dp_plan_last_variant(self._h).decode()

    def schedule(self):
        co = (ctypes.c_int32 * MAX_DIM)()
        nd, lo, hi, w = ctypes.c_int(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
        _check(lib().dp_plan_get_schedule(self._h, co, ctypes.byref(nd), ctypes.byref(lo), ctypes.byref(hi),
                                          ctypes.byref(w)), "dp_plan_get_schedule")
        return {"a": tuple(co[i] for i in range(nd.value)), "p_lo": lo.value, "p_hi": hi.value, "window": w.value}

    def _debug_codes(self, cat, limit):
        if DEBUG and cat is not None and cat.numel():
            if int(cat.max()) >= limit:
                raise ValueError(f"alphabet code >= {limit}")

    def solve_batch(self, a_cat, a_off, b_cat=None, b_off=None, *, max_len_a=None, max_len_b=None, out=None,
                    stream=None):
        """Device tensors in, device scores out (int32, or float32 log-likelihood for HMM_FORWARD)."""
        import torch
        n = a_off.numel() - 1
        if max_len_a is None:
            max_len_a = int((a_off[1:] - a_off[:-1]).max().item()) if n > 0 else 0
        if max_len_b is None:
            max_len_b = int((b_off[1:] - b_off[:-1]).max().item()) if (b_off is not None and n > 0) else 0
        limit = 4 if self.kind == NUSSINOV else (256 if self.kind == DIAG_LCS else self.alphabet_size)
        self._debug_codes(a_cat, limit)
        self._debug_codes(b_cat, limit)
        if out is None:
            dt = torch.float32 if self.kind in FLOAT_KINDS else torch.int32
            out = torch.empty(max(n, 0), dtype=dt, device=a_off.device)
        self._last_inputs = (a_cat, a_off, b_cat, b_off)  # must outlive dp_traceback
        _check(lib().dp_solve_batch(self._h, n, _ptr(a_cat), _ptr(a_off), _ptr(b_cat), _ptr(b_off), int(max_len_a),
                                    int(max_len_b), _ptr(out), _stream_ptr(stream)), "dp_solve_batch")
        return out

    def solve(self, a, b=None, *, out=None, stream=None):
        """dp_solve: one problem from device tensors a (and b for the alignment kinds); returns a
        1-element device tensor (int32, or float32 log-likelihood for HMM_FORWARD)."""
        import torch
        if out is None:
            out = torch.empty(1, dtype=torch.float32 if self.kind in FLOAT_KINDS else torch.int32, device=a.device)
        self._last_inputs = (a, None, b, None)  # must outlive dp_traceback
        _check(lib().dp_solve(self._h, _ptr(a), int(a.numel()), _ptr(b), int(b.numel()) if b is not None else 0,
                              _ptr(out), _stream_ptr(stream)), "dp_solve")
        return out

    def traceback(self, first, count, stride, *, coords=True, stream=None, device="cuda"):
        import torch
        out = torch.empty((count, stride), dtype=torch.uint8, device=device)
        ln = torch.empty(count, dtype=torch.int32, device=device)
        co = torch.empty((count, 4), dtype=torch.int32, device=device) if coords else None
        _check(lib().dp_traceback(self._h, int(first), int(count), _ptr(out), int(stride), _ptr(ln), _ptr(co),
                                  _stream_ptr(stream)), "dp_traceback")
        return out, ln, co

    def traceback_into(self, first, count, out, stride, out_len, coords=None, stream=None):
        """dp_traceback into preallocated device tensors."""
        _check(lib().dp_traceback(self._h, int(first), int(count), _ptr(out), int(stride), _ptr(out_len),
                                  _ptr(coords), _stream_ptr(stream)), "dp_traceback")

    def solve_batch_host_into(self, a_cat, a_off, b_cat, b_off, scores, tb=None, tb_stride=0, tb_len=None,
                              tb_coords=None, stream=None):
        """dp_solve_batch_host into preallocated (pinned) numpy buffers."""
        _check(lib().dp_solve_batch_host(self._h, len(a_off) - 1, _ptr(a_cat), _ptr(a_off), _ptr(b_cat),
                                         _ptr(b_off), _ptr(scores), _ptr(tb), int(tb_stride), _ptr(tb_len),
                                         _ptr(tb_coords), _stream_ptr(stream)), "dp_solve_batch_host")

    def solve_batch_host(self, a_cat, a_off, b_cat=None, b_off=None, *, tb_stride=0, stream=None):
        """Host (numpy, ideally pinned) buffers in and out; synchronous (includes H2D/D2H)."""
        n = len(a_off) - 1
        scores = np.empty(n, dtype=np.float32 if self.kind in FLOAT_KINDS else np.int32)
        tb = tbl = tbc = None
        if self.want_traceback and tb_stride:
            tb = np.empty((n, tb_stride), dtype=np.uint8)
            tbl = np.empty(n, dtype=np.int32)
            if self.kind in (EDIT, SW_LINEAR, SW_AFFINE):
                tbc = np.empty((n, 4), dtype=np.int32)
        _check(lib().dp_solve_batch_host(self._h, n, _ptr(a_cat), _ptr(a_off), _ptr(b_cat), _ptr(b_off),
                                         _ptr(scores), _ptr(tb), int(tb_stride), _ptr(tbl), _ptr(tbc),
                                         _stream_ptr(stream)), "dp_solve_batch_host")
        return scores, tb, tbl, tbc


def pinned(arr):
    """Page-locked host copy of a numpy array (torch pinned memory)."""
    import torch
    t = torch.from_numpy(np.ascontiguousarray(arr)).pin_memory()
    return t.numpy(), t
