"""fp64 CPU oracle for BFAST-Monitor -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_icde_giesekerhvo20_b200``) never imports it and
shares no code with it; see the header of ``bfast_oracle.c`` for the paper
passages each function follows and DESIGN.md for the readings (R1-R14).

This module is argument marshalling (ctypes) around ``liboracle.so``, built
by ``build()`` below from ``bfast_oracle.c`` with gcc (no -ffast-math).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bfast_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

NO_BREAK = -1
INVALID = -2
DEG_REASONS = {0: "ok", 1: "nbar<K+1", 2: "h<1", 3: "no monitoring data",
               4: "rank deficient", 5: "sigma ~ 0"}


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc -O2 -fopenmp, IEEE semantics)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared",
               "-fno-fast-math", "-ffp-contract=off", _SRC, "-o", _LIB + ".tmp", "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i64, i32, f32, f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_float, ctypes.c_double
        lib.oracle_bfast_monitor.argtypes = [P, i64, i64, i64, P, i32, i32, f32, f32,
                                             P, P, P, P, P, P, P, P, P, P, P, ctypes.c_int]
        lib.oracle_bfast_monitor.restype = ctypes.c_int
        lib.oracle_design_row.argtypes = [P, i64, i32, P]
        lib.oracle_scatter_f64.argtypes = [P, i64, P, P, i64]
        lib.oracle_filter_missing.argtypes = [P, i64, i64, P, P, P, P, P, P, P]
        lib.oracle_filter_missing.restype = i32
        lib.oracle_gauss_jordan_inverse.argtypes = [P, i32, P, P]
        lib.oracle_gauss_jordan_inverse.restype = ctypes.c_int
        lib.oracle_fit.argtypes = [P, P, i32, i32, P, P]
        lib.oracle_fit.restype = ctypes.c_int
        lib.oracle_decode_i16.argtypes = [P, i64, f32, f32, ctypes.c_int32, P]
        lib.oracle_decode_i16.restype = None
        lib.oracle_boundary.argtypes = [f64, i32, i64]
        lib.oracle_boundary.restype = f64
        lib.oracle_mosum.argtypes = [P, i32, i32, i32, f64, P]
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def monitor(Y, dates, n_hist, k, hf, lam, threads: int = 0, ldY: int | None = None):
    """Run the oracle over all pixels of a time-major stack Y[N][P] (float32).

    Returns a dict of numpy arrays: break (int32), magnitude (f64),
    beta ([P][K] f64, basis (1, t, sin 2 pi d, cos 2 pi d, ...), t 1-based),
    sigma, nbar, Nbar, h, max_ratio, near_tie, cond, deg_reason.
    """
    lib = _load()
    Y = np.ascontiguousarray(Y, dtype=np.float32)
    if Y.ndim != 2:
        raise ValueError("Y must be [N][P]")
    N, P = Y.shape
    if ldY is not None:
        raise ValueError("pass a contiguous [N][P] view")
    dates = np.ascontiguousarray(dates, dtype=np.float64)
    K = 2 + 2 * int(k)
    out = {
        "break": np.empty(P, np.int32), "magnitude": np.empty(P, np.float64),
        "beta": np.empty((P, K), np.float64), "sigma": np.empty(P, np.float64),
        "nbar": np.empty(P, np.int32), "Nbar": np.empty(P, np.int32),
        "h": np.empty(P, np.int32), "max_ratio": np.empty(P, np.float64),
        "near_tie": np.empty(P, np.int32), "cond": np.empty(P, np.float64),
        "deg_reason": np.empty(P, np.int32),
    }
    rc = lib.oracle_bfast_monitor(
        _ptr(Y), N, P, P, _ptr(dates), int(n_hist), int(k), float(hf), float(lam),
        _ptr(out["break"]), _ptr(out["magnitude"]), _ptr(out["beta"]), _ptr(out["sigma"]),
        _ptr(out["nbar"]), _ptr(out["Nbar"]), _ptr(out["h"]), _ptr(out["max_ratio"]),
        _ptr(out["near_tie"]), _ptr(out["cond"]), _ptr(out["deg_reason"]), int(threads))
    if rc != 0:
        raise ValueError("oracle_bfast_monitor: invalid arguments")
    return out


# --- individual steps, exposed for the pins in tests/test_oracle_pins.py ---

def design_row(dates, t0, k):
    x = np.empty(2 + 2 * k, np.float64)
    d = np.ascontiguousarray(dates, np.float64)
    _load().oracle_design_row(_ptr(d), int(t0), int(k), _ptr(x))
    return x


def scatter(x, idx, vals):
    x = np.array(x, dtype=np.float64)
    idx = np.ascontiguousarray(idx, dtype=np.int64)
    vals = np.ascontiguousarray(vals, dtype=np.float64)
    _load().oracle_scatter_f64(_ptr(x), x.size, _ptr(idx), _ptr(vals), idx.size)
    return x


def filter_missing(y):
    y = np.ascontiguousarray(y, dtype=np.float32)
    N = y.size
    vs = np.empty(N, np.float64)
    ks = np.empty(N, np.int64)
    tfs = np.empty(N, np.int32)
    indsT = np.empty(N, np.int32)
    inds = np.empty(N, np.int64)
    vec = np.empty(N, np.float64)
    iota = np.empty(N, np.int64)
    Nbar = _load().oracle_filter_missing(_ptr(y), N, 1, _ptr(vs), _ptr(ks), _ptr(tfs),
                                         _ptr(indsT), _ptr(inds), _ptr(vec), _ptr(iota))
    return int(Nbar), vs, ks


def gauss_jordan_inverse(M):
    M = np.ascontiguousarray(M, dtype=np.float64)
    K = M.shape[0]
    Minv = np.empty_like(M)
    cond = np.zeros(1)
    rc = _load().oracle_gauss_jordan_inverse(_ptr(M), K, _ptr(Minv), _ptr(cond))
    return (None if rc else Minv), float(cond[0])


def fit(Xbar, ybar, nbar):
    Xbar = np.ascontiguousarray(Xbar, dtype=np.float64)
    ybar = np.ascontiguousarray(ybar, dtype=np.float64)
    K = Xbar.shape[1]
    beta = np.empty(K, np.float64)
    cond = np.zeros(1)
    rc = _load().oracle_fit(_ptr(Xbar), _ptr(ybar), int(nbar), K, _ptr(beta), _ptr(cond))
    return None if rc else beta


def boundary(lam, nbar, j):
    return float(_load().oracle_boundary(float(lam), int(nbar), int(j)))


def mosum(rbar, nbar, Nbar, h, sigma):
    rbar = np.ascontiguousarray(rbar, dtype=np.float64)
    m = np.empty(max(Nbar - nbar, 0), np.float64)
    _load().oracle_mosum(_ptr(rbar), int(nbar), int(Nbar), int(h), float(sigma), _ptr(m))
    return m


def drop_empty_dates(Y, dates, n_hist, P: int | None = None):
    """PAPER.md L291 ("removal of slices only containing
    NaN values", a preprocessing step after each chunk reaches the GPU) and
    L379 (about 350 of 6873 Africa dates hold any data).  Plain definition:
    slice t is kept iff some pixel p < P has y[t, p] == y[t, p] (not NaN, any
    payload, reading R9); the kept slices in their original order, their
    dates, and n_hist' = the number of kept dates before n_hist (the history
    of the compacted stack).  Returns (Yc, dates_c, n_hist_c, keep_idx)."""
    Y = np.asarray(Y)
    P = Y.shape[1] if P is None else int(P)
    keep_idx = np.flatnonzero(~np.all(np.isnan(Y[:, :P]), axis=1))
    d = np.asarray(dates, dtype=np.float64)
    return (np.ascontiguousarray(Y[keep_idx, :P]), d[keep_idx],
            int(np.count_nonzero(keep_idx < int(n_hist))), keep_idx)


def decode_i16(codes, scale: float, offset: float, nodata: int):
    """f4 (reading R15): y = fmaf(scale, code, offset) in fp32, nodata -> NaN
    (oracle_decode_i16, C99 fmaf).  Same shape as `codes`."""
    c = np.ascontiguousarray(np.asarray(codes, dtype=np.int16))
    y = np.empty(c.shape, dtype=np.float32)
    _load().oracle_decode_i16(_ptr(c), int(c.size), float(scale), float(offset), int(nodata), _ptr(y))
    return y


def monitor_periods(Y, dates, periods, k, hf, lam, threads: int = 0):
    """PAPER.md L391 (monitoring periods 2010-2011,
    2011-2012, ... over one data cube): period (n_i, N_i) is Algorithm 1 on
    the first N_i dates with history [0, n_i).  Plain definition: one
    oracle run per period on that slice of the stack."""
    Y = np.asarray(Y)
    d = np.asarray(dates, dtype=np.float64)
    return [monitor(np.ascontiguousarray(Y[:int(N_i)]), d[:int(N_i)], int(n_i), k, hf, lam, threads=threads)
            for n_i, N_i in periods]
