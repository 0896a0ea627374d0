"""Parity comparison of the CUDA path against the fp64 oracle -- TEST
INFRASTRUCTURE (used by tests/, __graft_entry__.smoke() and bench.py).

Tolerances are BASELINE.json's north star, with the readings DESIGN.md
"Parity bar" states:
  break      identical, except pixels whose oracle max_j |m_j|/B_j lies within
             1e-3 of 1 (the literal rule); the refined rule (a near tie at
             some j <= j*) is reported beside it.  Invalid-pixel (-2)
             classification must match exactly.
  magnitude  |gpu - oracle| <= 1e-4 * max(1, |oracle|)
  beta       per component, column-scaled: |d beta_j| s_j <= 1e-4 max_i |beta_i s_i|
             with s_j the RMS of design column j over the history dates.
"""
from __future__ import annotations

import math

import numpy as np

MAG_TOL = 1e-4
BETA_TOL = 1e-4
TIE_TOL = 1e-3


def column_scales(dates, n_hist, k):
    """RMS of each design column of Eq. (3) over the history dates."""
    t = np.arange(1, n_hist + 1, dtype=np.float64)
    d = np.asarray(dates, np.float64)[:n_hist]
    cols = [np.ones(n_hist), t]
    for j in range(1, k + 1):
        cols += [np.sin(2 * math.pi * j * d), np.cos(2 * math.pi * j * d)]
    return np.sqrt(np.mean(np.stack(cols, 1) ** 2, axis=0))


def compare(gpu: dict, orc: dict, dates=None, n_hist=None, k=None, mag_tol=MAG_TOL,
            beta_tol=BETA_TOL, tie_tol=TIE_TOL) -> dict:
    gb = np.asarray(gpu["break"]).astype(np.int64)
    ob = np.asarray(orc["break"]).astype(np.int64)
    gm = np.asarray(gpu["magnitude"], np.float64)
    om = np.asarray(orc["magnitude"], np.float64)
    P = ob.size
    rep = {"pixels": int(P)}
    g_inv, o_inv = gb == -2, ob == -2
    rep["invalid_oracle"] = int(o_inv.sum())
    rep["invalid_mismatch"] = int((g_inv != o_inv).sum())
    both = ~g_inv & ~o_inv
    mism = both & (gb != ob)
    ratio = np.asarray(orc["max_ratio"], np.float64)
    literal = np.abs(ratio - 1.0) <= tie_tol
    refined = np.asarray(orc["near_tie"]).astype(bool)
    rep["break_mismatch"] = int(mism.sum())
    rep["break_mismatch_excused_literal"] = int((mism & literal).sum())
    rep["break_mismatch_excused_refined"] = int((mism & refined).sum())
    rep["break_mismatch_unexcused"] = int((mism & ~literal).sum())
    rep["near_tie_pixels_literal"] = int((both & literal).sum())
    rep["near_tie_pixels_refined"] = int((both & refined).sum())
    rep["breaks_oracle"] = int((both & (ob >= 0)).sum())
    err = np.abs(gm - om) / np.maximum(1.0, np.abs(om))
    err = np.where(both, err, 0.0)
    rep["mag_max_scaled_err"] = float(np.nanmax(err)) if P else 0.0
    rep["mag_fail"] = int((both & ~(err <= mag_tol)).sum())
    rep["mag_nan_mismatch"] = int((np.isnan(gm) != np.isnan(om)).sum())
    if "beta" in gpu and "beta" in orc and dates is not None:
        s = column_scales(dates, n_hist, k)
        gbeta = np.asarray(gpu["beta"], np.float64)
        obeta = np.asarray(orc["beta"], np.float64)
        fit = np.isfinite(obeta).all(1)
        ref = np.max(np.abs(obeta * s), axis=1)
        be = np.max(np.abs(gbeta - obeta) * s, axis=1) / np.where(ref > 0, ref, 1.0)
        be = np.where(fit, be, 0.0)
        rep["beta_max_scaled_err"] = float(np.nanmax(be)) if P else 0.0
        rep["beta_fail"] = int((fit & ~(be <= beta_tol)).sum())
    if "flags" in gpu:
        rep["refit_fp64"] = int((np.asarray(gpu["flags"]) & 2).astype(bool).sum())
    rep["ok"] = bool(rep["invalid_mismatch"] == 0 and rep["break_mismatch_unexcused"] == 0
                     and rep["mag_fail"] == 0 and rep.get("beta_fail", 0) == 0
                     and rep["mag_nan_mismatch"] == 0)
    return rep
