"""Pins of the fp64 oracle against what the paper and mathematics fix (P1-P8).

None of these tests re-types the oracle's formula: each compares the oracle
with a hand-worked example, a closed form, a different algorithm (LAPACK
least squares, prefix sums), an invariant, or the paper's own example.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle

TWO_PI = 2.0 * math.pi


def _design(dates, k):
    """Eq. (3) (L65): x_t = (1, t, sin 2 pi j d_t, cos 2 pi j d_t ...), t 1-based.
    Built here independently with numpy for the lstsq pin."""
    N = len(dates)
    cols = [np.ones(N), np.arange(1, N + 1, dtype=np.float64)]
    for j in range(1, k + 1):
        cols += [np.sin(TWO_PI * j * dates), np.cos(TWO_PI * j * dates)]
    return np.stack(cols, axis=1)


def _rand_stack(rng, N, P, k, miss, noise=0.05):
    dates = 2000.0 + np.arange(1, N + 1) / 23.0
    X = _design(dates, k)
    beta = rng.normal(size=(P, X.shape[1])) * np.array([1, 0.01] + [0.2] * (2 * k))
    Y = (X @ beta.T + rng.normal(scale=noise, size=(N, P))).astype(np.float32)
    Y[rng.random((N, P)) < miss] = np.nan
    return Y, dates


# ---------------------------------------------------------------- P1
def test_p1_worked_example(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "p1_worked_example.json")))
    inp, exp = g["input"], g["expected"]
    y = np.array([np.nan if v == "nan" else v for v in inp["Y"]], np.float32)[:, None]
    out = oracle.monitor(y, np.array(inp["dates"]), inp["n_hist"], inp["k"], inp["hf"], inp["lambda"])
    assert out["nbar"][0] == exp["nbar"] and out["Nbar"][0] == exp["Nbar"] and out["h"][0] == exp["h"]
    np.testing.assert_allclose(out["beta"][0], exp["beta"], rtol=1e-12)
    assert out["sigma"][0] == pytest.approx(exp["sigma"], rel=1e-12)
    assert out["break"][0] == exp["break"]
    assert out["magnitude"][0] == pytest.approx(exp["magnitude"], rel=1e-12)
    # the individual steps
    Nbar, vs, ks = oracle.filter_missing(y[:, 0])
    assert Nbar == 6 and list(ks[:6]) == [0, 1, 3, 5, 6, 7]
    X = _design(np.array(inp["dates"]), 0)[ks[:6]]
    r = vs[:6] - X @ out["beta"][0]
    np.testing.assert_allclose(r * 14, exp["residuals_times_14"], atol=1e-11)
    m = oracle.mosum(r, 3, 6, 2, exp["sigma"])
    np.testing.assert_allclose(m, exp["mosum"], rtol=1e-12)
    assert [oracle.boundary(1.5, 3, j) for j in range(3)] == exp["boundary"]
    # the parity diagnostics (oracle/parity.py's excuse rules): max_j |m_j|/B_j
    # over the whole monitoring period and the refined near-tie flag
    assert out["max_ratio"][0] == pytest.approx(exp["max_ratio"], rel=1e-12)
    assert out["near_tie"][0] == exp["near_tie"]


def test_p9_near_tie_before_the_break():
    """Hand-built pixel (P1's history and its last two monitoring values):
    the first monitoring value is chosen so that m_0 = 1.49925, i.e.
    |m_0|/B_0 = 0.9995, within 1e-3 of 1 but no break; m_1 then crosses
    (j* = 1), m_2 is P1's -20.830952.  So near_tie = 1 (a tie at j = 0 <= j*)
    while the literal rule's max ratio is P1's 13.887301, far from 1: the
    pixel the refined rule excuses and the literal one does not.  A max taken
    over j <= j* only would give |m_1|/1.5 = 2.54 instead."""
    s14 = math.sqrt(3.0 / 14.0)                      # sigma sqrt(nbar) of P1
    r_hist_last = -1.0 / 14.0                        # residual of rank 2 (t = 4)
    r3 = 1.49925 * s14 - r_hist_last                 # m_0 = (r_2 + r_3) / s14
    y6 = r3 + (-0.5 + 23.0 * 6.0 / 14.0)             # + yhat(6) of P1's fit
    y = np.array([1.0, 3.0, np.nan, 6.0, np.nan, y6, 12.0, 2.0], np.float32)[:, None]
    out = oracle.monitor(y, np.arange(1.0, 9.0), 4, 0, 0.75, 1.5)
    assert out["near_tie"][0] == 1
    assert out["break"][0] == 2                      # rank nbar + 1 -> t = 7 -> 6 - n
    assert out["max_ratio"][0] == pytest.approx(135 * math.sqrt(14 / 3) / 21, rel=1e-12)
    r3f = float(y[5, 0]) - (-0.5 + 23.0 * 6.0 / 14.0)   # the fp32 input's residual
    m = np.array([r_hist_last + r3f, r3f + 1.0, 1.0 - 149.0 / 14.0]) / s14
    assert abs(m[0]) / 1.5 == pytest.approx(0.9995, abs=1e-6)
    assert out["magnitude"][0] == pytest.approx(m.mean(), rel=1e-9)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_p9_max_ratio_and_near_tie_brute_force(seed):
    """max_ratio / near_tie against a brute-force recomputation on tiny
    inputs where the boundary is NOT flat (n = N/4, 60% missing: (nbar+1+j)/
    nbar passes e): numpy lstsq residuals, direct window sums, and the
    boundary of the P2 table (lambda sqrt(max(1, ln x)), pinned there)."""
    rng = np.random.default_rng(90 + seed)
    N, n, k, P, hf, lam = 64, 16, 1, 48, 0.5, 0.9
    Y, dates = _rand_stack(rng, N, P, k, miss=0.6, noise=0.05)
    out = oracle.monitor(Y, dates, n, k, hf, lam)
    X = _design(dates, k)
    checked = flat = 0
    for p in range(P):
        if out["deg_reason"][p] != 0:
            continue
        ok = ~np.isnan(Y[:, p])
        I = np.nonzero(ok)[0]
        nbar = int((I < n).sum())
        beta = np.linalg.lstsq(X[I[:nbar]], Y[I[:nbar], p].astype(np.float64), rcond=None)[0]
        r = Y[I, p].astype(np.float64) - X[I] @ beta
        sig = math.sqrt((r[:nbar] ** 2).sum() / (nbar - X.shape[1]))
        h = int(np.float32(nbar) * np.float32(hf))
        J = len(I) - nbar
        m = np.array([r[nbar + j - h + 1: nbar + j + 1].sum() for j in range(J)]) / (sig * math.sqrt(nbar))
        x = (nbar + 1 + np.arange(J)) / nbar
        B = lam * np.sqrt(np.maximum(1.0, np.log(x)))
        flat += int((x > math.e).any())
        ratio = np.abs(m) / B
        hit = np.nonzero(np.abs(m) > B)[0]
        jstar = hit[0] if hit.size else J - 1
        assert out["max_ratio"][p] == pytest.approx(ratio.max(), rel=1e-6)
        assert out["near_tie"][p] == int((np.abs(ratio[:jstar + 1] - 1) <= 1e-3).any())
        checked += 1
    assert checked >= 20 and flat >= 10


# ---------------------------------------------------------------- P2
def test_p2_boundary_table(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "p2_boundary.json")))
    got = [oracle.boundary(g["lambda"], g["nbar"], j) for j in range(len(g["expected"]))]
    np.testing.assert_allclose(got, g["expected"], rtol=1e-14)
    # log+ switches exactly at t/nbar = e (reading R6): below e the bound is lambda
    assert oracle.boundary(2.0, 100, 170) == 2.0          # 271/100 < e
    assert oracle.boundary(2.0, 100, 171) > 2.0           # 272/100 > e


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("k", [0, 1, 2, 3])
def test_p3_fit_matches_lapack_lstsq(k):
    rng = np.random.default_rng(30 + k)
    N, P, n = 40, 64, 24
    Y, dates = _rand_stack(rng, N, P, k, miss=0.3)
    out = oracle.monitor(Y, dates, n, k, 0.25, 1.65)
    X = _design(dates, k)
    checked = 0
    for p in range(P):
        if out["deg_reason"][p] in (1, 2, 3, 4):
            continue
        rows = ~np.isnan(Y[:n, p])
        ref, *_ = np.linalg.lstsq(X[:n][rows], Y[:n, p][rows].astype(np.float64), rcond=None)
        scale = np.abs(X[:n][rows]).max(axis=0)
        err = np.abs(out["beta"][p] - ref) * scale
        assert err.max() <= 1e-9 * max(1.0, np.abs(ref * scale).max()), (p, err)
        # sigma from the lstsq residuals
        res = Y[:n, p][rows] - X[:n][rows] @ ref
        sig = math.sqrt((res ** 2).sum() / (rows.sum() - X.shape[1]))
        assert out["sigma"][p] == pytest.approx(sig, rel=1e-8)
        checked += 1
    assert checked > P // 2


def test_p3_gauss_jordan_inverse_vs_numpy():
    rng = np.random.default_rng(3)
    for K in (2, 4, 8, 14):
        A = rng.normal(size=(3 * K, K))
        M = A.T @ A
        Minv, cond = oracle.gauss_jordan_inverse(M)
        np.testing.assert_allclose(Minv @ M, np.eye(K), atol=1e-9)
        d = 1 / np.sqrt(np.diag(M))
        S = M * d[:, None] * d[None, :]
        assert cond == pytest.approx(np.linalg.cond(S, 1), rel=1e-8)
    # singular -> None (rank test of reading R4)
    A = rng.normal(size=(10, 3))
    A = np.concatenate([A, A[:, :1] * 2.0], axis=1)
    Minv, _ = oracle.gauss_jordan_inverse(A.T @ A)
    assert Minv is None


# ---------------------------------------------------------------- P4
def test_p4_mosum_direct_vs_prefix_and_fig12_scan():
    rng = np.random.default_rng(4)
    for trial in range(50):
        Nbar = int(rng.integers(4, 60))
        nbar = int(rng.integers(2, Nbar))
        h = int(rng.integers(1, nbar + 1))
        r = rng.normal(size=Nbar)
        sigma = float(rng.uniform(0.1, 2))
        m = oracle.mosum(r, nbar, Nbar, h, sigma)
        # prefix-difference form: S[c] = sum_{i<c} r_i
        S = np.concatenate([[0.0], np.cumsum(r)])
        pref = np.array([S[nbar + j + 1] - S[nbar + j - h + 1] for j in range(Nbar - nbar)])
        np.testing.assert_allclose(m, pref / (sigma * math.sqrt(nbar)), rtol=1e-10, atol=1e-12)
        # Fig. 12: m^fst = sum_{i<h} r[i+nbar-h+1]; then scan of
        # r[nbar+t] - r[nbar-h+t]
        mfst = sum(r[i + nbar - h + 1] for i in range(h))
        inc = [mfst] + [r[nbar + t] - r[nbar - h + t] for t in range(1, Nbar - nbar)]
        np.testing.assert_allclose(m, np.cumsum(inc) / (sigma * math.sqrt(nbar)), rtol=1e-9, atol=1e-12)


# ---------------------------------------------------------------- P5
def _run(Y, dates, n, k, hf=0.25, lam=1.65):
    return oracle.monitor(Y, dates, n, k, hf, lam)


def test_p5_normal_equations_residual_orthogonality():
    rng = np.random.default_rng(51)
    Y, dates = _rand_stack(rng, 60, 16, 2, miss=0.4)
    n = 30
    X = _design(dates, 2)
    for p in range(16):
        Nbar, vs, ks = oracle.filter_missing(Y[:, p])
        nbar = int((~np.isnan(Y[:n, p])).sum())
        beta = oracle.fit(X[ks[:Nbar]], vs[:Nbar], nbar)
        if beta is None:
            continue
        r = vs[:nbar] - X[ks[:nbar]] @ beta
        assert abs(r.sum()) < 1e-9                       # intercept column
        np.testing.assert_allclose(X[ks[:nbar]].T @ r, 0, atol=1e-7)


def test_p5_offset_scale_nan_payload_permutation():
    rng = np.random.default_rng(52)
    N, P, n, k = 80, 48, 40, 2
    Y, dates = _rand_stack(rng, N, P, k, miss=0.35)
    base = _run(Y, dates, n, k)
    ok = base["break"] != -2
    assert ok.sum() > P // 2
    # (ii) offset: only beta_0 moves (by C)
    Y2 = (Y.astype(np.float64) + 0.5).astype(np.float32)
    o2 = _run(Y2, dates, n, k)
    # Y + 0.5 is rounded to f32, so compare with tolerance
    np.testing.assert_allclose(o2["beta"][ok, 0], base["beta"][ok, 0] + 0.5, atol=1e-5)
    np.testing.assert_allclose(o2["magnitude"][ok], base["magnitude"][ok], atol=1e-4)
    # (iii) scale by a power of two: exact in f32, so results scale exactly
    Y3 = Y * np.float32(4.0)
    o3 = _run(Y3, dates, n, k)
    np.testing.assert_array_equal(o3["break"], base["break"])
    np.testing.assert_allclose(o3["magnitude"][ok], base["magnitude"][ok], rtol=1e-12)
    np.testing.assert_allclose(o3["sigma"][ok], 4 * base["sigma"][ok], rtol=1e-12)
    np.testing.assert_allclose(o3["beta"][ok], 4 * base["beta"][ok], rtol=1e-10, atol=1e-12)
    # (iv) NaN payloads: negative quiet NaN and a signalling-pattern NaN
    bits = Y.view(np.uint32).copy()
    nanpos = np.isnan(Y)
    alt = np.where(rng.random(Y.shape) < 0.5, np.uint32(0xFFC00001), np.uint32(0x7F800001))
    bits[nanpos] = alt[nanpos]
    o4 = _run(bits.view(np.float32), dates, n, k)
    np.testing.assert_array_equal(o4["break"], base["break"])
    np.testing.assert_array_equal(o4["magnitude"][ok], base["magnitude"][ok])
    # (v) permutation of pixels permutes outputs
    perm = rng.permutation(P)
    o5 = _run(np.ascontiguousarray(Y[:, perm]), dates, n, k)
    np.testing.assert_array_equal(o5["break"], base["break"][perm])
    np.testing.assert_array_equal(o5["magnitude"], base["magnitude"][perm])


def test_p5_nan_free_shared_inverse():
    """(vi) no NaN: every pixel shares Mbar, so beta = (X^T X)^-1 X^T Y for all
    pixels at once -- the special case of prior work [27] (L93)."""
    rng = np.random.default_rng(53)
    N, P, n, k = 50, 32, 30, 3
    Y, dates = _rand_stack(rng, N, P, k, miss=0.0)
    out = _run(Y, dates, n, k)
    X = _design(dates, k)[:n]
    B = np.linalg.solve(X.T @ X, X.T @ Y[:n].astype(np.float64)).T
    scale = np.abs(X).max(axis=0)
    np.testing.assert_allclose(out["beta"] * scale, B * scale, atol=1e-8)


def test_p5_k0_closed_form_linear_regression():
    """(vii) k = 0: slope = S_ty / S_tt, intercept = ybar - slope tbar."""
    rng = np.random.default_rng(54)
    N, P, n = 30, 20, 15
    Y, dates = _rand_stack(rng, N, P, 0, miss=0.3)
    out = _run(Y, dates, n, 0)
    for p in range(P):
        if out["break"][p] == -2:
            continue
        t = np.arange(1, n + 1)[~np.isnan(Y[:n, p])].astype(np.float64)
        y = Y[:n, p][~np.isnan(Y[:n, p])].astype(np.float64)
        slope = ((t - t.mean()) * (y - y.mean())).sum() / ((t - t.mean()) ** 2).sum()
        icpt = y.mean() - slope * t.mean()
        assert out["beta"][p][1] == pytest.approx(slope, rel=1e-9, abs=1e-12)
        assert out["beta"][p][0] == pytest.approx(icpt, rel=1e-9, abs=1e-12)


# ---------------------------------------------------------------- P6
def test_p6_injected_breaks_are_found_at_the_first_valid_date_after_t0():
    """A step of -delta at t0 with delta >> lambda sigma sqrt(nbar) + 6 sigma
    sqrt(h): the first window containing a post-break residual crosses, so
    the break is the first valid date >= t0 (offset from n), unless the
    MOSUM already crossed earlier (a false alarm; the estimation error of the
    extrapolated trend makes these possible, so they are counted, not
    forbidden, and must stay rare)."""
    from paper_conf_icde_giesekerhvo20_b200 import synth
    spec = synth.StackSpec(P=1024, N=200, n_hist=100, k=3, miss=0.4, mask="iid",
                           break_frac=1.0, seed=6, noise_lo=0.0005, noise_hi=0.001)
    Y, dates, truth = synth.generate(spec, "cpu", return_truth=True)
    lam = 6.0
    out = oracle.monitor(Y.numpy(), dates, spec.n_hist, 3, spec.hf, lam)
    Yn = Y.numpy()
    t0 = truth["t0"].numpy()
    checked = early = 0
    for p in range(spec.P):
        if out["break"][p] == -2:
            continue
        valid_after = np.nonzero(~np.isnan(Yn[t0[p]:, p]))[0]
        if 0 <= out["break"][p] < t0[p] - spec.n_hist:
            early += 1
            continue
        if len(valid_after) == 0:
            assert out["break"][p] == -1
            continue
        assert out["break"][p] == t0[p] + valid_after[0] - spec.n_hist, p
        checked += 1
    assert checked > 900 and early <= 10


def test_p6_no_break_no_alarm_with_large_lambda():
    from paper_conf_icde_giesekerhvo20_b200 import synth
    spec = synth.StackSpec(P=256, N=120, n_hist=60, k=2, miss=0.3, break_frac=0.0, seed=7)
    Y, dates = synth.generate(spec, "cpu")
    out = oracle.monitor(Y.numpy(), dates, 60, 2, 0.25, 6.0)
    assert ((out["break"] == -1) | (out["break"] == -2)).all()
    assert (out["break"] == -1).sum() > 200


# ---------------------------------------------------------------- P7
def test_p7_degenerate_table():
    rng = np.random.default_rng(7)
    N, n, k = 46, 23, 1                      # K = 4
    dates = 2000.0 + np.arange(1, N + 1) / 23.0
    X = _design(dates, k)
    clean = (X @ np.array([0.5, 0.001, 0.1, -0.05]) + rng.normal(scale=0.02, size=N)).astype(np.float32)
    cols, want = [], []

    def add(y, reason):
        cols.append(y.astype(np.float32)); want.append(reason)

    add(np.full(N, np.nan), 1)                               # all NaN
    y = clean.copy(); y[:n][4:] = np.nan; add(y, 1)          # nbar = K
    y = clean.copy(); y[:n][5:] = np.nan; add(y, 0)          # nbar = K+1, h = 1
    y = clean.copy(); y[n:] = np.nan; add(y, 3)              # no monitoring data
    # an exact fit: the constant 0.5 is in the model, sigma-hat is fp64
    # rounding residue (reading R4: <= 1e-10 max|y| -> invalid)
    add(np.full(N, 0.5, np.float32), 5)
    # noise-free but fp32-rounded: sigma-hat ~ 3e-8 max|y| is a value, the
    # pixel is valid (R4 is a rule on exactness, not on fp32 resolution)
    rounded = (X @ np.array([0.25, 0.0, 0.125, 0.0])).astype(np.float32)
    add(rounded, 0)
    # rank deficiency: valid history dates congruent mod 23 -> sin/cos constant
    N2 = 23 * 12
    dates2 = 2000.0 + np.arange(1, N2 + 1) / 23.0
    X2 = _design(dates2, k)
    y2 = (X2 @ np.array([0.5, 0.001, 0.1, -0.05]) + rng.normal(scale=0.02, size=N2)).astype(np.float32)
    n2 = N2 // 2
    y2[:n2][np.arange(n2) % 23 != 0] = np.nan               # 6 valid, all same phase
    o = oracle.monitor(y2[:, None], dates2, n2, k, 1.0, 1.65)
    assert o["deg_reason"][0] == 4 and o["break"][0] == -2 and np.isnan(o["magnitude"][0])
    Y = np.stack(cols, axis=1)
    out = oracle.monitor(Y, dates, n, k, 0.25, 1.65)
    assert list(out["deg_reason"]) == want
    ymax = float(np.nanmax(np.abs(rounded[:n])))
    assert out["sigma"][4] <= 1e-10 * 0.5
    assert 1e-9 * ymax < out["sigma"][5] < 1e-6 * ymax
    for i, w in enumerate(want):
        if w:
            assert out["break"][i] == -2 and np.isnan(out["magnitude"][i])
        else:
            assert out["break"][i] >= -1 and np.isfinite(out["magnitude"][i])
    # h < 1: hf small enough that floor(hf * nbar) = 0
    o = oracle.monitor(clean[:, None], dates, n, k, 0.04, 1.65)
    assert o["deg_reason"][0] == 2


def test_p7_window_width_is_f32_product():
    """Fig. 12: h = t32((r32 nbar) * hf) evaluated in f32 (reading R3).
    With hf = 0.7f and nbar = 10 the f32 product rounds to 7.0 although the
    exact product 6.99999988... floors to 6."""
    assert int(np.float32(10) * np.float32(0.7)) == 7
    N, n = 40, 20
    dates = np.arange(1, N + 1) / 23.0
    rng = np.random.default_rng(8)
    y = (0.5 + rng.normal(scale=0.05, size=N)).astype(np.float32)
    y[:n][10:] = np.nan                                       # nbar = 10
    o = oracle.monitor(y[:, None], dates, n, 0, 0.7, 1.65)
    assert o["nbar"][0] == 10 and o["h"][0] == 7


# ---------------------------------------------------------------- P8
def test_p8_scatter_example(golden_dir):
    g = json.load(open(os.path.join(golden_dir, "p8_scatter.json")))
    assert list(oracle.scatter(g["x"], g["is"], g["vs"])) == g["expected"]


def test_filter_missing_is_order_preserving():
    y = np.array([np.nan, 2, 3, np.nan, np.nan, 6, 7, np.nan], np.float32)
    Nbar, vs, ks = oracle.filter_missing(y)
    assert Nbar == 4
    assert list(vs[:4]) == [2, 3, 6, 7] and np.isnan(vs[4:]).all()
    assert list(ks[:4]) == [1, 2, 5, 6] and (ks[4:] == 0).all()


def test_design_row_order_sin_before_cos():
    d = np.array([0.1, 0.35])
    x = oracle.design_row(d, 1, 2)
    np.testing.assert_allclose(x, [1, 2, math.sin(TWO_PI * 0.35), math.cos(TWO_PI * 0.35),
                                   math.sin(2 * TWO_PI * 0.35), math.cos(2 * TWO_PI * 0.35)])


def test_p10_drop_empty_dates_brute_force():
    """f2 (L291, L379): the kept slices of the oracle's date filter against a
    loop over every element, on a stack built to trip the plausible mistakes:
    values only in the padding columns (>= P) of an otherwise empty slice,
    non-canonical NaN payloads, empty slices at n-1 and n (the history count
    n_hist' of the compacted stack), a slice whose only value is the last
    pixel."""
    rng = np.random.default_rng(11)
    N, P, ldY, n = 40, 37, 44, 20
    Y = rng.normal(size=(N, ldY)).astype(np.float32)
    Y[rng.random((N, ldY)) < 0.5] = np.nan
    empty = [0, 3, n - 1, n, 31, N - 1]
    Y[empty, :P] = np.nan
    Y[3, P:] = 1.0                      # values only in the padding
    bits = Y.view(np.uint32)
    bits[31, :P] = np.uint32(0xFFC00001)  # negative, non-canonical NaNs
    Y[7, :P] = np.nan
    Y[7, P - 1] = 2.5                   # only the last pixel
    dates = np.arange(1, N + 1) / 23.0 + 2000.0
    Yc, dc, nc, keep = oracle.drop_empty_dates(Y, dates, n, P=P)
    brute = []
    for t in range(N):
        has = False
        for p in range(P):
            v = float(Y[t, p])
            if v == v:
                has = True
                break
        if has:
            brute.append(t)
    assert keep.tolist() == brute
    assert set(empty).isdisjoint(brute) and 7 in brute
    assert nc == sum(1 for t in brute if t < n) == n - 3
    assert np.array_equal(Yc.view(np.uint32), Y[brute, :P].view(np.uint32))
    assert np.array_equal(dc, dates[brute])


def test_p11_decode_i16_is_one_rounding_of_the_exact_value():
    """f4 (reading R15): every int16 code decodes to the fp32 nearest the
    exact scale*code + offset (a multiply-then-add in fp32, two roundings,
    misses it for some codes), the nodata code to NaN; a power-of-two scale
    is exact."""
    from fractions import Fraction
    codes = np.arange(-32768, 32768, dtype=np.int64).astype(np.int16)
    scale, offset = np.float32(1e-4), np.float32(0.1)
    y = oracle.decode_i16(codes, scale, offset, -32768)
    assert np.isnan(y[0]) and not np.isnan(y[1:]).any()
    fs, fo = Fraction(float(scale)), Fraction(float(offset))
    up = np.nextafter(y, np.float32(np.inf))
    dn = np.nextafter(y, np.float32(-np.inf))
    bad = 0
    for i in range(1, len(codes), 7):
        ex = fs * int(codes[i]) + fo
        e0 = abs(Fraction(float(y[i])) - ex)
        if e0 > abs(Fraction(float(up[i])) - ex) or e0 > abs(Fraction(float(dn[i])) - ex):
            bad += 1
    assert bad == 0
    two = (codes[1:].astype(np.float32) * scale + offset).astype(np.float32)  # two roundings
    assert np.any(two != y[1:])
    y2 = oracle.decode_i16(codes, np.float32(2.0 ** -14), np.float32(0.5), 7)
    ok = codes != 7
    assert np.array_equal(y2[ok].astype(np.float64), codes[ok].astype(np.float64) * 2.0 ** -14 + 0.5)
    assert np.isnan(y2[~ok]).all()


def test_p12_periods_use_only_their_own_dates():
    """f1 (L391): a period (n_i, N_i) is Algorithm 1 on the first N_i dates:
    its result does not change when every date at or after N_i is replaced,
    and the period ending at N equals the single-period oracle."""
    rng = np.random.default_rng(12)
    N, P = 160, 300
    dates = 2000.0 + np.arange(1, N + 1) / 23.0
    t = np.arange(N)[:, None]
    Y = (0.5 + 0.1 * np.sin(2 * np.pi * dates)[:, None] + 0.02 * rng.normal(size=(N, P))).astype(np.float32)
    Y[rng.random((N, P)) < 0.3] = np.nan
    Y -= (np.float32(0.3) * ((t >= 120) & (rng.random(P) < 0.5)[None, :])).astype(np.float32)
    periods = [(80, 103), (103, 126), (126, 160)]
    res = oracle.monitor_periods(Y, dates, periods, 3, 0.25, 1.65)
    Y2 = Y.copy()
    Y2[103:] = np.float32(7.0)
    r2 = oracle.monitor_periods(Y2, dates, periods[:1], 3, 0.25, 1.65)[0]
    for key in ("break", "magnitude", "sigma", "nbar"):
        np.testing.assert_array_equal(res[0][key], r2[key])
    full = oracle.monitor(Y, dates, 126, 3, 0.25, 1.65)
    for key in ("break", "magnitude", "nbar"):
        np.testing.assert_array_equal(res[2][key], full[key])
    assert (res[2]["break"] >= 0).sum() > 50  # the step at t = 120 is inside period 3 only
