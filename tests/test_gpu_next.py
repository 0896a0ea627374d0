"""GPU parity of the SURVEY.md 8(f) NEXT rows built in round 2.

f3  NaN-free histories share one Gram (the [27] special case):
    its factor is computed once on the host in fp64; every warp whose 32
    histories are complete skips its own factorisation.
f2  all-NaN date slices dropped before the hot path (L291, L379): the scan
    and gather kernels, bit-exact against numpy, and the monitoring result on
    the compacted stack against the oracle on the same compacted stack.

Every case compares the CUDA path (through the C ABI) with the fp64 oracle on
the same device bytes (oracle/parity.py tolerances).
"""
import json

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from oracle import parity
from paper_conf_icde_giesekerhvo20_b200 import binding, synth

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _compare(out, Y, dates, n, k, hf, lam):
    orc = oracle.monitor(np.ascontiguousarray(Y.cpu().numpy()), dates, n, k, hf, lam)
    gpu = {key: v.cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
    rep = parity.compare(gpu, orc, dates, n, k)
    assert rep["ok"], json.dumps(rep)
    np.testing.assert_array_equal(gpu["nbar"], orc["nbar"])
    return rep, gpu, orc


def _dense_history(spec, dense_cols=None):
    """i.i.d. gaps in the monitoring period only (or, with dense_cols, a
    complete history only for those columns): the mask-free draw of the same
    seed supplies the history values (synth draws the mask after the values)."""
    Y, dates = synth.generate(spec, DEV)
    Y0, _ = synth.generate(synth.StackSpec(**{**spec.asdict(), "mask": "none"}), DEV)
    ok = ~torch.isnan(Y)
    assert torch.equal(Y[ok], Y0[ok])
    cols = slice(None) if dense_cols is None else dense_cols
    Y[: spec.n_hist, cols] = Y0[: spec.n_hist, cols]
    return Y, dates


@pytest.mark.parametrize("shared", ["1", "0"])
@pytest.mark.parametrize("N,k", [(228, 3), (400, 3), (250, 5), (100, 1), (1000, 2)])
def test_f3_nan_free_history(N, k, shared, monkeypatch):
    monkeypatch.setenv("BFAST_SHARED_FACTOR", shared)
    spec = synth.StackSpec(P=20_000 + 37, N=N, n_hist=N // 2, k=k, miss=0.3, mask="iid", seed=700 + N + k)
    Y, dates = _dense_history(spec)
    out = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    rep, gpu, _ = _compare(out, Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    assert np.all(gpu["nbar"] == spec.n_hist)
    assert rep["breaks_oracle"] > 0


def test_f3_mixed_warps_and_paths_agree(monkeypatch):
    """Half the columns with a complete history, half with gaps: warps of
    either kind (and the boundary warp) in one launch; the shared-factor and
    per-pixel-factor runs agree to fp32 rounding and both match the oracle."""
    spec = synth.StackSpec(P=40_000, N=400, n_hist=200, miss=0.5, mask="iid", seed=733)
    Y, dates = _dense_history(spec, dense_cols=slice(0, 20_011))
    res = {}
    for shared in ("1", "0"):
        monkeypatch.setenv("BFAST_SHARED_FACTOR", shared)
        out = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
        torch.cuda.synchronize()
        _compare(out, Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
        res[shared] = {key: v.cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
    a, b = res["1"], res["0"]
    np.testing.assert_array_equal(a["nbar"], b["nbar"])
    same = a["break"] == b["break"]
    assert same.mean() > 0.9999
    fin = np.isfinite(a["magnitude"])
    assert np.max(np.abs(a["magnitude"][fin] - b["magnitude"][fin]) / np.maximum(1, np.abs(b["magnitude"][fin]))) < 1e-4


def _stack_with_empty_slices(P, ldY, N, n, seed, frac_empty=0.4):
    """A stack with a share of all-NaN date slices (the Africa case, L379),
    padding columns holding values, and a slice whose only value is the last
    pixel."""
    spec = synth.StackSpec(P=P, N=N, n_hist=n, miss=0.4, mask="iid", seed=seed)
    Y, dates = synth.generate(spec, DEV, ldY=ldY)
    rng = np.random.default_rng(seed)
    empty = np.sort(rng.choice(np.arange(1, N - 1), size=int(frac_empty * N), replace=False))
    Y[torch.from_numpy(empty).to(DEV), :P] = float("nan")
    if ldY > P:
        Y[torch.from_numpy(empty).to(DEV), P:] = 3.0  # values outside the P pixels do not count
    Y[N - 1, :P] = float("nan")
    Y[N - 1, P - 1] = 0.5
    return spec, Y, dates


@pytest.mark.parametrize("P,ldY", [(50_000, 50_000), (40_001, 40_007), (3, 8), (300_000, 300_004)])
def test_f2_valid_dates_and_gather_bit_exact(P, ldY):
    spec, Y, dates = _stack_with_empty_slices(P, ldY, 160, 80, seed=900 + P % 97)
    keep = binding.bfast_valid_dates(Y, P=P).cpu().numpy()
    assert binding.last_launch_count() == 1
    _, _, _, keep_idx = oracle.drop_empty_dates(Y.cpu().numpy(), dates, spec.n_hist, P=P)
    assert np.flatnonzero(keep).tolist() == keep_idx.tolist()
    idx = torch.from_numpy(keep_idx.astype(np.int32)).to(DEV)
    Yc = binding.bfast_gather_dates(Y, idx, P=P)
    torch.cuda.synchronize()
    ref = Y[idx.long(), :P]
    assert torch.equal(Yc.view(torch.int32), ref.contiguous().view(torch.int32))


def test_f2_monitoring_on_the_compacted_stack():
    """drop_empty_dates + the hot path = the oracle run on the oracle's own
    compacted stack; break offsets map back to a valid original date."""
    spec, Y, dates = _stack_with_empty_slices(30_000, 30_000, 400, 200, seed=931, frac_empty=0.5)
    Yc, dc, nc, keep_idx = binding.drop_empty_dates(Y, dates, spec.n_hist)
    Yo, do, nco, ko = oracle.drop_empty_dates(Y.cpu().numpy(), dates, spec.n_hist)
    assert nc == nco and np.array_equal(keep_idx, ko) and np.array_equal(dc, do)
    out = binding.bfast_monitor_ex(Yc, dc, nc, spec.k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    assert np.array_equal(Yc.cpu().numpy().view(np.uint32), Yo.view(np.uint32))
    rep, gpu, orc = _compare(out, Yc, dc, nc, spec.k, spec.hf, spec.lam)
    ob = binding.original_break_offsets(gpu["break"], keep_idx, nc, spec.n_hist)
    hit = np.flatnonzero(ob >= 0)
    assert len(hit) > 100
    Yh = Y.cpu().numpy()
    assert np.all(~np.isnan(Yh[spec.n_hist + ob[hit], hit]))  # the break date holds the pixel's value
    assert np.all(ob[gpu["break"] < 0] == gpu["break"][gpu["break"] < 0])


def test_f2_tile_level_resume_is_identical():
    """A scene streamed from host memory in tiles, interrupted after two
    tiles and resumed, gives the bytes of one uninterrupted call."""
    spec = synth.StackSpec(P=300_000, N=228, n_hist=114, miss=0.5, mask="iid", seed=955)
    Y, dates = synth.generate(spec, DEV)
    Yh = Y.cpu().pin_memory()
    b1, m1 = binding.bfast_monitor_host(Yh, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    b2 = np.full(spec.P, 7, np.int32)
    m2 = np.full(spec.P, 7.0, np.float32)
    done = binding.bfast_monitor_host_resume(Yh, dates, spec.n_hist, spec.k, spec.hf, spec.lam, b2, m2,
                                             done=0, tile=70_000, max_tiles=2)
    assert done == 140_000 and np.all(b2[done:] == 7)
    done = binding.bfast_monitor_host_resume(Yh, dates, spec.n_hist, spec.k, spec.hf, spec.lam, b2, m2,
                                             done=done, tile=70_000)
    assert done == spec.P
    np.testing.assert_array_equal(b1, b2)
    np.testing.assert_array_equal(m1.view(np.uint32), m2.view(np.uint32))


@pytest.mark.parametrize("N,n,k,mask,miss,scale,offset,nodata,P,ldY", [
    (228, 114, 3, "iid", 0.5, 1e-4, 0.0, -32768, 30_000, 30_000),      # tails of both periods (n % 16 = 2)
    (400, 200, 3, "cloud", 0.6, 2e-4, -1.0, 0, 50_000, 50_008),        # nodata mid-range, padding columns
    (250, 125, 5, "iid", 0.5, -1.5e-4, 0.25, 32767, 20_000, 20_000),  # negative scale: MOSUM sign flips
    (100, 50, 1, "iid", 0.9, 1e-4, 0.0, -32768, 20_000, 20_000),       # mostly degenerate pixels
])
def test_f4_int16_codec_parity(N, n, k, mask, miss, scale, offset, nodata, P, ldY):
    """f4: the hot path on int16 codes against the oracle on the decoded
    stack (oracle.decode_i16: fmaf(scale, code, offset), nodata -> NaN)."""
    spec = synth.StackSpec(P=P, N=N, n_hist=n, k=k, miss=miss, mask=mask, seed=1300 + N + k)
    Y, dates = synth.generate(spec, DEV, ldY=ldY)
    codes = synth.quantize_i16(Y, scale, offset, nodata)
    out = binding.bfast_monitor_i16(codes, dates, n, k, spec.hf, spec.lam, scale, offset, nodata, P=P,
                                    diagnostics=True)
    torch.cuda.synchronize()
    assert binding.last_launch_count() >= 2
    Yd = oracle.decode_i16(codes[:, :P].cpu().numpy(), np.float32(scale), np.float32(offset), nodata)
    orc = oracle.monitor(np.ascontiguousarray(Yd), dates, n, k, spec.hf, spec.lam)
    gpu = {key: v.cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
    rep = parity.compare(gpu, orc, dates, n, k)
    assert rep["ok"], json.dumps(rep)
    np.testing.assert_array_equal(gpu["nbar"], orc["nbar"])


def test_f4_int16_rejects_misaligned_rows():
    spec = synth.StackSpec(P=1000, N=100, n_hist=50, miss=0.3, seed=3)
    Y, dates = synth.generate(spec, DEV, ldY=1004)
    codes = synth.quantize_i16(Y, 1e-4, 0.0)
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_i16(codes, dates, 50, 3, 0.25, 1.65, 1e-4, 0.0, -32768, P=1000)
    assert e.value.status == -2  # BFAST_EUNSUPPORTED: TMA rows need ldY % 8 == 0


def _yearly(n0, M, year=23):
    return [(n0 + year * i, n0 + year * (i + 1)) for i in range(M)]


@pytest.mark.parametrize("N,periods,k,mask", [
    (400, _yearly(230, 7), 3, "cloud"),                              # L391: yearly periods from 2010
    (228, [(114, 228), (100, 180), (60, 77), (150, 201)], 1, "iid"),  # unordered, partial chunks
    (320, _yearly(120, 8), 5, "iid"),                               # the maximum of 8 periods
])
def test_f1_several_periods_in_one_launch(N, periods, k, mask, monkeypatch):
    """Every period against the oracle on its own date slice (the MOSUM ring
    sized from a sample: wider windows refitted in fp64), and -- both with
    the full ring (BFAST_WINDOW_PROBE=0), so that the same pixels take the
    same path -- bit-equal to a separate single-period run."""
    spec = synth.StackSpec(P=20_000 + 11, N=N, n_hist=periods[0][0], k=k, miss=0.5, mask=mask, seed=1500 + N + k)
    Yp, dates = synth.generate(spec, DEV, ldY=20_016)  # TMA rows: ldY % 4 == 0; a ragged last tile
    Y = Yp[:, :spec.P]
    out = binding.bfast_monitor_periods(Y, dates, periods, k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    assert binding.last_launch_count() == 1 + len(periods)
    Yh = np.ascontiguousarray(Y.cpu().numpy())
    orcs = oracle.monitor_periods(Yh, dates, periods, k, spec.hf, spec.lam)
    for i, ((n_i, N_i), orc) in enumerate(zip(periods, orcs)):
        gpu = {key: v[i].cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
        rep = parity.compare(gpu, orc, dates[:N_i], n_i, k)
        assert rep["ok"], (i, json.dumps(rep))
        np.testing.assert_array_equal(gpu["nbar"], orc["nbar"])
    monkeypatch.setenv("BFAST_WINDOW_PROBE", "0")
    full = binding.bfast_monitor_periods(Y, dates, periods, k, spec.hf, spec.lam)
    for i, (n_i, N_i) in enumerate(periods):
        single = binding.bfast_monitor_ex(Y[:N_i], dates[:N_i], n_i, k, spec.hf, spec.lam)
        torch.cuda.synchronize()
        assert torch.equal(single["break"], full["break"][i])
        assert torch.equal(single["magnitude"].view(torch.int32), full["magnitude"][i].view(torch.int32))


def test_f1_split_schedule_is_bit_identical(monkeypatch):
    """BFAST_PERIODS=split (one launch per period) gives the bytes of the
    one-pass launch."""
    spec = synth.StackSpec(P=30_000, N=400, n_hist=230, miss=0.6, mask="cloud", seed=1577)
    Y, dates = synth.generate(spec, DEV)
    per = _yearly(230, 5)
    a = binding.bfast_monitor_periods(Y, dates, per, 3, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    assert binding.last_launch_count() == 1 + len(per)
    monkeypatch.setenv("BFAST_PERIODS", "split")
    b = binding.bfast_monitor_periods(Y, dates, per, 3, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    assert binding.last_launch_count() == 2 * len(per)
    for key in ("break", "magnitude", "beta", "sigma", "nbar"):
        assert torch.equal(a[key].view(torch.int32) if a[key].dtype == torch.float32 else a[key],
                           b[key].view(torch.int32) if b[key].dtype == torch.float32 else b[key]), key


def test_f1_rejects_bad_period_sets():
    spec = synth.StackSpec(P=1000, N=200, n_hist=100, miss=0.3, seed=5)
    Y, dates = synth.generate(spec, DEV)
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_periods(Y, dates, [(50 + i, 150 + i) for i in range(9)], 3, 0.25, 1.65)
    assert e.value.status == -2
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_periods(Y, dates, [(100, 150), (100, 150)], 3, 0.25, 1.65)
    assert e.value.status == -1
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_periods(Y, dates, [(100, 201)], 3, 0.25, 1.65)
    assert e.value.status == -1


def test_f2_edge_cases():
    """An all-empty stack keeps no date; P = 0 and Nc = 0 are no-ops; a stack
    without empty slices keeps every date."""
    spec = synth.StackSpec(P=5000, N=64, n_hist=32, miss=0.3, seed=961)
    Y, dates = synth.generate(spec, DEV)
    keep = binding.bfast_valid_dates(Y).cpu().numpy()
    assert keep.tolist() == [1] * 64
    Yn = torch.full_like(Y, float("nan"))
    assert binding.bfast_valid_dates(Yn).cpu().numpy().sum() == 0
    Yc, dc, nc, kept = binding.drop_empty_dates(Yn, dates, spec.n_hist)
    assert Yc.shape == (0, spec.P) and nc == 0 and len(kept) == 0
    assert binding.bfast_valid_dates(Y, P=0).cpu().numpy().sum() == 0
    bad = torch.tensor([3, 64, -1, 5], dtype=torch.int32, device=DEV)  # indices outside [0, N) -> NaN rows
    Yc = binding.bfast_gather_dates(Y, bad)
    torch.cuda.synchronize()
    assert torch.equal(Yc[0].view(torch.int32), Y[3].view(torch.int32))
    assert torch.equal(Yc[3].view(torch.int32), Y[5].view(torch.int32))
    assert torch.isnan(Yc[1]).all() and torch.isnan(Yc[2]).all()


@pytest.mark.parametrize("k", [4, 5, 6])
def test_f4_int16_wide_designs(k):
    """The int16 kernel at the wide designs (K = 10, 12, 14: fewer tiles per
    CTA, more TMEM per tile)."""
    spec = synth.StackSpec(P=12_000, N=300, n_hist=150, k=k, miss=0.4, mask="iid", seed=1700 + k)
    Y, dates = synth.generate(spec, DEV)
    codes = synth.quantize_i16(Y, 1e-4, 0.0, -32768)
    out = binding.bfast_monitor_i16(codes, dates, 150, k, spec.hf, spec.lam, 1e-4, 0.0, -32768, diagnostics=True)
    torch.cuda.synchronize()
    Yd = oracle.decode_i16(codes.cpu().numpy(), np.float32(1e-4), np.float32(0.0), -32768)
    orc = oracle.monitor(np.ascontiguousarray(Yd), dates, 150, k, spec.hf, spec.lam)
    gpu = {key: v.cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
    rep = parity.compare(gpu, orc, dates, 150, k)
    assert rep["ok"], json.dumps(rep)


def test_f4_int16_long_history_sampled_ring():
    """int16 codes at the Sentinel-2 shape (N = 700, n = 350): the window
    probe reads codes (nodata = missing) to size the ring; parity on a
    sample."""
    spec = synth.StackSpec(P=300_000, N=700, n_hist=350, miss=0.5, mask="iid", f=73.0, year0=2016.0, seed=1811)
    Y, dates = synth.generate(spec, DEV)
    codes = synth.quantize_i16(Y, 1e-4, 0.0, -32768)
    out = binding.bfast_monitor_i16(codes, dates, 350, 3, spec.hf, spec.lam, 1e-4, 0.0, -32768, diagnostics=True)
    torch.cuda.synchronize()
    idx = np.sort(np.random.default_rng(4).choice(spec.P, 20_000, replace=False))
    Yd = oracle.decode_i16(codes[:, torch.from_numpy(idx).to(DEV)].cpu().numpy(), np.float32(1e-4),
                           np.float32(0.0), -32768)
    orc = oracle.monitor(np.ascontiguousarray(Yd), dates, 350, 3, spec.hf, spec.lam)
    gpu = {key: v.cpu().numpy()[idx] for key, v in out.items() if torch.is_tensor(v)}
    rep = parity.compare(gpu, orc, dates, 350, 3)
    assert rep["ok"], json.dumps(rep)


def test_f1_sampled_ring_refits_wider_windows():
    """The multi-period launch sizes its ring from a sample of the longest
    history; complete histories placed outside the sampled 32-pixel groups
    have wider windows in every period and are refitted in fp64 -- all of
    them and a sample of the rest match the oracle, period by period."""
    P = 1 << 18
    spec = synth.StackSpec(P=P, N=400, n_hist=230, miss=0.6, mask="iid", seed=1901)
    Y, dates = synth.generate(spec, DEV)
    Y0, _ = synth.generate(synth.StackSpec(**{**spec.asdict(), "mask": "none"}), DEV)
    gstride = P // 2048
    wide = np.arange(gstride // 2, P, gstride)  # never in a sampled group (the first 32 of each stride)
    it = torch.from_numpy(wide).to(DEV)
    Y[:391, it] = Y0[:391, it]
    per = _yearly(230, 7)
    out = binding.bfast_monitor_periods(Y, dates, per, 3, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    rng = np.random.default_rng(8)
    idx = np.unique(np.concatenate([wide, rng.choice(P, 4000, replace=False)]))
    Ys = np.ascontiguousarray(Y[:, torch.from_numpy(idx).to(DEV)].cpu().numpy())
    orcs = oracle.monitor_periods(Ys, dates, per, 3, spec.hf, spec.lam)
    for i, ((n_i, N_i), orc) in enumerate(zip(per, orcs)):
        gpu = {key: v[i].cpu().numpy()[idx] for key, v in out.items() if torch.is_tensor(v)}
        assert np.all(out["flags"][i].cpu().numpy()[wide] & 2), i
        rep = parity.compare(gpu, orc, dates[:N_i], n_i, 3)
        assert rep["ok"], (i, json.dumps(rep))
