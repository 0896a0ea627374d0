"""GPU-vs-oracle parity through the C ABI (needs a B200).

Inputs are generated on the device by the seeded generator (synth.py, no
method arithmetic), copied to the host and handed to the fp64 oracle, so
both sides consume identical bytes.  Tolerances: oracle/parity.py.
"""
import json
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")

import oracle
from oracle import parity
from paper_conf_icde_giesekerhvo20_b200 import binding, synth

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


@pytest.fixture(params=["fused", "simt"])
def mode(request, monkeypatch):
    """Run the test on the fused tensor-core kernel (monitor_fused.cuh) and on
    the CUDA-core-only kernel (monitor_simt.cuh, the path for stacks whose
    row pitch TMA cannot read)."""
    monkeypatch.setenv("BFAST_KERNEL", request.param)
    return request.param


def _run_both(Y, dates, n, k, hf, lam, P=None):
    out = binding.bfast_monitor_ex(Y, dates, n, k, hf, lam, P=P, diagnostics=True)
    torch.cuda.synchronize()
    P = Y.shape[1] if P is None else P
    gpu = {key: v.cpu().numpy() for key, v in out.items() if hasattr(v, "cpu")}
    Yh = Y[:, :P].cpu().numpy()
    orc = oracle.monitor(np.ascontiguousarray(Yh), dates, n, k, hf, lam)
    return gpu, orc


def _assert_parity(gpu, orc, dates, n, k, **kw):
    rep = parity.compare(gpu, orc, dates, n, k, **kw)
    assert rep["ok"], json.dumps(rep)
    # integer diagnostics are exact
    np.testing.assert_array_equal(gpu["nbar"], orc["nbar"])
    return rep


def test_tiny_config_full_parity(mode):
    spec = synth.CONFIGS["tiny"]
    Y, dates = synth.generate(spec, DEV)
    gpu, orc = _run_both(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    rep = _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)
    assert rep["breaks_oracle"] > 500          # 30% injected breaks are found
    ok = orc["break"] != -2
    np.testing.assert_allclose(gpu["sigma"][ok], orc["sigma"][ok], rtol=1e-4)


@pytest.mark.parametrize("P,ldY", [(1000, 1000), (1000, 1003), (1000, 1004), (129, 132), (1, 1), (31, 64), (384, 384)])
def test_ragged_tails_and_leading_dimension(P, ldY, mode):
    spec = synth.StackSpec(P=P, N=150, n_hist=75, miss=0.45, seed=11 + P)
    Y, dates = synth.generate(spec, DEV, ldY=ldY)
    gpu, orc = _run_both(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, P=P)
    _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)


@pytest.mark.parametrize("k", [0, 1, 2, 3, 4, 5, 6])
def test_all_harmonic_orders(k, mode):
    spec = synth.StackSpec(P=2048, N=240, n_hist=120, k=k, miss=0.4, seed=20 + k)
    Y, dates = synth.generate(spec, DEV)
    gpu, orc = _run_both(Y, dates, spec.n_hist, k, spec.hf, spec.lam)
    _assert_parity(gpu, orc, dates, spec.n_hist, k)


@pytest.mark.parametrize("hf,lam", [(1.0, 1.65), (0.7, 1.0), (0.05, 3.0), (0.5, 0.25)])
def test_window_and_boundary_variants(hf, lam, mode):
    spec = synth.StackSpec(P=2048, N=200, n_hist=60, miss=0.3, seed=31)
    Y, dates = synth.generate(spec, DEV)
    gpu, orc = _run_both(Y, dates, spec.n_hist, spec.k, hf, lam)
    _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)


@pytest.mark.parametrize("N", [100, 250, 500, 1000])
@pytest.mark.parametrize("miss", [0.1, 0.5, 0.9])
@pytest.mark.parametrize("k", [1, 3, 5])
def test_sweep_shapes(N, miss, k, mode):
    """configs[2] shapes at a reduced pixel count (full size: sampled test below)."""
    idx = [100, 250, 500, 1000].index(N) * 9 + [0.1, 0.5, 0.9].index(miss) * 3 + [1, 3, 5].index(k)
    spec = synth.sweep_spec(N, miss, k, P=4096, index=idx)
    Y, dates = synth.generate(spec, DEV)
    gpu, orc = _run_both(Y, dates, spec.n_hist, k, spec.hf, spec.lam)
    _assert_parity(gpu, orc, dates, spec.n_hist, k)


def test_edge_cases_degenerate_pixels(mode):
    N, n, k = 92, 46, 1
    dates = synth.make_dates(N)
    rng = np.random.default_rng(5)
    base = (0.5 + 0.1 * np.sin(2 * np.pi * dates) + rng.normal(scale=0.02, size=N)).astype(np.float32)
    cols = []
    cols.append(np.full(N, np.nan, np.float32))                 # all missing
    y = base.copy(); y[:n][4:] = np.nan; cols.append(y)         # nbar = K
    y = base.copy(); y[:n][5:] = np.nan; cols.append(y)         # nbar = K + 1
    y = base.copy(); y[n:] = np.nan; cols.append(y)             # no monitoring data
    y = base.copy(); y[n:] = np.nan; y[N - 1] = base[N - 1]; cols.append(y)  # one monitoring value
    cols.append(base.copy())                                    # no NaN at all
    cols.append(np.full(N, 0.25, np.float32))                   # constant: sigma = 0
    y = base.copy(); y[n:] -= 1.0; cols.append(y)               # break at the first date
    Y = torch.tensor(np.stack(cols * 32, 1), device=DEV).contiguous()   # 256 px: two full tiles
    gpu, orc = _run_both(Y, dates, n, k, 0.25, 1.65)
    _assert_parity(gpu, orc, dates, n, k)
    assert list(gpu["break"][:4]) == [-2, -2, gpu["break"][2], -2]
    assert gpu["break"][2] != -2 and gpu["break"][6] == -2 and gpu["break"][7] == 0


@pytest.mark.parametrize("N", [1000, 3600])
def test_refit_of_long_series(N, mode):
    """Pixels pushed towards the fp64 refit (an offset of 20 under noise
    0.01-0.05: the fp32 fit's cancellation triggers fire for a share of
    them, none is degenerate by reading R4), on series long enough that the refit
    CTA narrows to fit its per-warp buffers (N = 3600: 2 warps per CTA),
    several per refit warp; compared with the oracle."""
    spec = synth.StackSpec(P=65536, N=N, n_hist=N // 2, k=2, miss=0.5, seed=71)
    Y, dates = synth.generate(spec, DEV)
    Y[:, ::3] += 20.0                            # every third pixel
    try:
        gpu, orc = _run_both(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    except binding.BfastError as e:             # a series the fused kernels cannot hold
        assert e.status == binding.BFAST_EUNSUPPORTED and N > 1000, str(e)
        pytest.skip(str(e))
    assert int(((gpu["flags"][::3] & 2) != 0).sum()) > spec.P // 60   # ~10% measured at N = 1000
    assert int((gpu["break"][::3] == -2).sum()) == 0
    _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)


def test_empty_input_is_a_noop():
    Y = torch.empty((10, 0), device=DEV)
    out = binding.bfast_monitor_ex(Y, synth.make_dates(10), 5, 1, 0.25, 1.65)
    torch.cuda.synchronize()
    assert out["break"].numel() == 0


def test_invalid_arguments_raise():
    Y = torch.zeros((10, 8), device=DEV)
    d = synth.make_dates(10)
    for args in [(0, 1, 0.25, 1.65), (10, 1, 0.25, 1.65), (5, -1, 0.25, 1.65), (5, 1, 0.0, 1.65),
                 (5, 1, 1.5, 1.65), (5, 1, 0.25, 0.0), (5, 1, 0.25, float("nan"))]:
        with pytest.raises(binding.BfastError) as e:
            binding.bfast_monitor_ex(Y, d, *args)
        assert e.value.status == binding.BFAST_EINVAL
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_ex(Y, d[::-1].copy(), 5, 1, 0.25, 1.65)
    assert e.value.status == binding.BFAST_EINVAL
    with pytest.raises(binding.BfastError) as e:
        binding.bfast_monitor_ex(Y, d, 5, 7, 0.25, 1.65)
    assert e.value.status == binding.BFAST_EUNSUPPORTED


def test_host_path_and_multi_match_device_path():
    spec = synth.StackSpec(P=70_000, N=180, n_hist=90, miss=0.5, seed=41)
    Y, dates = synth.generate(spec, DEV)
    dev = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    torch.cuda.synchronize()
    Yh = Y.cpu().pin_memory()
    b, m = binding.bfast_monitor_host(Yh, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    np.testing.assert_array_equal(b, dev["break"].cpu().numpy())
    np.testing.assert_array_equal(m, dev["magnitude"].cpu().numpy())
    ndev = torch.cuda.device_count()
    b2, m2 = binding.bfast_monitor_multi(Yh, dates, spec.n_hist, spec.k, spec.hf, spec.lam,
                                         devices=[i % ndev for i in range(3)])
    np.testing.assert_array_equal(b2, b)
    np.testing.assert_array_equal(m2, m)


def test_plan_execute_is_deterministic_and_stream_ordered(mode):
    spec = synth.StackSpec(P=50_000, N=200, n_hist=100, miss=0.6, mask="cloud", seed=51)
    Y, dates = synth.generate(spec, DEV)
    plan = binding.Plan(0, spec.N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        o1 = plan.execute(Y, diagnostics=True)
        o2 = plan.execute(Y, diagnostics=True)
    s.synchronize()
    for key in ("break", "magnitude", "beta", "sigma", "nbar", "flags"):
        assert torch.equal(o1[key].nan_to_num(), o2[key].nan_to_num()), key
    plan.close()


@pytest.mark.slow
def test_landsat_full_size_sampled_parity(mode):
    """configs[1] at full size (P = 4096^2, N = 400, 60% cloud-masked), in the
    launch configuration bench.py times (Plan.execute on one stream), with
    2^16 sampled pixels checked against the oracle and all-pixel properties."""
    spec = synth.CONFIGS["landsat"]
    Y, dates = synth.generate(spec, DEV)
    plan = binding.Plan(0, spec.N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    out = plan.execute(Y, diagnostics=True)
    torch.cuda.synchronize()
    idx = synth.sample_columns(Y, spec.P, 1 << 16, seed=3)
    it = torch.tensor(idx, device=DEV)
    Ys = Y.index_select(1, it).cpu().numpy()
    orc = oracle.monitor(Ys, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    gpu = {key: v.index_select(0, it).cpu().numpy() for key, v in out.items()}
    rep = _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)
    miss = float(torch.isnan(Y[:, :: 97]).float().mean())
    assert 0.5 < miss < 0.7, miss
    b = out["break"]
    assert int(((b < -2) | (b >= spec.N - spec.n_hist)).sum()) == 0
    assert torch.equal(torch.isnan(out["magnitude"]), b == -2)
    assert rep["breaks_oracle"] > 0.05 * len(idx)
    del Y
    torch.cuda.empty_cache()


@pytest.mark.slow
def test_landsat_every_refitted_pixel_matches_oracle(mode):
    """configs[1] at full size: every pixel the fused kernel handed to the
    fp64 refit (flags bit 1; ~0.1% of the scene, so each refit warp walks
    several items with the next column in flight) against the oracle."""
    spec = synth.CONFIGS["landsat"]
    Y, dates = synth.generate(spec, DEV)
    out = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    it = torch.nonzero((out["flags"].to(torch.int32) & 2) != 0).flatten()
    assert 1000 < it.numel() < spec.P // 100, it.numel()
    Ys = Y.index_select(1, it).cpu().numpy()
    orc = oracle.monitor(Ys, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    gpu = {key: v.index_select(0, it).cpu().numpy() for key, v in out.items() if torch.is_tensor(v)}
    _assert_parity(gpu, orc, dates, spec.n_hist, spec.k)
    del Y
    torch.cuda.empty_cache()


def test_tc_and_simt_paths_agree_closely(monkeypatch):
    """The two kernels compute the same definitions with different fp32
    contraction orders: breaks equal up to near ties, magnitudes within the
    parity tolerance of each other."""
    spec = synth.StackSpec(P=8192, N=300, n_hist=150, miss=0.5, seed=61)
    Y, dates = synth.generate(spec, DEV)
    outs = {}
    for m in ("fused", "simt"):
        monkeypatch.setenv("BFAST_KERNEL", m)
        o = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
        torch.cuda.synchronize()
        outs[m] = {key: v.cpu().numpy() for key, v in o.items() if hasattr(v, "cpu")}
    a, b = outs["fused"], outs["simt"]
    assert (a["break"] != b["break"]).mean() < 1e-3
    ok = (a["break"] != -2) & (b["break"] != -2)
    d = np.abs(a["magnitude"][ok] - b["magnitude"][ok]) / np.maximum(1, np.abs(b["magnitude"][ok]))
    assert d.max() < 1e-4


def test_tc_path_is_deterministic_at_scale(monkeypatch):
    """Race detector for the warp-specialised pipeline: many persistent tiles
    per CTA, repeated runs must agree bit for bit."""
    monkeypatch.setenv("BFAST_KERNEL", "fused")
    spec = synth.StackSpec(P=1 << 21, N=400, n_hist=200, miss=0.6, mask="cloud", seed=71)
    Y, dates = synth.generate(spec, DEV)
    plan = binding.Plan(0, spec.N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    ref = plan.execute(Y, diagnostics=True)
    ref = {key: v.clone() for key, v in ref.items()}
    for _ in range(4):
        o = plan.execute(Y, diagnostics=True)
        for key in ("break", "magnitude", "sigma", "beta"):
            assert torch.equal(o[key].nan_to_num(), ref[key].nan_to_num()), key
    plan.close()
