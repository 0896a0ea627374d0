"""Diagnostic: per-pixel TC vs SIMT vs oracle on one sweep shape."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from oracle import parity
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
N, miss, k = int(sys.argv[1]), float(sys.argv[2]), int(sys.argv[3])
idx = [100, 250, 500, 1000].index(N) * 9 + [0.1, 0.5, 0.9].index(miss) * 3 + [1, 3, 5].index(k)
spec = synth.sweep_spec(N, miss, k, P=4096, index=idx)
Y, dates = synth.generate(spec, "cuda:0")
res = {}
for m in ("fused", "simt"):
    os.environ["BFAST_KERNEL"] = m
    o = binding.bfast_monitor_ex(Y, dates, spec.n_hist, k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    res[m] = {kk: v.cpu().numpy() for kk, v in o.items() if hasattr(v, "cpu")}
orc = oracle.monitor(Y.cpu().numpy(), dates, spec.n_hist, k, spec.hf, spec.lam)
s = parity.column_scales(dates, spec.n_hist, k)
for m in ("fused", "simt"):
    g = res[m]
    ok = (orc["break"] != -2) & (g["break"] != -2)
    err = np.abs(g["magnitude"] - orc["magnitude"]) / np.maximum(1, np.abs(orc["magnitude"]))
    bad = np.nonzero(ok & (err > 1e-4))[0]
    print(m, "fails", len(bad))
    for p in bad[:12]:
        be = np.abs(g["beta"][p] - orc["beta"][p]) * s
        print(f"  p={p} nbar={orc['nbar'][p]} Nbar={orc['Nbar'][p]} h={orc['h'][p]} cond={orc['cond'][p]:.3g} "
              f"mag_o={orc['magnitude'][p]:.6g} mag_g={g['magnitude'][p]:.6g} err={err[p]:.2e} "
              f"sig_o={orc['sigma'][p]:.4g} sig_g={g['sigma'][p]:.4g} flags={g['flags'][p]} "
              f"beta_err={be.max()/np.max(np.abs(orc['beta'][p]*s)):.2e} maxabsbeta_s={np.max(np.abs(orc['beta'][p]*s)):.3g}")
