"""Diagnostic: TC kernel vs oracle on one StackSpec (argv: json of StackSpec
fields + optional hf/lam), the worst pixels by scaled magnitude error."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from oracle import parity
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
kw = json.loads(sys.argv[1])
spec = synth.StackSpec(**kw)
Y, dates = synth.generate(spec, "cuda:0")
o = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
torch.cuda.synchronize()
g = {kk: v.cpu().numpy() for kk, v in o.items() if hasattr(v, "cpu")}
orc = oracle.monitor(Y.cpu().numpy(), dates, spec.n_hist, spec.k, spec.hf, spec.lam)
s = parity.column_scales(dates, spec.n_hist, spec.k)
ok = (orc["break"] != -2) & (g["break"] != -2)
err = np.abs(g["magnitude"] - orc["magnitude"]) / np.maximum(1, np.abs(orc["magnitude"]))
err[~ok] = 0
sig = np.abs(g["sigma"] - orc["sigma"]) / orc["sigma"]
print("max err %.3g  p99.9 %.3g  median %.3g  sigma rel max %.3g" % (err.max(), np.quantile(err[ok], .999), np.median(err[ok]), np.nanmax(sig[ok])))
for p in np.argsort(-err)[:int(os.environ.get("DIAG_TOP", "8"))]:
    be = np.abs(g["beta"][p] - orc["beta"][p]) * s
    print(f"  p={p} nbar={orc['nbar'][p]} Nbar={orc['Nbar'][p]} h={orc['h'][p]} cond={orc['cond'][p]:.3g} "
          f"mag_o={orc['magnitude'][p]:.6g} err={err[p]:.2e} sig_rel={sig[p]:.2e} flags={g['flags'][p]} "
          f"beta_err={be.max()/np.max(np.abs(orc['beta'][p]*s)):.2e}")
