"""Small TC + SIMT invocation for compute-sanitizer runs."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
spec = synth.StackSpec(P=1000, N=120, n_hist=60, miss=0.5, seed=3)
Y, dates = synth.generate(spec, "cuda:0")
for m in ("fused", "simt"):
    os.environ["BFAST_KERNEL"] = m
    o = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    print(m, int((o["break"] >= 0).sum()), int((o["break"] == -2).sum()))
