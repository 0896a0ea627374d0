"""One multi-period launch (yearly7) and the 7 single-period launches, for
an ncu metrics capture of every monitor_fused launch."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")
per = [(230 + 23 * i, 253 + 23 * i) for i in range(7)]
binding.bfast_monitor_periods(Y, dates, per, 3, spec.hf, spec.lam)
for b, e in per:
    binding.bfast_monitor_ex(Y[:e], dates[:e], b, 3, spec.hf, spec.lam)
torch.cuda.synchronize()
