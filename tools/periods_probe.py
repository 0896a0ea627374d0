"""Launch bfast_monitor_periods on the Landsat scene twice (the second is the
one ncu captures): python tools/periods_probe.py [M]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
M = int(sys.argv[1]) if len(sys.argv) > 1 else 7
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")
periods = [(230 + 23 * i, 253 + 23 * i) for i in range(M)]
for _ in range(2):
    binding.bfast_monitor_periods(Y, dates, periods, spec.k, spec.hf, spec.lam)
torch.cuda.synchronize()
print("ok", M)
