"""Count the pixels the fused kernel hands to the fp64 refit (flags bit 1)
on a bench config, and time the two kernels of one call with CUDA events.
    python tools/refit_probe.py [--config landsat] [--P 16777216]"""
import argparse
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="landsat")
ap.add_argument("--P", type=int, default=None)
a = ap.parse_args()
spec = synth.CONFIGS[a.config]
if a.P:
    spec = dataclasses.replace(spec, P=a.P)
Y, dates = synth.generate(spec, "cuda")
out = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
torch.cuda.synchronize()
f = out["flags"].to(torch.int32)
ref = int(((f & 2) != 0).sum())
deg = int(((f & 1) != 0).sum())
print(f"{a.config} P={spec.P} refitted={ref} ({100 * ref / spec.P:.3f}%) degenerate={deg}")
for _ in range(3):
    binding.bfast_monitor(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
torch.cuda.synchronize()
s.record()
for _ in range(10):
    binding.bfast_monitor(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
e.record()
torch.cuda.synchronize()
print(f"call avg {s.elapsed_time(e) / 10:.3f} ms")
