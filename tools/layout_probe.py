"""Time the TC kernel on a Landsat-shaped slab whose tile count divides
evenly over 2 or 3 CTAs per SM (no tail), printing the layout the launcher
picks (BFAST_VERBOSE=1) -- layout / occupancy experiments:
    BFAST_TC_LAYOUT=sy,nop,per_sm python tools/layout_probe.py [--hf 0.15]"""
import argparse
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--hf", type=float, default=0.25)
ap.add_argument("--tiles", type=int, default=20, help="tiles per CTA at 888 CTAs")
ap.add_argument("--iters", type=int, default=5)
a = ap.parse_args()
spec = dataclasses.replace(synth.CONFIGS["landsat"], P=148 * 6 * 128 * a.tiles, hf=a.hf)
Y, dates = synth.generate(spec, "cuda")
run = lambda: binding.bfast_monitor(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
run()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(a.iters):
    run()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / a.iters
print(f"hf={a.hf} P={spec.P} ms={ms:.3f} Mpx/s={spec.P / ms / 1e3:.1f} layout={os.environ.get('BFAST_TC_LAYOUT', 'auto')}")
