"""Cycle accounting of the fused kernel (diagnostics build, -DBFAST_FZ_TIMING):
where each warp's time goes on the Landsat config.

  python tools/fz_timing.py LIB.so   (GPU box; LIB built with _build.build(out=..., defines=["BFAST_FZ_TIMING"]))
"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["BFAST_LIB"] = os.path.abspath(sys.argv[1])
import torch  # noqa: E402

from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402

NAMES = ["cons A: wait operand buffer (g-2)", "cons: wait yhat", "-", "cons: acquire stack half",
         "ctl: on_publish work (after the wait)", "ctl: wait publish", "ctl: wait table", "ctl: wait release",
         "kernel (per warp, all warps)", "cons: solve wait Gram", "cons: refine wait db", "-",
         "ctl: load_half (TMA issue)", "ctl: wait mdone g-1 (table release)"]
mode = sys.argv[2] if len(sys.argv) > 2 else "landsat"
spec = synth.CONFIGS["landsat" if mode in ("periods", "single7") else mode]
Y, dates = synth.generate(spec, "cuda:0")
PER = [(230 + 23 * i, 253 + 23 * i) for i in range(7)]


def run():
    if mode == "periods":  # f1: one multi-period launch
        return binding.bfast_monitor_periods(Y, dates, PER, spec.k, spec.hf, spec.lam)
    if mode == "single7":  # the same periods as separate launches
        return [binding.bfast_monitor_ex(Y[:e], dates[:e], b, spec.k, spec.hf, spec.lam) for b, e in PER]
    return binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
L = binding.lib()
L.bfast_debug_fz_timing.argtypes = [ctypes.c_void_p, ctypes.c_int]
buf = (ctypes.c_ulonglong * 16)()
for rep in range(2):
    L.bfast_debug_fz_timing(buf, 16)
    out = run()
    torch.cuda.synchronize()
L.bfast_debug_fz_timing(buf, 16)
tot = buf[8]
for i, nm in enumerate(NAMES):
    v = buf[i]
    print(f"{nm:40s} {v:>20d}  {100.0 * v / tot:6.2f}%")
