"""Count the pixels the fused kernel sends to the fp64 refit, by trigger.
Needs a diagnostics build:  python -c "from paper_conf_icde_giesekerhvo20_b200 import _build;
_build.build(out='ab/libbfast_why.so', defines=['BFAST_REFIT_WHY'])"  then
    BFAST_LIB=$PWD/ab/libbfast_why.so python tools/refit_stats.py [--config landsat] [--P 4194304]"""
import argparse
import dataclasses
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="landsat")
ap.add_argument("--P", type=int, default=1 << 22)
a = ap.parse_args()
spec = dataclasses.replace(synth.CONFIGS[a.config], P=a.P)
Y, dates = synth.generate(spec, "cuda")
out = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
torch.cuda.synchronize()
f = out["flags"].to(torch.int32).cpu()
P = spec.P
names = {0x01: "degenerate", 0x02: "refitted (fp64)", 0x10: "pivot ratio", 0x20: "sigma cancellation",
         0x40: "sigma < 2e-3 max|y|", 0x80: "near tie"}
print(f"{a.config} P={P}")
for b, nm in names.items():
    c = int(((f & b) != 0).sum())
    print(f"  {nm:22s} {c:9d}  {100 * c / P:7.3f}%")
