"""Run the full Landsat scene several times on the TC path; report run-to-run
and TC-vs-SIMT differences (race detection)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")
outs = []
for m in ["fused"] * 6 + ["simt"]:
    os.environ["BFAST_KERNEL"] = m
    o = binding.bfast_monitor_ex(Y, dates, spec.n_hist, spec.k, spec.hf, spec.lam, diagnostics=True)
    torch.cuda.synchronize()
    outs.append({k: v.clone() for k, v in o.items() if hasattr(v, "clone")})
for i in range(1, 7):
    a, b = outs[0], outs[i]
    db = (a["break"] != b["break"]).nonzero().flatten()
    dm = ((a["magnitude"] - b["magnitude"]).abs() > 1e-3 * (1 + b["magnitude"].abs())).nonzero().flatten()
    print(i, "break diffs", db.numel(), "mag diffs", dm.numel(), db[:10].tolist(), dm[:10].tolist())
    if dm.numel():
        p = dm[0].item()
        print("   pix", p, "mag", a["magnitude"][p].item(), b["magnitude"][p].item(), "nbar", a["nbar"][p].item(), b["nbar"][p].item(),
              "sigma", a["sigma"][p].item(), b["sigma"][p].item(), "flags", a["flags"][p].item(), b["flags"][p].item(),
              "tile", p // 128, "lane", p % 128)
