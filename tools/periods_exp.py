"""f1 experiments: one multi-period launch vs the same periods as separate
single-period launches, for period sets of different shapes."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


sets = {"same_n": [(200, 300 + 10 * i) for i in range(4)],
        "yearly4": [(230 + 23 * i, 253 + 23 * i) for i in range(4)],
        "yearly7": [(230 + 23 * i, 253 + 23 * i) for i in range(7)]}
for name, per in sets.items():
    sep = timed(lambda: [binding.bfast_monitor_ex(Y[:e], dates[:e], b, 3, spec.hf, spec.lam) for b, e in per])
    res = {"set": name, "separate_ms": round(sep, 2)}
    for env in ("", "BFAST_FZ_PFD=128", "BFAST_FZ_T=2"):
        for kv in [env] if env else []:
            k, v = kv.split("=")
            os.environ[k] = v
        res["one_launch_ms" + (":" + env if env else "")] = round(
            timed(lambda: binding.bfast_monitor_periods(Y, dates, per, 3, spec.hf, spec.lam)), 2)
        if env:
            os.environ.pop(env.split("=")[0])
    print(json.dumps(res), flush=True)
