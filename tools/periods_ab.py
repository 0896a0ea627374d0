"""Per-period timing: the single-period kernel (bfast_monitor_ex on Y[:N_i])
vs the multi-period kernel with that one period, then all periods at once."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_icde_giesekerhvo20_b200 import binding, synth
spec = synth.CONFIGS["landsat"]
Y, dates = synth.generate(spec, "cuda:0")
periods = [(230 + 23 * i, 253 + 23 * i) for i in range(7)]


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


os.environ["BFAST_VERBOSE"] = "1"
for b, e in periods:
    t1 = timed(lambda: binding.bfast_monitor_ex(Y[:e], dates[:e], b, 3, spec.hf, spec.lam))
    tm = timed(lambda: binding.bfast_monitor_periods(Y, dates, [(b, e)], 3, spec.hf, spec.lam))
    print(json.dumps({"period": [b, e], "single_ms": round(t1, 3), "multi1_ms": round(tm, 3)}), flush=True)
print(json.dumps({"all": timed(lambda: binding.bfast_monitor_periods(Y, dates, periods, 3, spec.hf, spec.lam))}))
