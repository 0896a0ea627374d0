"""BASELINE configs[2] on one B200: N in {100, 250, 500, 1000} x missing
{10, 50, 90}% (i.i.d.) x k in {1, 3, 5}, P = 4096^2 pixels each.

Per point: Mpx/s of the whole step (fused kernel + fp64 refit, CUDA events
on the launch stream, bench.py's protocol), the fused kernel's time and its
HBM roofline fraction (algorithmic bytes P(4N + 8) / kernel time / measured
peak), the share of the step in the refit kernel, the refitted and the
degenerate (-2) pixel shares, and the kernel launches per step.

  python tools/sweep_table.py [out.json] [--steps K] [--points N:miss:k,...]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_icde_giesekerhvo20_b200 import binding, synth  # noqa: E402


def main():
    out_path = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("--") else None
    steps = 5
    points = [(N, m, k) for N in (100, 250, 500, 1000) for m in (0.1, 0.5, 0.9) for k in (1, 3, 5)]
    if "--steps" in sys.argv:
        steps = int(sys.argv[sys.argv.index("--steps") + 1])
    if "--points" in sys.argv:
        points = [(int(a), float(b), int(c)) for a, b, c in
                  (p.split(":") for p in sys.argv[sys.argv.index("--points") + 1].split(","))]
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    rows = []
    for (N, miss, k) in points:
        idx = [100, 250, 500, 1000].index(N) * 9 + [0.1, 0.5, 0.9].index(miss) * 3 + [1, 3, 5].index(k)
        spec = synth.sweep_spec(N, miss, k, index=idx)
        Y, dates = synth.generate(spec, "cuda:0")
        plan = binding.Plan(0, spec.N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
        st = torch.cuda.Stream()
        out = {"break": torch.empty(spec.P, dtype=torch.int32, device="cuda:0"),
               "magnitude": torch.empty(spec.P, dtype=torch.float32, device="cuda:0"),
               "flags": torch.empty(spec.P, dtype=torch.uint8, device="cuda:0")}
        with torch.cuda.stream(st):
            for _ in range(3):
                plan.execute(Y, stream=st, out=out)
        torch.cuda.synchronize()
        binding.profile_enable(True)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        launches = 0
        for _ in range(steps):
            plan.execute(Y, stream=st, out=out)
            launches += binding.last_launch_count()
        e1.record(st)
        torch.cuda.synchronize()
        kms = binding.profile_collect()
        binding.profile_enable(False)
        ms = e0.elapsed_time(e1) / steps
        k_ms = sum(kms) / len(kms)
        alg = spec.P * (4 * N + 8)
        refit = int(((out["flags"].to(torch.int32) & 2) != 0).sum())
        deg = int((out["break"] == -2).sum())
        row = {"N": N, "miss": miss, "k": k, "Mpx_s": spec.P / ms / 1e3, "ms_per_step": ms,
               "fused_kernel_ms": k_ms, "hbm_frac": alg / (k_ms / 1e3) / 1e9 / peak,
               "refit_share_of_step": (ms - k_ms) / ms, "refit_pixels": refit / spec.P,
               "degenerate_pixels": deg / spec.P, "launches_per_step": launches / steps}
        rows.append(row)
        print(json.dumps(row), flush=True)
        plan.close()
        del Y, out
        torch.cuda.empty_cache()
    if out_path:
        json.dump({"peak_gbs": peak, "when": time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime()),
                   "gpu": torch.cuda.get_device_name(0), "rows": rows}, open(out_path, "w"), indent=1)


if __name__ == "__main__":
    main()
