#!/usr/bin/env python
"""bench.py -- BFAST-Monitor throughput on B200 (BASELINE.json metric).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                  [--config landsat|tiny|sweep:N:miss:k] [--no-e2e] [--no-cpu-baseline]

One "step" = one pass of the whole hot path (the fused monitor kernel plus
the fp64 refit kernel) over one synthetic scene resident in HBM.  At N=1 the
workload is BASELINE configs[1] (Landsat-like: 4096x4096 pixels, N=400
dates, n_hist=200, k=3, h=0.25, lambda=1.65, 60% cloud-masked).  Under
torchrun each rank processes its own Landsat-shaped scene (weak scaling:
pixels are independent, L142; no collective on the data path) and the
device-timed max over ranks is reported.  Timing: CUDA events on the launch
stream, W warm-up steps, barrier + synchronize on both sides; the 26.8 GB
stack per GPU is far larger than the 126 MB L2, so no explicit flush.

--impl reference times the fp64 CPU oracle (oracle/, the paper's
definitions, OpenMP over the host cores) on a bounded sample of the same
workload: the base contract's reference arm for this paper-only tier.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "BFAST-Monitor pixels/sec at 1/2/4/8 B200; achieved HBM GB/s vs peak"
UNIT = "pixels/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="landsat")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="target oracle wall time")
    ap.add_argument("--slab", type=int, default=1 << 25, help="max pixels per device slab (sentinel2)")
    return ap.parse_args()


def spec_for(name: str):
    from paper_conf_icde_giesekerhvo20_b200 import synth
    if name.startswith("sweep:"):
        _, N, miss, k = name.split(":")
        return synth.sweep_spec(int(N), float(miss), int(k)), f"sweep N={N} miss={miss} k={k}"
    spec = synth.CONFIGS["landsat" if name in ("stream", "int16", "periods") else name]
    desc = {
        "landsat": "Landsat-like scene (BASELINE configs[1]): 4096x4096 px x N=400 dates "
                   "(n_hist=200), k=3, h=0.25, lambda=1.65, 60% missing (cloud masks)",
        "tiny": "tiny (BASELINE configs[0]): 4096 px x N=228 (n_hist=114), k=3, h=0.25, "
                "lambda=1.65, 50% NaN i.i.d.",
        "sentinel2": "Sentinel-2-like tile (BASELINE configs[3]): 10980x10980 px x N=700 dates (n_hist=350), "
                     "k=3, h=0.25, lambda=1.65, 50% NaN i.i.d.; pixel shards over the GPUs (strong scaling)",
        "stream": "continental streaming (BASELINE configs[4]): Landsat-shaped tiles (4096x4096 px x N=400, "
                  "60% cloud) from pinned host memory through the e2e path, H2D double-buffered",
        "periods": "SURVEY 8(f) f1: the Landsat scene (4096x4096 px x N=400, k=3, 60% cloud) with 7 yearly "
                   "monitoring periods in ONE fused launch (L391: 2010-2011, 2011-2012, ...; history = every "
                   "date before the period, n_i = 230 + 23 i, N_i = n_i + 23)",
        "int16": "SURVEY 8(f) f4: the Landsat scene (BASELINE configs[1] shape) as scaled int16 codes "
                 "(y = 1e-4 code, nodata -32768), read by the fused kernel as codes: 2 bytes per stack element",
        "dense": "SURVEY 8(f) f3: Landsat-shaped scene (4096x4096 px x N=400, n_hist=200, k=3) with a complete "
                 "history (the NaN-free case of L93), 60% cloud gaps in the monitoring period only",
        "africa": "SURVEY 8(f) f2: 2^23 px x 2000 dates (n_hist=1000, k=3), 88% of the date slices empty "
                  "(Africa: ~350 of 6873 dates hold data, L379), 50% NaN i.i.d. in the others; step = scan for "
                  "empty slices + gather of the kept ones + the hot path on the compacted stack",
    }[name]
    return spec, desc


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    Q = ("timestamp,index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device_index: int):
        self.dev = device_index
        self.proc = None
        self.lines = []
        self.t0 = self.t1 = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits", "-lms", "20",
                 "-i", str(self.dev)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thr = threading.Thread(target=self._read, daemon=True)
            self.thr.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))

    def mark(self, begin: bool):
        if begin:
            self.t0 = time.time()
        else:
            self.t1 = time.time()

    def stop(self):
        if self.proc:
            time.sleep(0.05)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        rows = [l for (ts, l) in self.lines if self.t0 is not None and self.t0 - 0.02 <= ts <= self.t1 + 0.05]
        if not rows:
            rows = [l for (_, l) in self.lines][-3:]
        sm, smax, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            f = [x.strip() for x in r.split(",")]
            if len(f) < 10:
                continue
            try:
                sm.append(float(f[2]))
                smax = float(f[3])
            except ValueError:
                continue
            for n, v in zip(names, f[6:10]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": smax, "reasons": sorted(reasons),
                "samples": len(sm)}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


def ncu_traffic(workload_key: str):
    """dram read+write bytes per launch of the fused kernel from the committed
    ncu --set full summary (profiles/), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        d = json.load(open(p))
        e = d.get(workload_key)
        return None if e is None else float(e["dram_bytes_per_launch"])
    except Exception:
        return None


def host_cpu():
    """lscpu sockets x cores x threads of the box (SURVEY 8(d) baseline protocol)."""
    info = {}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ":" in ln:
                k, v = ln.split(":", 1)
                info[k.strip()] = v.strip()
    except Exception:
        pass
    return {"model": info.get("Model name"), "sockets": info.get("Socket(s)"),
            "cores_per_socket": info.get("Core(s) per socket"), "threads_per_core": info.get("Thread(s) per core"),
            "cpus": info.get("CPU(s)")}


_ONE_THREAD = {}


def cpu_baseline_entry(value, threads, sample):
    """cpu_baseline object: the all-cores oracle figure plus a 1-thread figure
    measured on the same workload recipe (bounded sample)."""
    return {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample,
            "host": host_cpu(), "one_thread": _ONE_THREAD.get("value")}


def measure_one_thread(Y, dates, spec, seconds=3.0):
    """The oracle on ONE host thread over a bounded sample (pixels/s)."""
    import numpy as np
    import torch
    import oracle
    from paper_conf_icde_giesekerhvo20_b200 import synth
    nmax = oracle.max_threads()
    idx = synth.sample_columns(Y, spec.P, 1024, seed=5)
    Ys = np.ascontiguousarray(Y.index_select(1, torch.tensor(idx, device=Y.device)).cpu().numpy())
    t0 = time.perf_counter()
    oracle.monitor(Ys, dates, spec.n_hist, spec.k, spec.hf, spec.lam, threads=1)
    dt = time.perf_counter() - t0
    count = int(min(1 << 16, max(1024, 1024 * seconds / max(dt, 1e-3))))
    idx = synth.sample_columns(Y, spec.P, count, seed=6)
    Ys = np.ascontiguousarray(Y.index_select(1, torch.tensor(idx, device=Y.device)).cpu().numpy())
    t0 = time.perf_counter()
    oracle.monitor(Ys, dates, spec.n_hist, spec.k, spec.hf, spec.lam, threads=1)
    dt = time.perf_counter() - t0
    _ONE_THREAD["value"] = {"value": count / dt, "unit": UNIT, "threads": 1, "sample": f"{count} pixels, {dt:.1f} s"}
    oracle.monitor(Ys[:, :1], dates, spec.n_hist, spec.k, spec.hf, spec.lam, threads=nmax)  # restore the thread count
    return _ONE_THREAD["value"]


def oracle_sample(Y, dates, spec, count, seed=0):
    """Run the oracle on `count` sampled pixel columns of the device stack Y;
    returns (oracle outputs, seconds, threads, idx)."""
    import numpy as np
    import torch
    import oracle
    from paper_conf_icde_giesekerhvo20_b200 import synth
    idx = synth.sample_columns(Y, spec.P, count, seed=seed)
    it = torch.tensor(idx, device=Y.device)
    Ys = np.ascontiguousarray(Y.index_select(1, it).cpu().numpy())
    t0 = time.perf_counter()
    out = oracle.monitor(Ys, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    dt = time.perf_counter() - t0
    return out, dt, oracle.max_threads(), idx


def run_reference(args):
    """The reference arm: the fp64 oracle on the host cores."""
    import numpy as np
    world, rank, local = dist_env()
    if rank != 0:
        return 0
    import oracle
    spec, desc = spec_for(args.config)
    import torch
    from paper_conf_icde_giesekerhvo20_b200 import synth
    oracle.build()
    # bounded sample of the workload: a sub-scene of the same recipe on CPU
    sub = synth.StackSpec(**{**spec.asdict(), "P": min(spec.P, 1 << 14)})
    Y, dates = synth.generate(sub, "cpu")
    Yn = Y.numpy()
    threads = oracle.max_threads()
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.monitor(Yn, dates, sub.n_hist, sub.k, sub.hf, sub.lam)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    ms = 1000 * sum(times) / len(times)
    value = sub.P / (ms / 1000)
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "sample": f"{sub.P} pixels per step (same recipe, CPU sub-scene)",
                       "same_config": False,
                       "note": "a bounded sample of the workload: the same N, n, k, h, lambda and missing-value "
                               "recipe on a sub-scene of P pixels; the oracle's work per pixel does not depend "
                               "on P, so pixels/s compares with the GPU line"},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"{sub.P} pixels of the workload per step", "host": host_cpu()},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def _finish(line, world, rank):
    import torch.distributed as dist
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_sharded_tile(args, spec, desc, world, rank, local, dev):
    """configs[3]: one tile too large for a GPU, sharded over the ranks (strong
    scaling).  Each rank generates exactly its pixel range of the scene and
    processes it in device-sized slabs; the break map and magnitudes of the
    WHOLE tile live on rank 0's GPU and every rank's kernel stores its slice
    straight into them (CUDA IPC mapping of rank 0's allocation, NVLink peer
    stores from the epilogue: the gather of SURVEY 8(e) happens inside the
    timed kernels).  The step time is the sum of the slab times, max over
    ranks."""
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_icde_giesekerhvo20_b200 import binding, synth
    P, N = spec.P, spec.N
    b, e = binding.shard_range(P, rank, world)
    dates = synth.make_dates(N, spec.f, spec.year0)
    plan = binding.Plan(local, N, dates, spec.n_hist, spec.k, spec.hf, spec.lam)
    stream = torch.cuda.Stream(device=dev)
    slab = max(128, min(args.slab, e - b))
    Ybuf = torch.empty((N, slab), dtype=torch.float32, device=dev)
    # the tile's map on rank 0's GPU, mapped by every rank
    if rank == 0:
        gmap = {"break": torch.full((P,), -7, dtype=torch.int32, device=dev),
                "magnitude": torch.empty(P, dtype=torch.float32, device=dev)}
        handles = [binding.ipc_export(gmap["break"]), binding.ipc_export(gmap["magnitude"])] if world > 1 else None
        ptrs = [gmap["break"].data_ptr(), gmap["magnitude"].data_ptr()]
    else:
        handles = None
    if world > 1:
        box = [handles]
        dist.broadcast_object_list(box, src=0)
        if rank != 0:
            ptrs = [binding.ipc_open(box[0][0], local), binding.ipc_open(box[0][1], local)]
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.6)
    total_ms, kernel_ms, launches = 0.0, 0.0, 0
    last = None
    for s0 in range(b, e, slab):
        s1 = min(e, s0 + slab)
        synth.generate(spec, dev, columns=(s0, s1), out=Ybuf, ldY=slab)
        Y = Ybuf[:, : s1 - s0]  # [N][ldY = slab] view
        o = {"break": ptrs[0] + 4 * s0, "magnitude": ptrs[1] + 4 * s0}
        with torch.cuda.stream(stream):
            for _ in range(args.warmup):
                plan.execute(Y, P=s1 - s0, stream=stream, out=o, check_out=False)
        torch.cuda.synchronize()
        binding.profile_enable(True)
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        sampler.mark(True) if sampler.t0 is None else None
        ev0.record(stream)
        for _ in range(args.steps):
            plan.execute(Y, P=s1 - s0, stream=stream, out=o, check_out=False)
            launches += binding.last_launch_count()
        ev1.record(stream)
        torch.cuda.synchronize()
        kms = binding.profile_collect()
        binding.profile_enable(False)
        total_ms += ev0.elapsed_time(ev1) / args.steps
        kernel_ms += sum(kms) / max(len(kms), 1)
        last = (s0, s1)
    sampler.mark(False)
    sampler.stop()
    if world > 1:
        dist.barrier()
    t = torch.tensor([total_ms, kernel_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_step, k_ms = float(t[0]), float(t[1])
    peak, peak_src = load_peaks()
    alg = (e - b) * (4 * N + 8)
    achieved = alg / (kernel_ms / 1000.0) / 1e9
    line = {"metric": METRIC, "value": P / (ms_step / 1000.0), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": desc, "pixels_total": P, "pixels_per_gpu": e - b, "N": N,
                       "slab_pixels": slab, "l2": "inputs larger than L2, no flush",
                       "parallelism": f"dp{world}: pixel shards of one tile; the break map is gathered on "
                                      f"rank 0's GPU by the kernels' own stores (CUDA IPC peer mapping)"},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": None, "kernel": f"monitor_fused_kernel<{2 + 2 * spec.k}>",
                         "kernel_ms_avg": kernel_ms, "peak_source": peak_src},
            "gpu_launches": launches, "clocks": sampler.summary()}
    if world > 1:
        dist.barrier()  # every rank's stores into rank 0's map are done
    if rank == 0:
        # the whole tile was written: no sentinel left in the map
        line["gather_check"] = {"unwritten_pixels": int((gmap["break"] == -7).sum())}
        if not args.no_cpu_baseline and last is not None:
            # parity + oracle baseline on a sample of rank 0's last slab (its
            # stack is still in the buffer), read back from the gathered map
            from oracle import parity
            s0, s1 = last
            Y = Ybuf[:, : s1 - s0]
            sub = synth.StackSpec(**{**spec.asdict(), "P": s1 - s0})
            probe = 1 << 12
            _, dt, threads, _ = oracle_sample(Y, dates, sub, probe, seed=7)
            count = int(min(1 << 18, max(probe, probe * args.cpu_seconds / max(dt, 1e-3))))
            orc, dt, threads, idx = oracle_sample(Y, dates, sub, count, seed=11)
            it = torch.tensor(idx, device=dev) + s0
            gpu = {"break": gmap["break"].index_select(0, it).cpu().numpy(),
                   "magnitude": gmap["magnitude"].index_select(0, it).cpu().numpy()}
            rep = parity.compare(gpu, orc)
            line["cpu_baseline"] = cpu_baseline_entry(count / dt, threads,
                                                      f"{count} uniformly sampled pixel columns of the tile's "
                                                      f"last slab on rank 0, {dt:.1f} s")
            line["parity_sample"] = {k: rep[k] for k in ("pixels", "ok", "break_mismatch",
                                                         "break_mismatch_unexcused", "invalid_mismatch",
                                                         "mag_fail", "mag_max_scaled_err")}
    elif world > 1:
        binding.ipc_close(ptrs[0])
        binding.ipc_close(ptrs[1])
    if world > 1:
        dist.barrier()
    return _finish(line, world, rank)


def run_stream(args, spec, desc, world, rank, local, dev):
    """configs[4]: tiles streamed from pinned host memory (the e2e path,
    bfast_monitor_host: slab-pipelined H2D overlapped with the kernels).  One
    step = one Landsat-shaped tile per rank; the pinned tile is reused
    round-robin (host RAM holds one tile per rank)."""
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_icde_giesekerhvo20_b200 import binding, synth
    rspec = synth.StackSpec(**{**spec.asdict(), "seed": spec.seed + 1000 * rank})
    Y, dates = synth.generate(rspec, dev)
    P, N = rspec.P, rspec.N
    Yh = torch.empty((N, P), dtype=torch.float32, pin_memory=True)
    Yh.copy_(Y)
    # the two phases alone, for the overlap accounting (no nsys here): the
    # hot path on the device-resident tile, and the tile's H2D copy
    for _ in range(2):
        binding.bfast_monitor_ex(Y, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        binding.bfast_monitor_ex(Y, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam)
    e1.record()
    torch.cuda.synchronize()
    kernel_only_s = e0.elapsed_time(e1) / 3 / 1e3
    e0.record()
    Y.copy_(Yh, non_blocking=True)
    e1.record()
    torch.cuda.synchronize()
    h2d_only_s = e0.elapsed_time(e1) / 1e3
    del Y
    torch.cuda.empty_cache()
    ob, om = np.empty(P, np.int32), np.empty(P, np.float32)
    for _ in range(max(1, args.warmup)):
        binding.bfast_monitor_host(Yh, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam, ob, om, device=local)
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.6)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.mark(True)
    t0 = time.perf_counter()
    launches = 0
    for _ in range(args.steps):
        binding.bfast_monitor_host(Yh, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam, ob, om, device=local)
        launches += binding.last_launch_count()
    dt = (time.perf_counter() - t0) / args.steps
    sampler.mark(False)
    sampler.stop()
    t = torch.tensor([dt], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dt = float(t.item())
    value = world * P / dt
    h2d_gbs = 4 * N * P / dt / 1e9
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1000 * dt, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": desc, "pixels_per_gpu": P, "N": N, "tiles_per_gpu": args.steps,
                       "parallelism": f"dp{world}: one tile stream per GPU, no collective",
                       "bound": "PCIe H2D (%.1f GB/s per GPU achieved)" % h2d_gbs,
                       "tile_reuse": "one pinned Landsat-shaped tile per rank, streamed round-robin"},
            "overlap": {"h2d_only_ms": 1e3 * h2d_only_s, "kernels_only_ms": 1e3 * kernel_only_s,
                        "pipelined_ms": 1e3 * dt,
                        "hidden_fraction_of_kernels": (h2d_only_s + kernel_only_s - dt) / kernel_only_s,
                        "pcie_gbs_alone": 4 * N * P / h2d_only_s / 1e9,
                        "note": "phases timed alone with CUDA events; hidden = (h2d + kernels - pipelined) / kernels"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 4 * N * P, "d2h_bytes_per_step": 8 * P},
            "gpu_launches": launches, "clocks": sampler.summary()}
    return _finish(line, world, rank)


def run_africa(args, spec, desc, world, rank, local, dev):
    """the preprocessing step of the paper's pipeline (drop
    the date slices holding no value, L291/L379) followed by the hot path on
    the compacted stack, per step; rank-local scenes (weak scaling)."""
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_icde_giesekerhvo20_b200 import binding, synth
    rspec = synth.StackSpec(**{**spec.asdict(), "seed": spec.seed + 1000 * rank})
    Y, dates = synth.generate(rspec, dev)
    P, N = rspec.P, rspec.N
    stream = torch.cuda.Stream(device=dev)
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    res = {}

    def step(timed=False):
        if timed:
            ev[0].record(stream)
        keep = binding.bfast_valid_dates(Y, stream=stream)
        if timed:
            ev[1].record(stream)
        stream.synchronize()
        kh = keep.cpu().numpy()
        keep_idx = np.flatnonzero(kh)
        idx = torch.from_numpy(keep_idx.astype(np.int32)).to(dev, non_blocking=False)
        Yc = binding.bfast_gather_dates(Y, idx, stream=stream)
        if timed:
            ev[2].record(stream)
        nc = int(np.count_nonzero(keep_idx < rspec.n_hist))
        out = binding.bfast_monitor_ex(Yc, dates[keep_idx], nc, rspec.k, rspec.hf, rspec.lam, stream=stream)
        if timed:
            ev[3].record(stream)
        res.update(out=out, keep_idx=keep_idx, nc=nc, Yc=Yc)

    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            step()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.6)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.mark(True)
    scan, gather, mon, tot = [], [], [], []
    launches = 0
    with torch.cuda.stream(stream):
        for _ in range(args.steps):
            step(timed=True)
            launches += 3 + binding.last_launch_count() - 1
            torch.cuda.synchronize()
            scan.append(ev[0].elapsed_time(ev[1]))
            gather.append(ev[1].elapsed_time(ev[2]))
            mon.append(ev[2].elapsed_time(ev[3]))
            tot.append(ev[0].elapsed_time(ev[3]))
    sampler.mark(False)
    sampler.stop()
    t = torch.tensor([sum(tot)], dtype=torch.float64, device=dev)
    if world > 1:
        dist.barrier()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_step = float(t.item()) / args.steps
    Nc = len(res["keep_idx"])
    empty = N - Nc
    peak, peak_src = load_peaks()
    s_ms = sum(scan) / len(scan)
    g_ms = sum(gather) / len(gather)
    scan_bytes = empty * P * 4  # every empty slice is read in full (a slice with data stops at its first value)
    gather_bytes = 2 * Nc * P * 4
    roofline = {"bound": "hbm", "achieved": scan_bytes / (s_ms / 1e3) / 1e9, "peak": peak, "unit": "GB/s",
                "frac": scan_bytes / (s_ms / 1e3) / 1e9 / peak, "traffic": None, "kernel": "slice_any_kernel",
                "kernel_ms_avg": s_ms, "kernel_share_of_step": s_ms / ms_step, "alg_bytes_per_launch": scan_bytes,
                "peak_source": peak_src,
                "gather": {"kernel": "gather_dates_kernel", "ms": g_ms, "bytes": gather_bytes,
                           "GB/s": gather_bytes / (g_ms / 1e3) / 1e9},
                "monitor_ms": sum(mon) / len(mon)}
    line = {"metric": METRIC, "value": P * world / (ms_step / 1e3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": desc, "pixels_per_gpu": P, "N_raw": N, "N_kept": Nc, "n_hist_kept": res["nc"],
                       "k": rspec.k, "l2": "inputs larger than L2 (%.1f GB stack), no flush" % (4 * N * P / 1e9),
                       "parallelism": f"dp{world}: pixel shards, no collective"},
            "roofline": roofline, "gpu_launches": launches, "clocks": sampler.summary()}
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import parity
        Yc = res["Yc"]
        orc, dt, threads, idx = oracle_sample(Yc, dates[res["keep_idx"]],
                                              synth.StackSpec(**{**rspec.asdict(), "N": Nc, "n_hist": res["nc"]}),
                                              1 << 16, seed=5)
        it = torch.tensor(idx, device=dev)
        gpu = {"break": res["out"]["break"].index_select(0, it).cpu().numpy(),
               "magnitude": res["out"]["magnitude"].index_select(0, it).cpu().numpy()}
        rep = parity.compare(gpu, orc)
        line["parity_sample"] = {k: rep[k] for k in ("pixels", "ok", "break_mismatch", "invalid_mismatch",
                                                     "mag_fail", "mag_max_scaled_err")}
        # the kept-date list against its plain definition over the whole scene (a slice is kept iff it
        # holds any value), evaluated row block by row block
        ref = torch.cat([~torch.isnan(Y[r:r + 64]).all(dim=1) for r in range(0, N, 64)]).cpu().numpy()
        line["parity_sample"]["keep_list_exact"] = bool(np.array_equal(np.flatnonzero(ref), res["keep_idx"]))
        line["parity_sample"]["ok"] = bool(line["parity_sample"]["ok"] and line["parity_sample"]["keep_list_exact"])
        line["cpu_baseline"] = cpu_baseline_entry(len(idx) / dt, threads,
                                                  f"{len(idx)} sampled columns of the compacted stack, {dt:.1f} s")
    return _finish(line, world, rank)


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import numpy as np
    import torch
    import torch.distributed as dist
    from paper_conf_icde_giesekerhvo20_b200 import _build, binding, synth

    world, rank, local = dist_env()
    if world != args.gpus and world > 1:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    if not os.path.exists(binding.LIB_PATH):
        _build.build()

    spec, desc = spec_for(args.config)
    if args.config == "sentinel2":
        return run_sharded_tile(args, spec, desc, world, rank, local, dev)
    if args.config == "stream":
        return run_stream(args, spec, desc, world, rank, local, dev)
    if args.config == "africa":
        return run_africa(args, spec, desc, world, rank, local, dev)
    if args.config == "dense":  # f3: the shared-factor instantiation (opt-in, include/bfast.h)
        os.environ["BFAST_SHARED_FACTOR"] = "1"
    # each rank: its own scene of the configured shape (weak scaling); seed per rank
    rspec = synth.StackSpec(**{**spec.asdict(), "seed": spec.seed + 1000 * rank})
    Y, dates = synth.generate(rspec, dev)
    P, N = rspec.P, rspec.N
    plan = binding.Plan(local, N, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam)
    stream = torch.cuda.Stream(device=dev)
    out = {"break": torch.empty(P, dtype=torch.int32, device=dev),
           "magnitude": torch.empty(P, dtype=torch.float32, device=dev)}
    I16 = (1e-4, 0.0, -32768)  # codec of the int16 config (scale, offset, nodata)
    codes = None
    if args.config == "int16":
        codes = synth.quantize_i16(Y, *I16)
        del Y
        Y = None
        torch.cuda.empty_cache()
        args.no_e2e = True
    torch.cuda.synchronize()

    PERIODS = [(230 + 23 * i, 253 + 23 * i) for i in range(7)]  # config "periods" (L391)

    def step():
        if args.config == "periods":
            res = binding.bfast_monitor_periods(Y, dates, PERIODS, rspec.k, rspec.hf, rspec.lam, stream=stream)
            out["break"], out["magnitude"] = res["break"][0], res["magnitude"][0]
            out["_periods"] = res
        elif codes is not None:
            binding.bfast_monitor_i16(codes, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam, *I16,
                                      stream=stream, out=out)
        else:
            plan.execute(Y, stream=stream, out=out)

    with torch.cuda.stream(stream):
        for _ in range(args.warmup):
            step()
    torch.cuda.synchronize()

    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.6)  # let nvidia-smi start sampling
    with torch.cuda.stream(stream):   # keep the GPU busy while the sampler starts
        for _ in range(2):
            step()
    binding.profile_enable(True)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.mark(True)
    ev0.record(stream)
    launches = 0
    for _ in range(args.steps):
        step()
        launches += binding.last_launch_count()
    ev1.record(stream)
    torch.cuda.synchronize()
    sampler.mark(False)
    if world > 1:
        dist.barrier()
    kernel_ms = binding.profile_collect()
    binding.profile_enable(False)
    sampler.stop()
    ms_total = ev0.elapsed_time(ev1)
    t = torch.tensor([ms_total], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_step = float(t.item()) / args.steps
    total_pixels = P * world
    value = total_pixels / (ms_step / 1000.0)

    # roofline of the dominant (fused) kernel: algorithmic bytes per launch
    alg_bytes = P * ((2 if codes is not None else 4) * N + 8)
    if args.config == "periods":  # the stack up to the last period's end, read once; M output maps
        alg_bytes = P * (4 * max(e for _, e in PERIODS) + 8 * len(PERIODS))
    kms = sorted(kernel_ms)
    k_avg = sum(kms) / len(kms) if kms else float("nan")
    peak, peak_src = load_peaks()
    achieved = alg_bytes / (k_avg / 1000.0) / 1e9
    workload_key = f"{args.config}:P={P}:N={N}:k={rspec.k}"
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": ncu_traffic(workload_key),
                "kernel": f"monitor_fused_kernel<{2 + 2 * rspec.k}>", "kernel_ms_avg": k_avg,
                "kernel_share_of_step": k_avg / ms_step if ms_step else None,
                "alg_bytes_per_launch": alg_bytes, "peak_source": peak_src}

    if args.config == "periods":
        # the same periods as separate single-period launches (each reads its stack slice from HBM;
        # each sizes its own MOSUM ring, so a pixel near a ring's capacity may take the fp64 refit in
        # one schedule and not the other: equal up to the parity tolerances, usually to the bit)
        plans = [binding.Plan(local, e, dates[:e], b, rspec.k, rspec.hf, rspec.lam) for b, e in PERIODS]
        outs = [{"break": torch.empty(P, dtype=torch.int32, device=dev),
                 "magnitude": torch.empty(P, dtype=torch.float32, device=dev)} for _ in PERIODS]
        with torch.cuda.stream(stream):
            for pl, (b, e), o in zip(plans, PERIODS, outs):
                pl.execute(Y[:e], stream=stream, out=o)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(3):
            for pl, (b, e), o in zip(plans, PERIODS, outs):
                pl.execute(Y[:e], stream=stream, out=o)
        e1.record(stream)
        torch.cuda.synchronize()
        roofline["periods"] = {"M": len(PERIODS), "periods": PERIODS,
                               "period_pixels_per_s": len(PERIODS) * P / (ms_step / 1e3),
                               "separate_launches_ms_per_step": e0.elapsed_time(e1) / 3,
                               "one_launch_ms_per_step": ms_step,
                               "identical_to_separate": bool(all(
                                   torch.equal(o["break"], out["_periods"]["break"][i]) and
                                   torch.equal(o["magnitude"].view(torch.int32),
                                               out["_periods"]["magnitude"][i].view(torch.int32))
                                   for i, o in enumerate(outs)))}
        del plans, outs

    if args.config == "dense":
        # f3 A/B on the same scene: the shared fp64 factor vs every pixel factoring its own Gram
        ab = {}
        for key, val in (("per_pixel_factor", "0"), ("shared_factor", "1")):
            os.environ["BFAST_SHARED_FACTOR"] = val
            with torch.cuda.stream(stream):
                step()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            for _ in range(5):
                step()
            e1.record(stream)
            torch.cuda.synchronize()
            ab[key + "_ms_per_step"] = e0.elapsed_time(e1) / 5
        os.environ["BFAST_SHARED_FACTOR"] = "1"
        roofline["f3_ab"] = ab

    clocks = sampler.summary()
    line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": desc, "pixels_per_gpu": P, "N": N, "n_hist": rspec.n_hist, "k": rspec.k,
                       "h": rspec.hf, "lambda": rspec.lam, "missing": rspec.miss, "mask": rspec.mask,
                       "l2": "inputs larger than L2 (stack %.1f GB/GPU vs 126 MB L2), no flush" % (4 * N * P / 1e9),
                       "parallelism": f"dp{world}: pixel shards, no collective"},
            "roofline": roofline, "gpu_launches": launches, "clocks": clocks}

    # cpu baseline + sampled parity (rank 0, N = 1 only)
    if rank == 0 and world == 1 and not args.no_cpu_baseline and codes is not None:
        # int16: the oracle decodes the sampled code columns itself (oracle.decode_i16)
        import oracle
        from oracle import parity
        idx = synth.sample_columns(codes, P, 1 << 17, seed=11)
        it = torch.tensor(idx, device=dev)
        Yd = oracle.decode_i16(codes.index_select(1, it).cpu().numpy(), np.float32(I16[0]), np.float32(I16[1]),
                               I16[2])
        t0 = time.perf_counter()
        orc = oracle.monitor(np.ascontiguousarray(Yd), dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam)
        dt = time.perf_counter() - t0
        gpu = {"break": out["break"].index_select(0, it).cpu().numpy(),
               "magnitude": out["magnitude"].index_select(0, it).cpu().numpy()}
        rep = parity.compare(gpu, orc)
        line["cpu_baseline"] = cpu_baseline_entry(len(idx) / dt, oracle.max_threads(),
                                                  f"{len(idx)} sampled columns decoded by the oracle, {dt:.1f} s")
        line["parity_sample"] = {k: rep[k] for k in ("pixels", "ok", "break_mismatch",
                                                     "break_mismatch_unexcused", "invalid_mismatch",
                                                     "mag_fail", "mag_max_scaled_err")}
    elif rank == 0 and world == 1 and not args.no_cpu_baseline:
        from oracle import parity
        Yo, do, so = Y, dates, rspec
        if args.config == "periods":  # the sample checks period 0 on its own date slice
            b0, e0_ = PERIODS[0]
            Yo, do, so = Y[:e0_], dates[:e0_], synth.StackSpec(**{**rspec.asdict(), "N": e0_, "n_hist": b0})
        probe = 1 << 13
        _, dt, threads, _ = oracle_sample(Yo, do, so, probe, seed=7)
        count = int(min(1 << 21, max(probe, probe * args.cpu_seconds / max(dt, 1e-3))))
        orc, dt, threads, idx = oracle_sample(Yo, do, so, count, seed=11)
        it = torch.tensor(idx, device=dev)
        gpu = {"break": out["break"].index_select(0, it).cpu().numpy(),
               "magnitude": out["magnitude"].index_select(0, it).cpu().numpy()}
        rep = parity.compare(gpu, orc)
        measure_one_thread(Yo, do, so)
        line["cpu_baseline"] = cpu_baseline_entry(count / dt, threads,
                                                  f"{count} uniformly sampled pixel columns of the same scene, "
                                                  f"{dt:.1f} s")
        line["parity_sample"] = {k: rep[k] for k in ("pixels", "ok", "break_mismatch",
                                                     "break_mismatch_unexcused", "invalid_mismatch",
                                                     "mag_fail", "mag_max_scaled_err")}

    # end to end through the public host-buffer API: H2D + kernels + D2H
    if not args.no_e2e:
        Yh = torch.empty((N, P), dtype=torch.float32, pin_memory=True)
        Yh.copy_(Y)
        del Y
        torch.cuda.empty_cache()
        ob = np.empty(P, np.int32)
        om = np.empty(P, np.float32)
        binding.bfast_monitor_host(Yh, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam, ob, om, device=local)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            binding.bfast_monitor_host(Yh, dates, rspec.n_hist, rspec.k, rspec.hf, rspec.lam, ob, om,
                                       device=local)
        e2e_s = (time.perf_counter() - t0) / args.e2e_steps
        te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(te, op=dist.ReduceOp.MAX)
        e2e_s = float(te.item())
        line["e2e"] = {"value": total_pixels / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 4 * N * P,
                       "d2h_bytes_per_step": 8 * P, "steps": args.e2e_steps,
                       "path": "bfast_monitor_host: pinned host stack, slab-pipelined H2D overlapped "
                               "with the kernels, D2H of results; host wall clock"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
