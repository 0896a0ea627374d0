"""Multi-GPU plumbing: pixel sharding, max-over-ranks timing, break-map gather.

Pixels are independent ("the computation of any pixel is
independent of any other"), so the data path has no collective: each rank
runs the fused kernel on its own contiguous, 128-pixel-aligned slice of the
scene.  The only exchange is the final gather of the 8-byte-per-pixel result
(out_break, out_magnitude) -- a plain torch.distributed all_gather (NCCL over
NVLink on GPUs, gloo in the CPU tests) -- and the max-over-ranks of the
device-timed step used by bench.py.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import binding


def shard(P: int, rank: int, world: int):
    """[begin, end) of rank's slice (C-ABI bfast_shard_range, host-only)."""
    return binding.shard_range(P, rank, world)


def max_over_ranks(value: float, device=None) -> float:
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def gather_break_map(local_break: torch.Tensor, local_mag: torch.Tensor, P: int):
    """All-gather the per-rank result slices into full [P] arrays on every
    rank (slices are the shard() ranges; padded to the largest slice)."""
    world = dist.get_world_size()
    sizes = [shard(P, r, world) for r in range(world)]
    width = max(e - b for b, e in sizes)
    dev = local_break.device
    pb = torch.full((width,), -3, dtype=torch.int32, device=dev)
    pm = torch.zeros((width,), dtype=torch.float32, device=dev)
    pb[: local_break.numel()] = local_break
    pm[: local_mag.numel()] = local_mag
    gb = [torch.empty_like(pb) for _ in range(world)]
    gm = [torch.empty_like(pm) for _ in range(world)]
    dist.all_gather(gb, pb)
    dist.all_gather(gm, pm)
    out_b = torch.cat([g[: e - b] for g, (b, e) in zip(gb, sizes)])
    out_m = torch.cat([g[: e - b] for g, (b, e) in zip(gm, sizes)])
    return out_b, out_m
