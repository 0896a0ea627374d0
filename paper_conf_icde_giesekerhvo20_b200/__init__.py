"""B200-native BFAST-Monitor (Gieseke et al., ICDE 2020) -- the data-parallel
hot path as a C-ABI CUDA library (libbfast.so, include/bfast.h) with a thin
ctypes binding.  Importing the package does not load the library; the first
call does, and raises if it is missing (no CPU fallback).
"""
from .binding import (  # noqa: F401
    BfastError, Plan, abi_version, bfast_monitor, bfast_monitor_ex, bfast_monitor_host,
    bfast_monitor_multi, last_error, last_launch_count, shard_range, NO_BREAK, INVALID_PIXEL,
    FLAG_DEGENERATE, FLAG_REFIT_FP64, LIB_PATH,
)

__all__ = ["bfast_monitor", "bfast_monitor_ex", "bfast_monitor_host", "bfast_monitor_multi",
           "Plan", "BfastError", "shard_range"]
