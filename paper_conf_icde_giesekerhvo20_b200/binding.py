"""ctypes binding of libbfast.so (include/bfast.h) -- argument marshalling only.

Every step of BFAST-Monitor runs in the library's CUDA kernels; this module
turns torch tensors / numpy arrays into pointers and statuses into
exceptions.  There is no CPU fallback: if libbfast.so is missing or the
device path fails, the call raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# BFAST_LIB: another in-tree build of the same ABI (A/B timing of kernel
# variants on one box, tools/ab_bench.sh); the default is the package's own
LIB_PATH = os.environ.get("BFAST_LIB") or os.path.join(_HERE, "libbfast.so")
_lib = None

BFAST_OK, BFAST_EINVAL, BFAST_EUNSUPPORTED, BFAST_ECUDA, BFAST_ENOMEM = 0, -1, -2, -3, -4
NO_BREAK, INVALID_PIXEL = -1, -2
FLAG_DEGENERATE, FLAG_REFIT_FP64 = 0x01, 0x02
K_MAX_HARMONICS = 6

# names declared in include/bfast.h (checked by tests/test_abi.py)
EXPORTS = ("bfast_monitor", "bfast_monitor_ex", "bfast_plan_create", "bfast_plan_execute",
           "bfast_plan_destroy", "bfast_monitor_host", "bfast_monitor_multi", "bfast_monitor_shards",
           "bfast_ipc_export", "bfast_ipc_open", "bfast_ipc_close",
           "bfast_shard_range", "bfast_last_launch_count", "bfast_last_error",
           "bfast_status_string", "bfast_abi_version", "bfast_profile_enable",
           "bfast_profile_collect", "bfast_valid_dates", "bfast_gather_dates",
           "bfast_monitor_host_resume", "bfast_monitor_i16", "bfast_monitor_periods")
IPC_HANDLE_BYTES = 72


class BfastError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{msg} (status {status})")
        self.status = status


class _CodecI16(ctypes.Structure):
    _fields_ = [("Y", ctypes.c_void_p), ("scale", ctypes.c_float), ("offset", ctypes.c_float),
                ("nodata", ctypes.c_int32)]


class _Args(ctypes.Structure):
    _fields_ = [("Y", ctypes.c_void_p), ("N", ctypes.c_int64), ("P", ctypes.c_int64),
                ("ldY", ctypes.c_int64), ("dates", ctypes.c_void_p), ("n_hist", ctypes.c_int32),
                ("k", ctypes.c_int32), ("h", ctypes.c_float), ("lambda_", ctypes.c_float),
                ("out_break", ctypes.c_void_p), ("out_magnitude", ctypes.c_void_p),
                ("out_beta", ctypes.c_void_p), ("out_sigma", ctypes.c_void_p),
                ("out_nbar", ctypes.c_void_p), ("out_flags", ctypes.c_void_p),
                ("stream", ctypes.c_void_p)]


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        V, i64, i32, f32, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_float, ctypes.c_int
        L.bfast_monitor.argtypes = [V, i64, i64, V, i32, i32, f32, f32, V, V]
        L.bfast_monitor.restype = I
        L.bfast_monitor_ex.argtypes = [ctypes.POINTER(_Args)]
        L.bfast_monitor_ex.restype = I
        L.bfast_plan_create.argtypes = [ctypes.POINTER(V), I, i64, V, i32, i32, f32, f32]
        L.bfast_plan_create.restype = I
        L.bfast_plan_execute.argtypes = [V, ctypes.POINTER(_Args)]
        L.bfast_plan_execute.restype = I
        L.bfast_plan_destroy.argtypes = [V]
        L.bfast_plan_destroy.restype = None
        L.bfast_monitor_host.argtypes = [V, i64, i64, i64, V, i32, i32, f32, f32, V, V, I]
        L.bfast_monitor_host.restype = I
        L.bfast_monitor_multi.argtypes = [V, i64, i64, i64, V, i32, i32, f32, f32, V, I, V, V]
        L.bfast_monitor_multi.restype = I
        L.bfast_monitor_shards.argtypes = [V, V, V, V, I, i64, V, i32, i32, f32, f32, I, V, V]
        L.bfast_monitor_shards.restype = I
        L.bfast_ipc_export.argtypes = [V, V]
        L.bfast_ipc_export.restype = I
        L.bfast_ipc_open.argtypes = [V, I, ctypes.POINTER(V)]
        L.bfast_ipc_open.restype = I
        L.bfast_ipc_close.argtypes = [V]
        L.bfast_ipc_close.restype = I
        L.bfast_shard_range.argtypes = [i64, I, I, ctypes.POINTER(i64), ctypes.POINTER(i64)]
        L.bfast_shard_range.restype = None
        L.bfast_last_launch_count.restype = I
        L.bfast_last_error.restype = ctypes.c_char_p
        L.bfast_status_string.argtypes = [I]
        L.bfast_status_string.restype = ctypes.c_char_p
        L.bfast_abi_version.restype = I
        L.bfast_profile_enable.argtypes = [I]
        L.bfast_profile_enable.restype = I
        L.bfast_monitor_periods.argtypes = [ctypes.POINTER(_Args), V, V, i32]
        L.bfast_monitor_periods.restype = I
        L.bfast_monitor_i16.argtypes = [ctypes.POINTER(_CodecI16), ctypes.POINTER(_Args)]
        L.bfast_monitor_i16.restype = I
        L.bfast_valid_dates.argtypes = [V, i64, i64, i64, V, V]
        L.bfast_valid_dates.restype = I
        L.bfast_gather_dates.argtypes = [V, i64, i64, i64, V, i64, V, i64, V]
        L.bfast_gather_dates.restype = I
        L.bfast_monitor_host_resume.argtypes = [V, i64, i64, i64, V, i32, i32, f32, f32, V, V, I, i64, i64,
                                                ctypes.POINTER(i64)]
        L.bfast_monitor_host_resume.restype = I
        L.bfast_profile_collect.argtypes = [V, I]
        L.bfast_profile_collect.restype = I
        _lib = L
    return _lib


def _check(rc: int):
    if rc != BFAST_OK:
        L = lib()
        raise BfastError(rc, f"{L.bfast_status_string(rc).decode()}: {L.bfast_last_error().decode()}")


def _dates(dates) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(dates, dtype=np.float64))


def _dptr(t) -> Optional[int]:
    if t is None:
        return None
    if isinstance(t, int):  # a raw device pointer (IPC-mapped output)
        return t
    return int(t.data_ptr())


def _stream_ptr(stream):
    if stream is None:
        import torch
        return int(torch.cuda.current_stream().cuda_stream)
    return int(getattr(stream, "cuda_stream", stream))


def abi_version() -> int:
    return int(lib().bfast_abi_version())


def last_launch_count() -> int:
    return int(lib().bfast_last_launch_count())


def last_error() -> str:
    return lib().bfast_last_error().decode()


def profile_enable(on: bool = True):
    _check(lib().bfast_profile_enable(1 if on else 0))


def profile_collect(max_events: int = 100000):
    """Milliseconds of each fused-kernel launch recorded since enabling."""
    buf = (ctypes.c_float * max_events)()
    n = lib().bfast_profile_collect(ctypes.cast(buf, ctypes.c_void_p), max_events)
    if n < 0:
        _check(n)
    return [float(buf[i]) for i in range(n)]


def shard_range(P: int, rank: int, world: int):
    b, e = ctypes.c_int64(), ctypes.c_int64()
    lib().bfast_shard_range(int(P), int(rank), int(world), ctypes.byref(b), ctypes.byref(e))
    return int(b.value), int(e.value)


def _make_args(Y, dates_np, n_hist, k, h, lam, out_break, out_magnitude, P=None, ldY=None,
               out_beta=None, out_sigma=None, out_nbar=None, out_flags=None, stream=None) -> _Args:
    N = int(Y.shape[0])
    ldY = int(Y.stride(0)) if ldY is None else int(ldY)
    P = int(Y.shape[1]) if P is None else int(P)
    a = _Args()
    a.Y = _dptr(Y)
    a.N, a.P, a.ldY = N, P, ldY
    a.dates = dates_np.ctypes.data
    a.n_hist, a.k, a.h, a.lambda_ = int(n_hist), int(k), float(h), float(lam)
    a.out_break, a.out_magnitude = _dptr(out_break), _dptr(out_magnitude)
    a.out_beta, a.out_sigma = _dptr(out_beta), _dptr(out_sigma)
    a.out_nbar, a.out_flags = _dptr(out_nbar), _dptr(out_flags)
    a.stream = _stream_ptr(stream)
    return a


def _outputs(Y, P, k, want_diag):
    import torch
    dev = Y.device
    out = {"break": torch.empty(P, dtype=torch.int32, device=dev),
           "magnitude": torch.empty(P, dtype=torch.float32, device=dev)}
    if want_diag:
        out["beta"] = torch.empty((P, 2 + 2 * k), dtype=torch.float32, device=dev)
        out["sigma"] = torch.empty(P, dtype=torch.float32, device=dev)
        out["nbar"] = torch.empty(P, dtype=torch.int32, device=dev)
        out["flags"] = torch.empty(P, dtype=torch.uint8, device=dev)
    return out


def _check_stack(Y):
    import torch
    if not (isinstance(Y, torch.Tensor) and Y.is_cuda and Y.dtype == torch.float32 and Y.dim() == 2
            and Y.stride(1) == 1):
        raise TypeError("Y must be a CUDA float32 [N][P] tensor with unit column stride")


def _check_out(out, Y, P):
    """Every output tensor on Y's device with at least P (x K) elements: the
    library writes through raw pointers."""
    for name, t in out.items():
        if name.startswith("_") or t is None:
            continue
        if not t.is_cuda or t.device != Y.device:
            raise ValueError(f"output {name!r} is on {t.device}, the stack on {Y.device}")
        if t.shape[0] < P or not t.is_contiguous():
            raise ValueError(f"output {name!r} must be contiguous with >= {P} rows")


def bfast_monitor(Y, dates, n_hist, k, h, lam, out_break=None, out_magnitude=None):
    """North-star entry (synchronous).  Y: CUDA float32 [N][P] contiguous."""
    _check_stack(Y)
    N, P = Y.shape
    if Y.stride(0) != P:
        raise ValueError("bfast_monitor needs ldY == P; use bfast_monitor_ex")
    d = _dates(dates)
    if out_break is None or out_magnitude is None:
        o = _outputs(Y, P, k, False)
        out_break, out_magnitude = o["break"], o["magnitude"]
    _check(lib().bfast_monitor(_dptr(Y), N, P, d.ctypes.data, int(n_hist), int(k), float(h),
                               float(lam), _dptr(out_break), _dptr(out_magnitude)))
    return out_break, out_magnitude


def bfast_monitor_ex(Y, dates, n_hist, k, h, lam, P=None, diagnostics=False, stream=None, out=None):
    """Asynchronous extended entry on `stream` (default: torch's current
    stream of Y's device).  Y may be a [N][ldY] view with P <= ldY columns
    used.  The call runs on Y's device (the library uses the current one)."""
    import torch
    _check_stack(Y)
    P = int(Y.shape[1]) if P is None else int(P)
    out = out if out is not None else _outputs(Y, P, k, diagnostics)
    _check_out(out, Y, P)
    d = _dates(dates)
    with torch.cuda.device(Y.device):
        a = _make_args(Y, d, n_hist, k, h, lam, out["break"], out["magnitude"], P=P,
                       out_beta=out.get("beta"), out_sigma=out.get("sigma"), out_nbar=out.get("nbar"),
                       out_flags=out.get("flags"), stream=stream)
        _check(lib().bfast_monitor_ex(ctypes.byref(a)))
    out["_dates_keepalive"] = d
    return out


def bfast_monitor_i16(Y16, dates, n_hist, k, h, lam, scale, offset, nodata, P=None, diagnostics=False,
                      stream=None, out=None):
    """f4: the hot path on an int16-coded stack (CUDA int16 [N][ldY], ldY %
    8 == 0): y = fmaf(scale, code, offset), code == nodata missing.  Outputs
    as bfast_monitor_ex, in the units of y."""
    import torch
    if not (isinstance(Y16, torch.Tensor) and Y16.is_cuda and Y16.dtype == torch.int16 and Y16.dim() == 2
            and Y16.stride(1) == 1):
        raise TypeError("Y16 must be a CUDA int16 [N][P] tensor with unit column stride")
    P = int(Y16.shape[1]) if P is None else int(P)
    out = out if out is not None else _outputs(Y16, P, k, diagnostics)
    _check_out(out, Y16, P)
    d = _dates(dates)
    with torch.cuda.device(Y16.device):
        a = _make_args(Y16, d, n_hist, k, h, lam, out["break"], out["magnitude"], P=P,
                       out_beta=out.get("beta"), out_sigma=out.get("sigma"), out_nbar=out.get("nbar"),
                       out_flags=out.get("flags"), stream=stream)
        a.Y = None
        c = _CodecI16(_dptr(Y16), float(scale), float(offset), int(nodata))
        _check(lib().bfast_monitor_i16(ctypes.byref(c), ctypes.byref(a)))
    out["_dates_keepalive"] = d
    return out


def bfast_monitor_periods(Y, dates, periods, k, h, lam, P=None, diagnostics=False, stream=None):
    """f1 (L391): several monitoring periods [(n_hist_i, N_end_i), ...] in one
    fused launch over the stack (each period's fit on dates [0, N_end_i)).
    Returns the outputs of bfast_monitor_ex stacked period-major: break
    [M][P], magnitude [M][P] (+ beta [M][P][K], sigma, nbar, flags)."""
    import torch
    _check_stack(Y)
    P = int(Y.shape[1]) if P is None else int(P)
    M = len(periods)
    n_arr = np.ascontiguousarray([int(p[0]) for p in periods], dtype=np.int32)
    N_arr = np.ascontiguousarray([int(p[1]) for p in periods], dtype=np.int32)
    flat = _outputs(Y, M * P, k, diagnostics)
    d = _dates(dates)
    with torch.cuda.device(Y.device):
        a = _make_args(Y, d, int(n_arr[0]), k, h, lam, flat["break"], flat["magnitude"], P=P,
                       out_beta=flat.get("beta"), out_sigma=flat.get("sigma"), out_nbar=flat.get("nbar"),
                       out_flags=flat.get("flags"), stream=stream)
        _check(lib().bfast_monitor_periods(ctypes.byref(a), n_arr.ctypes.data, N_arr.ctypes.data, M))
    out = {key: (v.view(M, P, -1) if key == "beta" else v.view(M, P)) for key, v in flat.items()}
    out["_keepalive"] = (d, n_arr, N_arr)
    return out


class Plan:
    """bfast_plan_* wrapper: device constants for one (N, dates, n, k, h, lambda)."""

    def __init__(self, device: int, N: int, dates, n_hist: int, k: int, h: float, lam: float):
        self._h = ctypes.c_void_p()
        self.dates = _dates(dates)
        self.N, self.n_hist, self.k, self.hf, self.lam = int(N), int(n_hist), int(k), float(h), float(lam)
        self.device = int(device)
        _check(lib().bfast_plan_create(ctypes.byref(self._h), self.device, self.N, self.dates.ctypes.data,
                                       self.n_hist, self.k, self.hf, self.lam))

    def execute(self, Y, P=None, diagnostics=False, stream=None, out=None, check_out=True):
        """check_out=False: the output dict may hold raw pointers ({"break":
        int, "magnitude": int}), e.g. an IPC-mapped slice of another
        process's break map (ipc_open)."""
        import torch
        _check_stack(Y)
        if Y.device.index != self.device:
            raise ValueError(f"the plan is on cuda:{self.device}, the stack on {Y.device}")
        P = int(Y.shape[1]) if P is None else int(P)
        out = out if out is not None else _outputs(Y, P, self.k, diagnostics)
        if check_out:
            _check_out(out, Y, P)
        with torch.cuda.device(Y.device):
            a = _make_args(Y, self.dates, self.n_hist, self.k, self.hf, self.lam, out["break"],
                           out["magnitude"], P=P, out_beta=out.get("beta"), out_sigma=out.get("sigma"),
                           out_nbar=out.get("nbar"), out_flags=out.get("flags"), stream=stream)
            _check(lib().bfast_plan_execute(self._h, ctypes.byref(a)))
        return out

    def close(self):
        if self._h:
            lib().bfast_plan_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def _host_ptr(a):
    import torch
    if isinstance(a, torch.Tensor):
        assert not a.is_cuda and a.is_contiguous()
        return int(a.data_ptr())
    assert a.flags["C_CONTIGUOUS"]
    return int(a.ctypes.data)


def bfast_monitor_host(Y_host, dates, n_hist, k, h, lam, out_break=None, out_magnitude=None,
                       P=None, device=-1):
    """End-to-end on host buffers (pinned for full PCIe rate): H2D + kernels + D2H."""
    N, ldY = int(Y_host.shape[0]), int(Y_host.shape[1])
    P = ldY if P is None else int(P)
    if out_break is None:
        out_break = np.empty(P, np.int32)
    if out_magnitude is None:
        out_magnitude = np.empty(P, np.float32)
    d = _dates(dates)
    _check(lib().bfast_monitor_host(_host_ptr(Y_host), N, P, ldY, d.ctypes.data, int(n_hist), int(k),
                                    float(h), float(lam), _host_ptr(out_break), _host_ptr(out_magnitude),
                                    int(device)))
    return out_break, out_magnitude


def bfast_monitor_host_resume(Y_host, dates, n_hist, k, h, lam, out_break, out_magnitude, done=0,
                              tile=1 << 22, max_tiles=-1, P=None, device=-1) -> int:
    """Tile-by-tile host streaming with resume (f2): processes pixels
    [done, P) in tiles, at most max_tiles of them; returns the new `done`
    (pass it back to resume).  out_break / out_magnitude: host arrays [P]."""
    N, ldY = int(Y_host.shape[0]), int(Y_host.shape[1])
    P = ldY if P is None else int(P)
    d = _dates(dates)
    dn = ctypes.c_int64(int(done))
    _check(lib().bfast_monitor_host_resume(_host_ptr(Y_host), N, P, ldY, d.ctypes.data, int(n_hist), int(k),
                                           float(h), float(lam), _host_ptr(out_break), _host_ptr(out_magnitude),
                                           int(device), int(tile), int(max_tiles), ctypes.byref(dn)))
    return int(dn.value)


def bfast_valid_dates(Y, P=None, stream=None):
    """f2 scan (L291, L379): int32 device tensor keep[N], 1 where the date
    slice holds any value among pixels [0, P)."""
    import torch
    _check_stack(Y)
    N, ldY = int(Y.shape[0]), int(Y.shape[1])
    P = ldY if P is None else int(P)
    keep = torch.empty(N, dtype=torch.int32, device=Y.device)
    with torch.cuda.device(Y.device):
        _check(lib().bfast_valid_dates(_dptr(Y), N, P, ldY, _dptr(keep), _stream_ptr(stream)))
    return keep


def bfast_gather_dates(Y, idx, P=None, stream=None):
    """f2 gather: the slices idx (int32 device tensor) of Y as a compact
    [len(idx)][P] device stack."""
    import torch
    _check_stack(Y)
    ldY = int(Y.shape[1])
    P = ldY if P is None else int(P)
    assert idx.dtype == torch.int32 and idx.device == Y.device
    Yc = torch.empty((int(idx.numel()), P), dtype=torch.float32, device=Y.device)
    with torch.cuda.device(Y.device):
        _check(lib().bfast_gather_dates(_dptr(Y), int(Y.shape[0]), ldY, P, _dptr(idx), int(idx.numel()), _dptr(Yc), P,
                                        _stream_ptr(stream)))
    return Yc


def drop_empty_dates(Y, dates, n_hist, P=None):
    """f2 as the paper's pipeline runs it (L291): scan, then gather the
    slices holding any value.  Returns (Yc, dates_c, n_hist_c, keep_idx):
    the compact stack, its dates, the number of kept history dates and the
    original index of every kept date (host int64)."""
    import torch
    keep = bfast_valid_dates(Y, P).cpu().numpy()
    keep_idx = np.flatnonzero(keep).astype(np.int64)
    idx = torch.from_numpy(keep_idx.astype(np.int32)).to(Y.device)
    Yc = bfast_gather_dates(Y, idx, P)
    d = _dates(dates)
    return Yc, d[keep_idx], int(np.count_nonzero(keep_idx < int(n_hist))), keep_idx


def original_break_offsets(brk, keep_idx, n_hist_c, n_hist):
    """Break offsets on a compacted stack (relative to its monitoring start)
    as offsets from the original monitoring start: keep_idx[n_c + b] - n;
    -1 / -2 unchanged (index mapping only)."""
    b = np.asarray(brk)
    out = b.copy()
    hit = b >= 0
    out[hit] = np.asarray(keep_idx)[int(n_hist_c) + b[hit]] - int(n_hist)
    return out


def bfast_monitor_multi(Y_host, dates, n_hist, k, h, lam, devices, out_break=None, out_magnitude=None,
                        P=None):
    N, ldY = int(Y_host.shape[0]), int(Y_host.shape[1])
    P = ldY if P is None else int(P)
    if out_break is None:
        out_break = np.empty(P, np.int32)
    if out_magnitude is None:
        out_magnitude = np.empty(P, np.float32)
    devs = (ctypes.c_int * len(devices))(*devices)
    d = _dates(dates)
    _check(lib().bfast_monitor_multi(_host_ptr(Y_host), N, P, ldY, d.ctypes.data, int(n_hist), int(k),
                                     float(h), float(lam), ctypes.cast(devs, ctypes.c_void_p),
                                     len(devices), _host_ptr(out_break), _host_ptr(out_magnitude)))
    return out_break, out_magnitude


def bfast_monitor_shards(shards, dates, n_hist, k, h, lam, gather_device, out_break=None, out_magnitude=None):
    """Device-resident shards -> one break map on `gather_device` (each
    shard's kernel stores straight into it over peer access).  shards: list
    of CUDA float32 [N][ldY] tensors (any devices, unit column stride)."""
    import torch
    for Y in shards:
        _check_stack(Y)
    N = int(shards[0].shape[0])
    Ps = [int(Y.shape[1]) for Y in shards]
    total = sum(Ps)
    gdev = torch.device("cuda", int(gather_device))
    if out_break is None:
        out_break = torch.empty(total, dtype=torch.int32, device=gdev)
    if out_magnitude is None:
        out_magnitude = torch.empty(total, dtype=torch.float32, device=gdev)
    n = len(shards)
    ys = (ctypes.c_void_p * n)(*[Y.data_ptr() for Y in shards])
    ps = (ctypes.c_int64 * n)(*Ps)
    lds = (ctypes.c_int64 * n)(*[int(Y.stride(0)) for Y in shards])
    devs = (ctypes.c_int * n)(*[Y.device.index for Y in shards])
    d = _dates(dates)
    _check(lib().bfast_monitor_shards(ctypes.cast(ys, ctypes.c_void_p), ctypes.cast(ps, ctypes.c_void_p),
                                      ctypes.cast(lds, ctypes.c_void_p), ctypes.cast(devs, ctypes.c_void_p), n,
                                      N, d.ctypes.data, int(n_hist), int(k), float(h), float(lam),
                                      int(gather_device), _dptr(out_break), _dptr(out_magnitude)))
    return out_break, out_magnitude


def ipc_export(t) -> bytes:
    """IPC handle of tensor t's device memory (the CUDA handle of the
    allocation containing it plus t's offset in that allocation)."""
    buf = (ctypes.c_ubyte * IPC_HANDLE_BYTES)()
    _check(lib().bfast_ipc_export(ctypes.c_void_p(t.data_ptr()), ctypes.cast(buf, ctypes.c_void_p)))
    return bytes(buf)


def ipc_open(handle: bytes, device: int = -1) -> int:
    """Map another process's exported allocation; returns the device pointer."""
    buf = (ctypes.c_ubyte * IPC_HANDLE_BYTES).from_buffer_copy(handle)
    ptr = ctypes.c_void_p()
    _check(lib().bfast_ipc_open(ctypes.cast(buf, ctypes.c_void_p), int(device), ctypes.byref(ptr)))
    return int(ptr.value)


def ipc_close(ptr: int):
    _check(lib().bfast_ipc_close(ctypes.c_void_p(ptr)))
