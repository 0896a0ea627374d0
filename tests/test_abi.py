"""C-ABI checks that need no GPU: the library loads, exports every symbol
include/bfast.h declares, and host-side logic (validation, sharding) behaves.
No compute call is made here."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_icde_giesekerhvo20_b200 import binding

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "bfast.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[a-z_0-9]+\s*\**\s*(bfast_[a-z_0-9]+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_north_star_entry():
    names = _declared_functions()
    assert "bfast_monitor" in names and len(names) >= 10
    assert sorted(binding.EXPORTS) == names


def test_library_exports_every_declared_symbol():
    L = ctypes.CDLL(binding.LIB_PATH)
    for name in _declared_functions():
        assert hasattr(L, name), name


def test_abi_version_and_status_strings():
    assert binding.abi_version() == 1
    L = binding.lib()
    assert L.bfast_status_string(-1) == b"BFAST_EINVAL"
    assert L.bfast_status_string(0) == b"BFAST_OK"


def test_shard_range_partitions_in_tiles():
    for P in (0, 1, 127, 128, 1000, 16_777_216, 120_560_400):
        for world in (1, 2, 3, 4, 8):
            ranges = [binding.shard_range(P, r, world) for r in range(world)]
            assert ranges[0][0] == 0 and ranges[-1][1] == P
            for (b0, e0), (b1, e1) in zip(ranges, ranges[1:]):
                assert e0 == b1
            for b, e in ranges:
                assert b % 128 == 0 and e >= b
            sizes = [e - b for b, e in ranges]
            if P >= 128 * world:
                assert max(sizes) - min(sizes) <= 128


def test_validation_rejects_before_touching_the_device():
    """Argument errors return EINVAL from host code (no CUDA call), so they
    are testable without a GPU."""
    L = binding.lib()
    d = (np.arange(10) / 23.0).astype(np.float64)
    dp = d.ctypes.data
    # N < 2
    assert L.bfast_monitor(None, 1, 0, dp, 1, 1, 0.25, 1.65, None, None) == binding.BFAST_EINVAL
    # n_hist out of range
    assert L.bfast_monitor(None, 10, 0, dp, 10, 1, 0.25, 1.65, None, None) == binding.BFAST_EINVAL
    assert b"n_hist" in L.bfast_last_error()
    # hf out of (0, 1]
    assert L.bfast_monitor(None, 10, 0, dp, 5, 1, 1.5, 1.65, None, None) == binding.BFAST_EINVAL
    # lambda
    assert L.bfast_monitor(None, 10, 0, dp, 5, 1, 0.25, -1.0, None, None) == binding.BFAST_EINVAL
    # dates not increasing
    bad = d[::-1].copy()
    assert L.bfast_monitor(None, 10, 0, bad.ctypes.data, 5, 1, 0.25, 1.65, None, None) == binding.BFAST_EINVAL
    # k too large
    assert L.bfast_monitor(None, 10, 0, dp, 5, 7, 0.25, 1.65, None, None) == binding.BFAST_EUNSUPPORTED
    # NULL pointers with P > 0 (host path)
    assert L.bfast_monitor_host(None, 10, 5, 5, dp, 5, 1, 0.25, 1.65, None, None, -1) == binding.BFAST_EINVAL
    # P = 0 host path is a no-op that needs no device
    assert L.bfast_monitor_host(None, 10, 0, 0, dp, 5, 1, 0.25, 1.65, None, None, -1) == binding.BFAST_OK


def test_binding_fails_loudly_without_library(monkeypatch, tmp_path):
    monkeypatch.setattr(binding, "_lib", None)
    monkeypatch.setattr(binding, "LIB_PATH", str(tmp_path / "missing.so"))
    with pytest.raises(ImportError):
        binding.lib()
