"""Hardware check of the tcgen05 / TMEM / bulk-copy primitives (csrc/sm100.cuh)
by a standalone probe: every MMA shape the tensor-core kernel uses is
compared with a host fp64 GEMM of the same bf16 operands."""
import os
import subprocess

import pytest

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def test_umma_probe(tmp_path):
    exe = str(tmp_path / "umma_probe")
    subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O2", "-std=c++17",
                    os.path.join(HERE, "native", "umma_probe.cu"), "-o", exe], check=True)
    r = subprocess.run([exe], capture_output=True, text=True, timeout=120)
    print(r.stdout)
    assert r.returncode == 0 and "ALL OK" in r.stdout, r.stdout + r.stderr


def test_compute_sanitizer_clean():
    """memcheck / racecheck / synccheck on a small invocation of both kernels
    (and the fp64 refit kernel)."""
    import shutil
    import sys
    exe = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"
    script = os.path.join(os.path.dirname(HERE), "tools", "sanitize_case.py")
    for tool in ("memcheck", "racecheck", "synccheck"):
        r = subprocess.run([exe, "--tool", tool, "--error-exitcode", "3", sys.executable, script],
                           capture_output=True, text=True, timeout=900)
        out = r.stdout + r.stderr
        if "closed on this pool" in out:
            # the GPU pool replaces compute-sanitizer by a refusal (runs under it
            # left GPUs needing a reset); the kernels' own parity and the
            # determinism tests stand in for it there
            pytest.skip("compute-sanitizer is disabled on this GPU pool")
        assert r.returncode == 0, out[-3000:]
        assert "0 errors" in out, out[-3000:]
        assert "hazard" not in out.lower() or "0 hazards" in out.lower(), out[-3000:]
