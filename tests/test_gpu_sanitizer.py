"""compute-sanitizer memcheck / racecheck / synccheck on a small build + search +
HNSW + wide-row workload (SURVEY §4 test layer 2).  The kernels use shared
memory written by TMA (async proxy) and by single lanes; racecheck guards the
warp-level ordering (__syncwarp / fence.proxy.async / mbarrier phases)."""
import os
import shutil
import subprocess
import sys

import pytest
import torch

from conftest import ROOT

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

SAN = shutil.which("compute-sanitizer") or "/usr/local/cuda/bin/compute-sanitizer"


@pytest.mark.parametrize("tool", ["memcheck", "racecheck", "synccheck"])
def test_sanitizer_clean(tool):
    if not os.path.exists(SAN):
        pytest.skip("compute-sanitizer not found")
    r = subprocess.run([SAN, "--tool", tool, "--print-limit", "5", sys.executable,
                        os.path.join(ROOT, "tools", "sanitize_small.py")],
                       capture_output=True, text=True, timeout=900, cwd=ROOT)
    out = r.stdout + r.stderr
    if "closed on this pool" in out:
        # the GPU pool's compute-sanitizer wrapper refuses to run (it has left GPUs
        # needing a reset); parity against the oracle stays the correctness gate
        pytest.skip("compute-sanitizer is closed on this GPU pool")
    assert r.returncode == 0, out[-3000:]
    assert "ok" in r.stdout
    if tool == "racecheck":
        assert "0 hazards displayed (0 errors, 0 warnings)" in out, out[-3000:]
    else:
        assert "ERROR SUMMARY: 0 errors" in out, out[-3000:]
