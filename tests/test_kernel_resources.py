"""Register budgets of the build kernels, read from the built library (cuobjdump
-res-usage; no GPU needed).  A Phase-2 round of the C2 build is 1536 one-warp
searches = 10.4 per SM: above 168 registers per thread at most 10 one-warp CTAs fit
an SM and the round runs in two waves (measured: C2 build 0.41 -> 0.51 s).  The wide
(d > 256) build runs a warp group per search at <= 73 registers (7 CTAs of 4 warps
per SM, the shared-memory limit)."""
import os
import re
import shutil
import subprocess

import pytest

from conftest import ROOT

LIB = os.path.join(ROOT, "paper_conf_icde_yuwzqzl22_b200", "libganns.so")
CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"


def _usage():
    if not os.path.exists(LIB) or not os.path.exists(CUOBJDUMP):
        pytest.skip("library or cuobjdump missing")
    out = subprocess.run([CUOBJDUMP, "-res-usage", LIB], capture_output=True, text=True,
                         timeout=300).stdout.split("\n")
    res = {}
    for i, line in enumerate(out[:-1]):
        m = re.search(r"Function (\S+):", line)
        r = re.search(r"REG:(\d+)", out[i + 1])
        if m and r:
            res[m.group(1)] = int(r.group(1))
    return res


def test_build_kernels_register_budget():
    res = _usage()
    seen = 0
    for name, reg in res.items():
        m = re.search(r"(round_search_kernel|phase1_kernel)ILi(\d+)E", name)
        if not m:
            continue
        seen += 1
        nv4 = int(m.group(2))
        limit = 168 if nv4 <= 2 else 73
        assert reg <= limit, (name, reg, limit)
    assert seen >= 40, f"only {seen} build kernels found"
