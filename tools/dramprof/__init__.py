"""DRAM traffic of a host-delimited GPU region, from the hardware counters
(CUPTI Range Profiler, one pass, user range -- the region's kernels run as they
do unprofiled).  Measurement infrastructure for bench.py; not product code.

    with DramRegion(device) as r:
        ... enqueue work; synchronize ...
    r.read_bytes, r.write_bytes, r.l2_read_sectors, r.gpu_ns   (None if unavailable; r.error)
"""
from __future__ import annotations

import ctypes as ct
import os
import subprocess

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dramprof.cpp")
_LIB = os.path.join(_HERE, "libdramprof.so")
_CU = "/usr/local/cuda/targets/x86_64-linux"


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-fvisibility=hidden",
                               f"-I{_CU}/include", "-o", tmp, _SRC, f"-L{_CU}/lib", "-lcupti",
                               "-L/usr/local/cuda/lib64/stubs", "-lcuda", f"-Wl,-rpath,{_CU}/lib"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        _lib = ct.CDLL(build())
        _lib.dp_begin.argtypes = [ct.c_int]
        _lib.dp_end.argtypes = [ct.POINTER(ct.c_double), ct.c_int]
        _lib.dp_error.restype = ct.c_char_p
    return _lib


class DramRegion:
    def __init__(self, device: int = 0):
        self.device = device
        self.read_bytes = self.write_bytes = self.l2_read_sectors = self.gpu_ns = None
        self.error = None
        self._on = False

    def __enter__(self):
        try:
            lib = _load()
            rc = lib.dp_begin(self.device)
            if rc != 0:
                self.error = f"dp_begin rc={rc}: {lib.dp_error().decode()}"
            else:
                self._on = True
        except Exception as ex:  # noqa: BLE001
            self.error = repr(ex)
        return self

    def __exit__(self, *a):
        if not self._on:
            return False
        lib = _load()
        out = (ct.c_double * 4)()
        rc = lib.dp_end(out, 4)
        if rc != 0:
            self.error = f"dp_end rc={rc}: {lib.dp_error().decode()}"
            return False
        self.read_bytes, self.write_bytes = float(out[0]), float(out[1])
        self.l2_read_sectors, self.gpu_ns = float(out[2]), float(out[3])
        return False

    @property
    def dram_bytes(self):
        return None if self.read_bytes is None else self.read_bytes + self.write_bytes
