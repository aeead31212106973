"""Compile libganns.so for sm_100a in-tree (nvcc; objects built in parallel).

Called by __graft_entry__.build() and by the Python binding when the library is
missing or older than its sources.  Never falls back to anything else.
"""
from __future__ import annotations

import concurrent.futures as cf
import glob
import os
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libganns.so")
OBJ = os.path.join(PKG, "_obj")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden",
         "-I", os.path.join(ROOT, "include")] + os.environ.get("GANNS_NVCC_EXTRA", "").split()

# (source, extra defines, object name)
UNITS = [("api.cu", [], "api.o"), ("search.cu", [], "search.o"), ("knn.cu", [], "knn.o"),
         ("build.cu", [], "build.o")] + \
        [("search_inst.cu", [f"-DGANNS_NV4={v}"], f"search_nv{v}.o") for v in (1, 2, 4, 8)] + \
        [("build_inst.cu", [f"-DGANNS_NV4={v}"], f"build_nv{v}.o") for v in (1, 2, 4, 8)]
# GANNS_DEV=1: developer flavour with only the d <= 128 / d_max <= 32 / L2
# instances (fast rebuilds while tuning).  Never shipped: the flavour stamp
# makes build() rebuild the full library.
DEV_UNITS = [("api.cu", ["-DGANNS_DEV_NV1"], "dev_api.o"),
             ("search.cu", ["-DGANNS_DEV_NV1"], "dev_search.o"),
             ("knn.cu", [], "dev_knn.o"),
             ("build.cu", ["-DGANNS_DEV_NV1"], "dev_build.o"),
             ("search_inst.cu", ["-DGANNS_NV4=1", "-DGANNS_DEV_ONE"], "dev_search_nv1.o"),
             ("build_inst.cu", ["-DGANNS_NV4=1", "-DGANNS_DEV_ONE"], "dev_build_nv1.o")]
FLAVOR = os.path.join(PKG, "libganns.flavor")


def _flavor():
    return "dev" if os.environ.get("GANNS_DEV") == "1" else "full"


def _sources():
    return glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh")) + \
        glob.glob(os.path.join(CSRC, "*.h")) + [os.path.join(ROOT, "include", "ganns.h")]


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    if not os.path.exists(FLAVOR) or open(FLAVOR).read().strip() != _flavor():
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in _sources())


def _compile(unit):
    src, defs, obj = unit
    out = os.path.join(OBJ, obj)
    cmd = [NVCC, *ARCH, *FLAGS, *defs, "-c", os.path.join(CSRC, src), "-o", out]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"nvcc failed for {src} {defs}:\n{r.stderr}")
    return out


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not stale():
        return LIB
    os.makedirs(OBJ, exist_ok=True)
    units = DEV_UNITS if _flavor() == "dev" else UNITS
    with cf.ThreadPoolExecutor(max_workers=max(2, min(len(units), os.cpu_count() or 2))) as ex:
        objs = list(ex.map(_compile, units))
    tmp = LIB + f".{os.getpid()}.tmp"
    cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr}")
    os.replace(tmp, LIB)
    with open(FLAVOR, "w") as f:
        f.write(_flavor())
    if verbose:
        print("built", LIB)
    return LIB


def build_variant(out: str, defines: list[str], dev: bool = True) -> str:
    """A/B and profiling variants (tools/): the library with extra -D flags, linked to
    `out`, objects in their own directory; the default library is untouched.
    dev=True compiles only the d <= 128 / d_max <= 32 instances (the DEV_UNITS)."""
    tag = os.path.splitext(os.path.basename(out))[0]
    odir = os.path.join(OBJ, "var_" + tag)
    os.makedirs(odir, exist_ok=True)
    units = [(src, defs + defines, obj) for src, defs, obj in (DEV_UNITS if dev else UNITS)]

    def comp(u):
        src, defs, obj = u
        o = os.path.join(odir, obj)
        r = subprocess.run([NVCC, *ARCH, *FLAGS, *defs, "-c", os.path.join(CSRC, src), "-o", o],
                           capture_output=True, text=True)
        if r.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src} {defs}:\n{r.stderr}")
        return o
    with cf.ThreadPoolExecutor(max_workers=max(2, min(len(units), os.cpu_count() or 2))) as ex:
        objs = list(ex.map(comp, units))
    os.makedirs(os.path.dirname(os.path.abspath(out)), exist_ok=True)
    r = subprocess.run([NVCC, *ARCH, "-shared", "-o", out, *objs, "-lcudart"], capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"link failed:\n{r.stderr}")
    return out


if __name__ == "__main__":
    build(force=True, verbose=True)
