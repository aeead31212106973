"""Host-side checks that need no GPU: the C-ABI library loads and exports every
symbol include/ganns.h declares; the product package does not reach the oracle."""
import ctypes
import os
import re

from conftest import ROOT

HEADER = os.path.join(ROOT, "include", "ganns.h")
LIB = os.path.join(ROOT, "paper_conf_icde_yuwzqzl22_b200", "libganns.so")


def declared_symbols():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"GANNS_API\s+[\w\s\*]*?\b(ganns_\w+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ("ganns_build", "ganns_search"):
        assert s in syms
    assert len(syms) >= 15


def test_library_loads_and_exports_every_declared_symbol():
    lib = ctypes.CDLL(LIB)
    for s in declared_symbols():
        assert hasattr(lib, s), s


def test_binding_lists_every_symbol():
    import paper_conf_icde_yuwzqzl22_b200 as g
    assert sorted(g.ABI_SYMBOLS) == declared_symbols()


def test_product_path_never_imports_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icde_yuwzqzl22_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in text and "ganns_oracle" not in text, f
                assert "from oracle" not in text, f


def test_last_error_without_gpu_calls():
    lib = ctypes.CDLL(LIB)
    lib.ganns_last_error.restype = ctypes.c_char_p
    lib.ganns_graph_info.restype = ctypes.c_int
    assert lib.ganns_graph_info(None, None, None, None, None) == -1   # EINVAL on NULL graph
    assert b"NULL" in lib.ganns_last_error()


def test_binding_refuses_mis_shaped_output_buffers():
    """Buffers the library writes through raw pointers are checked in the binding."""
    import pytest
    import torch
    import paper_conf_icde_yuwzqzl22_b200 as g
    ok = torch.empty((4, 10), dtype=torch.int32)
    g._check_buf(ok, (4, 10), torch.int32, False, "x")
    for bad in (torch.empty((4, 9), dtype=torch.int32), torch.empty((4, 10), dtype=torch.int64),
                torch.empty((10, 4), dtype=torch.int32).t()):
        with pytest.raises(TypeError):
            g._check_buf(bad, (4, 10), torch.int32, False, "x")
    with pytest.raises(TypeError):   # host tensor where a CUDA one is required
        g._check_buf(ok, (4, 10), torch.int32, True, "x")


def test_graph_load_rejects_corrupt_headers_before_allocating(tmp_path):
    """ganns_graph_load validates the header (n, d, d_max, metric) and the exact file
    length before any allocation: a hostile n fails with GANNS_EIO (-5), no throw."""
    import struct
    lib = ctypes.CDLL(LIB)
    lib.ganns_graph_load.argtypes = [ctypes.c_char_p, ctypes.c_int, ctypes.POINTER(ctypes.c_void_p)]
    lib.ganns_graph_load.restype = ctypes.c_int
    lib.ganns_last_error.restype = ctypes.c_char_p
    cases = {
        "huge_n": struct.pack("<8sq4i", b"GANNSG01", 1 << 40, 128, 32, 0, 0),
        "neg_n": struct.pack("<8sq4i", b"GANNSG01", -5, 128, 32, 0, 0),
        "bad_d": struct.pack("<8sq4i", b"GANNSG01", 100, 130, 32, 0, 0),
        "bad_metric": struct.pack("<8sq4i", b"GANNSG01", 100, 128, 32, 7, 0),
        "truncated": struct.pack("<8sq4i", b"GANNSG01", 100, 128, 32, 0, 0) + b"\0" * 400,
        "bad_magic": struct.pack("<8sq4i", b"NOTAGRPH", 100, 128, 32, 0, 0),
    }
    for name, blob in cases.items():
        p = tmp_path / f"{name}.bin"
        p.write_bytes(blob)
        h = ctypes.c_void_p()
        assert lib.ganns_graph_load(str(p).encode(), 0, ctypes.byref(h)) == -5, name
        assert h.value is None


def test_profile_counters_need_a_profile_build():
    """ganns_profile_read is GANNS_ENOTSUP (-4) in the normal build (the per-phase
    timers are compiled in only with -DGANNS_PROFILE=1)."""
    lib = ctypes.CDLL(LIB)
    lib.ganns_profile_read.argtypes = [ctypes.c_void_p, ctypes.c_int]
    lib.ganns_profile_read.restype = ctypes.c_int
    out = (ctypes.c_uint64 * 8)()
    assert lib.ganns_profile_read(ctypes.cast(out, ctypes.c_void_p), 0) == -4
