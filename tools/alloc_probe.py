"""Host cost of the build's allocations: cudaMalloc / cudaFree of the build-scratch
sizes vs the stream-ordered pool (cudaMallocAsync / cudaFreeAsync, release threshold
raised), each repeated -- for the wall-vs-GPU build-time gap."""
import ctypes as ct
import json
import statistics
import time

import torch

torch.cuda.init()
torch.zeros(1, device="cuda")
rt = ct.CDLL("libcudart.so.12") if False else None
for name in ("libcudart.so.12", "libcudart.so"):
    try:
        rt = ct.CDLL(name)
        break
    except OSError:
        pass
P = ct.c_void_p
sizes = [128 << 20, 128 << 20, 64 << 20, 64 << 20, 4 << 20, 4 << 20, 4 << 20, 128 << 20]


def malloc_free():
    ptrs = []
    t0 = time.perf_counter()
    for s in sizes:
        p = P()
        assert rt.cudaMalloc(ct.byref(p), ct.c_size_t(s)) == 0
        ptrs.append(p)
    t1 = time.perf_counter()
    for p in ptrs:
        assert rt.cudaFree(p) == 0
    t2 = time.perf_counter()
    return t1 - t0, t2 - t1


def pool():
    dev = ct.c_int(0)
    mp = P()
    rt.cudaDeviceGetDefaultMemPool(ct.byref(mp), dev)
    thr = ct.c_uint64(2 ** 64 - 1)
    rt.cudaMemPoolSetAttribute(mp, 4, ct.byref(thr))   # cudaMemPoolAttrReleaseThreshold = 4
    s = P(torch.cuda.current_stream().cuda_stream)
    ptrs = []
    t0 = time.perf_counter()
    for sz in sizes:
        p = P()
        assert rt.cudaMallocAsync(ct.byref(p), ct.c_size_t(sz), s) == 0
        ptrs.append(p)
    t1 = time.perf_counter()
    for p in ptrs:
        assert rt.cudaFreeAsync(p, s) == 0
    rt.cudaStreamSynchronize(s)
    t2 = time.perf_counter()
    return t1 - t0, t2 - t1


for name, fn in (("cudaMalloc/Free", malloc_free), ("pool", pool)):
    res = [fn() for _ in range(10)]
    print(json.dumps({"api": name, "alloc_ms": [round(a * 1e3, 2) for a, _ in res],
                      "free_ms": [round(b * 1e3, 2) for _, b in res],
                      "median_total_ms": round(statistics.median(a + b for a, b in res) * 1e3, 2)}),
          flush=True)
