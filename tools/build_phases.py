"""Phase-resolved C2 build timing (the staged ABI with CUDA events around Phase 1 and
around the Phase-2 rounds), repeated, with SM and memory clocks sampled by NVML --
for the bimodal build-time question."""
import json
import os
import statistics
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pynvml as nv  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 8
warm = sys.argv[2] if len(sys.argv) > 2 else "gemm"
cfg = syn.CONFIGS["C2"]
X = torch.from_numpy(syn.points(cfg)).cuda()
nv.nvmlInit()
h = nv.nvmlDeviceGetHandleByIndex(0)
samples, stop = [], threading.Event()


def sampler():
    while not stop.is_set():
        try:
            samples.append((time.perf_counter(), nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM),
                            nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_MEM),
                            int(nv.nvmlDeviceGetCurrentClocksEventReasons(h))))
        except Exception:
            pass
        time.sleep(0.002)


th = threading.Thread(target=sampler, daemon=True)
th.start()
if warm == "gemm":
    a = torch.randn(8192, 8192, device="cuda")
    for _ in range(20):
        a @ a
g.build(X[:20000].contiguous(), degree=32, l_build=128, l_local=32)
torch.cuda.synchronize()


def ev():
    e = torch.cuda.Event(enable_timing=True)
    e.record()
    return e


for r in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    b = g.StagedBuild(X, degree=32, l_build=128, l_local=32)
    S, G, dm, dx = b.info()
    torch.cuda.synchronize()
    tb = time.perf_counter()
    e0 = ev()
    b.phase1(0, G)
    e1 = ev()
    for i in range(1, G):
        lo, hi = b.group_rows(i, i + 1)
        b.round_apply(i, *b.round_search(i, lo, hi))
    e2 = ev()
    e2.synchronize()
    tf = time.perf_counter()
    gr = b.finish()
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    t2 = time.perf_counter()
    del gr
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    win = [s for s in samples if t0 <= s[0] <= t1]
    print(json.dumps({"rep": r, "wall_s": round(t1 - t0, 4), "begin_s": round(tb - t0, 4),
                      "enqueue_to_done_s": round(tf - tb, 4), "finish_s": round(t1 - tf, 4),
                      "graph_free_s": round(t3 - t2, 4),
                      "phase1_s": round(e0.elapsed_time(e1) / 1e3, 4),
                      "phase2_s": round(e1.elapsed_time(e2) / 1e3, 4),
                      "sm_mhz": statistics.median([s[1] for s in win]) if win else None,
                      "mem_mhz": [min(s[2] for s in win), max(s[2] for s in win)] if win else None,
                      "reasons": sorted({s[3] for s in win})}), flush=True)
    time.sleep(0.5 if r % 2 else 0.0)
stop.set()
