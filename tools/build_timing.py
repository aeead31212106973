"""Repeated C2 builds: wall time of each with the SM clock sampled (NVML) during it."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import ClockSampler  # noqa: E402
cfg = syn.CONFIGS["C2"]
X = torch.from_numpy(syn.points(cfg)).cuda()
s = int(sys.argv[1]) if len(sys.argv) > 1 else 0
g.build(X[:20000].contiguous(), degree=32, l_build=128)
for rep in range(int(sys.argv[2]) if len(sys.argv) > 2 else 5):
    torch.cuda.synchronize()
    import contextlib
    with (ClockSampler(0) if os.environ.get("NOCLK") != "1" else contextlib.nullcontext()) as clk:
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        t0 = time.perf_counter()
        ev[0].record()
        g.build(X, degree=32, l_build=128, group_size=s, stop_after_phase1=True)
        ev[1].record()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        gpu1 = ev[0].elapsed_time(ev[1]) / 1e3
        g.build(X, degree=32, l_build=128, group_size=s)
        torch.cuda.synchronize()
        t2 = time.perf_counter()
    print(json.dumps({"group": s, "phase1_s": round(t1 - t0, 3), "phase1_gpu_s": round(gpu1, 3), "full_s": round(t2 - t1, 3),
                      "clocks": clk.summary() if clk else None}), flush=True)
