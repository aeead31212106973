"""Probe: DRAM bytes of a region via tools/dramprof (CUPTI range profiler) vs known
copy bytes, then around C2 search steps (timed unprofiled and profiled)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from tools.dramprof import DramRegion  # noqa: E402


def timed(body):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    body()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / 1e3


a = torch.empty(1 << 30, dtype=torch.float32, device="cuda")
b = torch.empty_like(a)
a.fill_(1.0)
torch.cuda.synchronize()
for reps in (2, 10):
    with DramRegion(0) as r:
        t = timed(lambda: [b.copy_(a) for _ in range(reps)])
    print(json.dumps({"copy_reps": reps, "expect_read": reps * a.numel() * 4, "read": r.read_bytes,
                      "write": r.write_bytes, "gpu_ns": r.gpu_ns, "t_events": t, "err": r.error}),
          flush=True)
t_plain = timed(lambda: [b.copy_(a) for _ in range(10)])
print(json.dumps({"copy10_unprofiled_s": t_plain}), flush=True)
del a, b
torch.cuda.empty_cache()

import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, Pipeline, make_workload  # noqa: E402

cfg = syn.CONFIGS["C2"]
X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
Qds = [torch.from_numpy(q).cuda() for q in Qs]
idx = BenchIndex(g, cfg, Xd, 128, 64)
pipe = Pipeline(torch, idx, Qds, cfg.k, 2)
pipe.run(8, 128, 109)
_, _, st = idx.search(torch.cat(Qds), cfg.k, 128, e=109, stats=True)
st = st.long()
alg = int((4 * cfg.d + 4 * cfg.degree * st[:, 0] + 4 * cfg.d * st[:, 1]).sum()) // 4
for steps in (20, 100):
    t0 = pipe.run(steps, 128, 109)
    with DramRegion(0) as r:
        t1 = pipe.run(steps, 128, 109)
    print(json.dumps({"c2_steps": steps, "ms_unprof": t0 / steps * 1e3, "ms_prof": t1 / steps * 1e3,
                      "dram_read_per_step": r.read_bytes and r.read_bytes / steps,
                      "dram_write_per_step": r.write_bytes and r.write_bytes / steps,
                      "l2_read_sectors_per_step": r.l2_read_sectors and r.l2_read_sectors / steps,
                      "alg_bytes_per_step": alg, "gpu_ns": r.gpu_ns, "err": r.error}), flush=True)
