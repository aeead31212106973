"""Search A/B on a config's bench workload: build the bench's graph (or HNSW), then
time K pipelined steps at (l, e) and read their DRAM bytes from the hardware
counters (tools/dramprof).  GANNS_LIB_PATH selects the library variant.
    python tools/search_ab.py --config C3 --l 288 --e 288 [--steps 20]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, Pipeline, make_workload, measure_dram  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--l", type=int, required=True)
ap.add_argument("--e", type=int, default=0)
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
Qds = [torch.from_numpy(q).cuda() for q in Qs]
idx = BenchIndex(g, cfg, Xd, 128, 32)
pipe = Pipeline(torch, idx, Qds, cfg.k, 2)
e = a.e or a.l
pipe.run(6, a.l, e)
ts = [pipe.run(a.steps, a.l, e) for _ in range(a.reps)]
t = sorted(ts)[len(ts) // 2]
dram = measure_dram(lambda: pipe.run(a.steps, a.l, e), 0)
nq = Qs[0].shape[0]
out = {"lib": g.LIB_PATH, "config": a.config, "l": a.l, "e": e, "qps": round(nq * a.steps / t),
       "ms_per_step": round(t / a.steps * 1e3, 4)}
if "error" not in dram:
    out.update(dram_read_per_step=int(dram["read"] / a.steps),
               dram_write_per_step=int(dram["write"] / a.steps),
               l2_read_per_step=int(dram["l2_read"] / a.steps))
else:
    out["dram_error"] = dram["error"]
print(json.dumps(out), flush=True)
