"""Time the oracle's Algorithm 2 on a full config (all host cores, and optionally
save the graph for the full-size GPU build parity test)."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import oracle  # noqa: E402
import ganns_synth as syn  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--n", type=int, default=0)
ap.add_argument("--group", type=int, default=1536)
ap.add_argument("--l-build", type=int, default=128)
ap.add_argument("--l-local", type=int, default=32)
ap.add_argument("--threads", type=int, default=0)
ap.add_argument("--save", default="")
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
if a.n:
    cfg = syn.with_size(cfg, n=a.n)
X = syn.points(cfg)
th = a.threads or oracle.ncores()
t0 = time.perf_counter()
ids, dists, st = oracle.alg2(X, cfg.degree // 2, cfg.degree, a.group, l_build=a.l_build,
                             l_local=a.l_local, metric=cfg.metric, threads=th)
dt = time.perf_counter() - t0
cpu = open("/proc/cpuinfo").read().split("model name")[1].split("\n")[0].strip(" :\t")
print(json.dumps({"config": cfg.name, "n": cfg.n, "threads": th, "seconds": round(dt, 2),
                  "stats": [int(x) for x in st], "cpu_model": cpu}), flush=True)
if a.save:
    np.save(a.save, ids)
