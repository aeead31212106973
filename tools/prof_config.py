"""Profiling driver on exactly the bench's workload: bench.make_workload + BenchIndex
(NSW with l_local, or HNSW for C4), then `--reps` searches of one batch at (l, e)
with an L2 flush between them, so ncu captures a cold launch of the bench's kernel.
    ncu --set full -k regex:search -s 2 -c 1 python tools/prof_config.py --config C4 --l 288 --e 288"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
import ganns_synth as syn  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--l", type=int, required=True)
ap.add_argument("--e", type=int, default=0)
ap.add_argument("--reps", type=int, default=4)
ap.add_argument("--l-build", type=int, default=128)
ap.add_argument("--l-local", type=int, default=32)
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
X, Qs = bench.make_workload(cfg, 0, 1)
Qs = Qs if isinstance(Qs, list) else [Qs]
Xd = torch.from_numpy(X).cuda()
Qd = torch.from_numpy(Qs[0]).cuda()
index = bench.BenchIndex(g, cfg, Xd, a.l_build, a.l_local)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(a.reps):
    flush.zero_()
    index.search(Qd, cfg.k, a.l, e=a.e)
torch.cuda.synchronize()
print("done", a.config, a.l, a.e, index.build_stats)
