"""Profiling driver: build the config's graph, then run the search kernel a few
times at a fixed l so ncu can capture exactly those launches.
    ncu --set full -k regex:search_kernel -s 2 -c 1 python tools/prof_search.py --l 96"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--l", type=int, default=96)
ap.add_argument("--e", type=int, default=0)
ap.add_argument("--reps", type=int, default=4)
ap.add_argument("--l-build", type=int, default=128)
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
X = torch.from_numpy(syn.points(cfg)).cuda()
Q = torch.from_numpy(syn.queries(cfg)).cuda()
graph = g.build(X, metric=cfg.metric, degree=cfg.degree, l_build=a.l_build)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(a.reps):
    flush.zero_()
    g.search(graph, X, Q, cfg.k, a.l, e=a.e)
torch.cuda.synchronize()
print("done", graph.build_stats)
