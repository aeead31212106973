"""Small search + build + HNSW workload for compute-sanitizer runs."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

cfg = syn.with_size(syn.CONFIGS["C1"], n=1500, nq=64)
X = torch.from_numpy(syn.points(cfg)).cuda()
Q = torch.from_numpy(syn.queries(cfg)).cuda()
gr = g.build(X, degree=16, l_build=32, group_size=200)
g.search(gr, X, Q, 10, 48, e=40)
idx = g.build_hnsw(X, syn.hnsw_levels(1500, 8, 1), degree=16, l_build=32, group_size=200)
g.hnsw_search(idx, X, Q, 10, 32)
X9 = torch.from_numpy(syn.random_int_points(600, 384, 0, 15, 3)).cuda()
gr9 = g.build(X9, degree=32, l_build=32, group_size=100)
g.search(gr9, X9, X9[:16].contiguous(), 5, 32)
torch.cuda.synchronize()
print("ok")
