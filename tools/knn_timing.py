"""KNN graph (NEXT-4) timing: neighbours-of-neighbours iterations from
random lists on C1/C2-shaped data (wall time of g.build_knn, iterations, recall of
the lists against exact ground truth on a query-free sample of points).
    python tools/knn_timing.py C2 16"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
K = int(sys.argv[2]) if len(sys.argv) > 2 else 16
X = syn.points(cfg)
Xd = torch.from_numpy(X).cuda()
init = syn.random_graph(len(X), K, 7)
m = min(20000, len(X))
g.build_knn(Xd[:m].contiguous(), syn.random_graph(m, K, 8), K, max_iters=3)   # warm-up
torch.cuda.synchronize()
t0 = time.perf_counter()
gr, it, ch = g.build_knn(Xd, init, K, max_iters=50)
torch.cuda.synchronize()
t = time.perf_counter() - t0
lists = gr.adjacency()
rng = np.random.default_rng(3)
sample = rng.choice(len(X), 200, replace=False)
# exact K nearest (excluding the point itself) of the sampled points, fp64 on the GPU
Xg = Xd.double()
S = Xg[torch.from_numpy(sample).cuda()]
d2 = (S * S).sum(1, keepdim=True) - 2 * S @ Xg.T + (Xg * Xg).sum(1)[None]
d2[torch.arange(len(sample)), torch.from_numpy(sample).cuda()] = float("inf")
gt = torch.topk(d2, K, largest=False).indices.cpu().numpy()
rec = np.mean([len(set(lists[v]) & set(gt[i])) / K for i, v in enumerate(sample)])
print({"config": cfg.name, "n": len(X), "K": K, "seconds": round(t, 3), "iterations": it,
       "changed_last": ch, "recall_at_K_sample200": round(float(rec), 4)}, flush=True)
