"""Group-size sweep of the GGraphCon build (R-C14): per group size, the build's wall
time (median of 3) and the graph's search quality/speed: recall@10 over 40K queries and
pipelined QPS at a few (l, e)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, Pipeline, ground_truth, make_workload, recall_at  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
groups = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "1024,2048").split(",")]
les = [tuple(int(y) for y in x.split(":")) for x in
       (sys.argv[3] if len(sys.argv) > 3 else "112:112,128:109,128:128").split(",")]
lb = int(os.environ.get("LB", "128"))
X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
Qd = torch.from_numpy(np.concatenate(Qs)).cuda()
gt = ground_truth(torch, Xd, Qd, cfg.k, cfg.metric)
g.build(Xd[:20000].contiguous(), degree=cfg.degree, l_build=lb)   # module warm-up
for s in groups:
    ts = []
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        gr = g.build(Xd, metric=cfg.metric, degree=cfg.degree, l_build=lb, group_size=s,
                     l_local=int(os.environ.get("LL", "0")))
        torch.cuda.synchronize()
        ts.append(time.perf_counter() - t0)
    idx = BenchIndex.__new__(BenchIndex)
    idx.g, idx.cfg, idx.Xd, idx.hnsw, idx.graph, idx.idx = g, cfg, Xd, False, gr, None
    nq = Qs[0].shape[0]
    pipe = Pipeline(torch, idx, [Qd[b * nq:(b + 1) * nq] for b in range(4)], cfg.k, 2)
    res = []
    for l, e in les:
        ids, _ = g.search(gr, Xd, Qd, cfg.k, l, e=e)
        r = recall_at(ids, gt)
        t = min(pipe.run(8, l, e) for _ in range(3))
        res.append({"l": l, "e": e, "recall": round(r, 4), "qps": round(8 * nq / t)})
    print(json.dumps({"group": s, "l_build": lb, "build_s": sorted(ts)[1], "build_all": [round(x, 3) for x in ts],
                      "search": res}), flush=True)
