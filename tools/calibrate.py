"""Generator calibration (SURVEY §8(d) "calibration rule"): recall@10 vs l on the
GPU-built NSW graph for a few (rank, noise) settings of the C2 recipe."""
import dataclasses
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import ground_truth, recall_at  # noqa: E402

base = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
settings = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [[24, 0.03, 64]]
for rank, noise, lb in settings:
    cfg = dataclasses.replace(base, rank=rank, noise=noise)
    t0 = time.time()
    X = torch.from_numpy(syn.points(cfg)).cuda()
    Q = torch.from_numpy(syn.queries(cfg)).cuda()
    tg = time.time() - t0
    t0 = time.time()
    graph = g.build(X, metric=cfg.metric, degree=cfg.degree, l_build=lb)
    torch.cuda.synchronize()
    tb = time.time() - t0
    gt = ground_truth(torch, X, Q, cfg.k)
    res = []
    for l in (32, 48, 64, 96, 128, 192, 256, 384, 512):
        ids, _ = g.search(graph, X, Q, cfg.k, l)
        res.append((l, round(recall_at(ids, gt), 4)))
    print(json.dumps({"rank": rank, "noise": noise, "l_build": lb, "gen_s": round(tg, 1),
                      "build_s": round(tb, 2), "recall": res}), flush=True)
