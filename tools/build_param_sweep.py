"""Build-parameter sweep (R-C13, R-C14, the explore budget e of P:402): for each
(l_build, e_build, l_local, group size) the build's wall time (median of 3, SM clock
sampled) and the graph's search QPS at recall@10 >= 0.95 (cheapest (l, e) found by a
small sweep, pipelined QPS as in bench.py).
    python tools/build_param_sweep.py C2 "128:128:64:0,128:112:64:0,..."   (lb:eb:ll:s)"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, ClockSampler, Pipeline, ground_truth, make_workload, recall_at  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
combos = [tuple(int(y) for y in x.split(":")) for x in sys.argv[2].split(",")]
X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
Qd = torch.from_numpy(np.concatenate(Qs)).cuda()
gt = ground_truth(torch, Xd, Qd, cfg.k, cfg.metric)     # also brings the GPU out of idle
g.build(Xd[:20000].contiguous(), degree=cfg.degree, l_build=128)
nq = Qs[0].shape[0]
for lb, eb, ll, s in combos:
    ts = []
    with ClockSampler(0) as clk:
        for _ in range(3):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            gr = g.build(Xd, metric=cfg.metric, degree=cfg.degree, l_build=lb, e_build=eb,
                         l_local=ll, group_size=s)
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
    idx = BenchIndex.__new__(BenchIndex)
    idx.g, idx.cfg, idx.Xd, idx.hnsw, idx.graph, idx.idx = g, cfg, Xd, False, gr, None
    pipe = Pipeline(torch, idx, [Qd[b * nq:(b + 1) * nq] for b in range(4)], cfg.k, 2)
    feas = []
    for l in range(96, 200, 8):
        for e in sorted({l, int(round(0.92 * l)), int(round(0.85 * l))}):
            ids, _ = g.search(gr, Xd, Qd, cfg.k, l, e=e)
            r = recall_at(ids, gt)
            if r >= 0.95:
                feas.append((e, l, round(r, 5)))
        if len(feas) >= 4:
            break
    best = None
    for e, l, r in sorted(feas)[:4]:
        t = min(pipe.run(12, l, e) for _ in range(3))
        q = 12 * nq / t
        if best is None or q > best["qps"]:
            best = {"l": l, "e": e, "recall": r, "qps": round(q)}
    print(json.dumps({"l_build": lb, "e_build": eb, "l_local": ll, "group": s or "auto",
                      "build_s": round(sorted(ts)[1], 4), "build_all": [round(x, 3) for x in ts],
                      "clocks": clk.summary(), "qps_at_0.95": best,
                      "stats": list(gr.build_stats)}), flush=True)
