"""Quick kernel timing: build the config's graph, time ganns_search at a few l."""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import ground_truth, recall_at  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--ls", default="64,128,256")
ap.add_argument("--l-build", type=int, default=0)
ap.add_argument("--group", type=int, default=0)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--nq-mult", default="1", help="comma list: time batches of m x nq queries")
ap.add_argument("--overlap", type=int, default=0, help="also time this many back-to-back "
                "batches on one stream and alternating over 2 and 3 streams (no flush between)")
ap.add_argument("--nqs", default="", help="comma list: also time the first m queries alone")
ap.add_argument("--orders", default="", help="comma list of pivot counts P: also time the batch "
                "reordered by each query's nearest of P evenly spaced points (locality experiment)")
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
X = torch.from_numpy(syn.points(cfg)).cuda()
Q = torch.from_numpy(syn.queries(cfg)).cuda()
torch.cuda.synchronize()
t0 = time.time()
graph = g.build(X, metric=cfg.metric, degree=cfg.degree, l_build=a.l_build, group_size=a.group)
torch.cuda.synchronize()
print(json.dumps({"build_s": round(time.time() - t0, 3), "stats": graph.build_stats}), flush=True)
gt = ground_truth(torch, X, Q, cfg.k)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for l in [int(x) for x in a.ls.split(",")]:
    ids, _, st = g.search(graph, X, Q, cfg.k, l, stats=True)
    st = st.long()
    byts = int((4 * cfg.d + 4 * cfg.degree * st[:, 0] + 4 * cfg.d * st[:, 1]).sum()) + 8 * cfg.k * len(Q)
    ts = []
    for _ in range(a.reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        g.search(graph, X, Q, cfg.k, l)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1) / 1e3)
    t = sorted(ts)[len(ts) // 2]
    for m in [int(x) for x in a.nq_mult.split(",")]:
        if m == 1:
            continue
        Qm = Q.repeat(m, 1)
        tm = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            g.search(graph, X, Qm, cfg.k, l)
            e1.record()
            e1.synchronize()
            tm.append(e0.elapsed_time(e1) / 1e3)
        tmm = sorted(tm)[len(tm) // 2]
        print(json.dumps({"l": l, "nq": len(Qm), "ms": round(tmm * 1e3, 3), "qps": round(len(Qm) / tmm)}))
    for m in [int(x) for x in a.nqs.split(",") if x]:
        Qm = Q[:m].contiguous()
        tm = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            g.search(graph, X, Qm, cfg.k, l)
            e1.record()
            e1.synchronize()
            tm.append(e0.elapsed_time(e1) / 1e3)
        tmm = sorted(tm)[len(tm) // 2]
        print(json.dumps({"l": l, "nq": m, "ms": round(tmm * 1e3, 3), "qps": round(m / tmm)}))
    if a.overlap:
        outs = [(torch.empty_like(ids), torch.empty(ids.shape, dtype=torch.float32, device="cuda"))
                for _ in range(a.overlap)]
        for ns in (1, 2, 3):
            strs = [torch.cuda.Stream() for _ in range(ns)]
            tt = []
            for _ in range(a.reps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
                e0.record()
                for s_ in strs:
                    s_.wait_event(e0)
                for b in range(a.overlap):
                    g.search(graph, X, Q, cfg.k, l, out=outs[b], stream=strs[b % ns])
                for s_ in strs:
                    ev = torch.cuda.Event()
                    ev.record(s_)
                    torch.cuda.current_stream().wait_event(ev)
                e1.record()
                e1.synchronize()
                tt.append(e0.elapsed_time(e1) / 1e3)
            tm_ = sorted(tt)[len(tt) // 2]
            print(json.dumps({"l": l, "batches": a.overlap, "streams": ns, "ms_per_batch": round(tm_ / a.overlap * 1e3, 3),
                              "qps": round(a.overlap * len(Q) / tm_)}))
    for P in [int(x) for x in a.orders.split(",") if x]:
        piv = X[:: max(1, len(X) // P)][:P]
        lab = torch.cdist(Q, piv).argmin(1)
        Qo = Q[torch.argsort(lab, stable=True)].contiguous()
        to = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record()
            g.search(graph, X, Qo, cfg.k, l)
            e1.record()
            e1.synchronize()
            to.append(e0.elapsed_time(e1) / 1e3)
        tom = sorted(to)[len(to) // 2]
        print(json.dumps({"l": l, "order_pivots": P, "ms": round(tom * 1e3, 3), "qps": round(len(Q) / tom)}))
    print(json.dumps({"l": l, "recall": round(recall_at(ids, gt), 4), "ms": round(t * 1e3, 3),
                      "qps": round(len(Q) / t), "alg_GBps": round(byts / t / 1e9, 1),
                      "iters": round(float(st[:, 0].float().mean()), 1),
                      "comps_per_iter": round(float(st[:, 1].sum() / st[:, 0].sum()), 2)}), flush=True)
