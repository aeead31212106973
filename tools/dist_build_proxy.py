"""NEXT-2 proxy on one GPU: where do Algorithm-2 rounds become throughput-bound, and
what would a W-GPU build (dist.build_distributed) take?

A large single graph is built with the staged ABI on one GPU.  Every `--every`-th
round, the round's searches are also run split in W chunks (W = 2, 4, 8), each
chunk timed alone with CUDA events (the search only reads the state, so the
repeats do not change the graph); the W-GPU round time is the slowest chunk.
Phase 1 of G/W groups is timed on a second state.  Exchange costs are MODELLED
(all-gather latency + bytes / bandwidth, stated in the output), not measured --
this box has one GPU.
    python tools/dist_build_proxy.py --n 20000000 [--every 25]"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--n", type=int, default=20_000_000)
ap.add_argument("--every", type=int, default=25)
ap.add_argument("--l-build", type=int, default=128)
ap.add_argument("--l-local", type=int, default=32)
ap.add_argument("--ag-latency-us", type=float, default=25.0,
                help="modelled NCCL all-gather latency per exchange (NVSwitch, small message)")
ap.add_argument("--ag-gbps", type=float, default=300.0,
                help="modelled all-gather bandwidth per GPU for the Phase-1 rows")
a = ap.parse_args()
cfg = syn.with_size(syn.CONFIGS[a.config], n=a.n)
X = torch.from_numpy(syn.points(cfg)).cuda()
torch.cuda.synchronize()
Ws = (1, 2, 4, 8)
kw = dict(metric=cfg.metric, degree=cfg.degree, l_build=a.l_build, l_local=a.l_local)


def ev_time(fn):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    out = fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / 1e3, out


g.build(X[:20000].contiguous(), degree=cfg.degree, l_build=a.l_build, l_local=a.l_local)
b = g.StagedBuild(X, **kw)
S, G, dm, dx = b.info()
t_p1 = {}
t_p1[1], _ = ev_time(lambda: b.phase1(0, G))
for W in Ws[1:]:
    c = g.StagedBuild(X, **kw)
    t_p1[W], _ = ev_time(lambda: c.phase1(0, (G + W - 1) // W))
    del c
    torch.cuda.empty_cache()
rounds = {W: 0.0 for W in Ws}
apply_s, sampled, t_search1 = 0.0, 0, 0.0
t0 = time.perf_counter()
for i in range(1, G):
    lo, hi = b.group_rows(i, i + 1)
    ts, f = ev_time(lambda: b.round_search(i, lo, hi))
    t_search1 += ts
    if i % a.every == 0:
        sampled += 1
        rounds[1] += ts
        for W in Ws[1:]:
            worst = 0.0
            for r in range(W):
                x0, x1 = lo + (hi - lo) * r // W, lo + (hi - lo) * (r + 1) // W
                tw, _ = ev_time(lambda: b.round_search(i, x0, x1))
                worst = max(worst, tw)
            rounds[W] += worst
    ta, _ = ev_time(lambda: b.round_apply(i, *f))
    apply_s += ta
gr = b.finish()
wall = time.perf_counter() - t0
nr = G - 1
row_bytes = a.n * (dx * 8 + dm * 8)
out = {"n": a.n, "d": cfg.d, "group_size": S, "groups": G, "rounds": nr,
       "l_build": a.l_build, "l_local": a.l_local, "sampled_rounds": sampled,
       "phase1_s": {str(W): round(t_p1[W], 4) for W in Ws},
       "phase2_search_s_1gpu": round(t_search1, 4), "phase2_apply_s": round(apply_s, 4),
       "round_search_ms_mean_sampled": {str(W): round(rounds[W] / max(1, sampled) * 1e3, 4)
                                        for W in Ws},
       "exchange_model": {"all_gather_latency_us": a.ag_latency_us, "GBps": a.ag_gbps}}
est = {}
for W in Ws:
    ex_rows = 0.0 if W == 1 else row_bytes * (W - 1) / W / (a.ag_gbps * 1e9) + a.ag_latency_us * 1e-6
    ex_rounds = 0.0 if W == 1 else nr * (a.ag_latency_us * 1e-6 + S * dm * 8 / (a.ag_gbps * 1e9))
    r_search = rounds[W] / max(1, sampled) * nr
    est[str(W)] = {"build_s": round(t_p1[W] + ex_rows + r_search + apply_s + ex_rounds, 4),
                   "phase1_s": round(t_p1[W], 4), "rows_exchange_s": round(ex_rows, 4),
                   "round_search_s": round(r_search, 4), "round_exchange_s": round(ex_rounds, 4),
                   "apply_s": round(apply_s, 4)}
out["estimated_build"] = est
out["speedup_vs_1"] = {w: round(est["1"]["build_s"] / e["build_s"], 3) for w, e in est.items()}
out["stats"] = list(gr.build_stats)
print(json.dumps(out), flush=True)
