"""Per-round tail of the Phase-2 searches (GANNS_PROFILE build): for every round of a
C2 build, the round-search kernel's time (CUDA events), the mean and the largest
loop cycles / iterations of its searches -- how far the round (= its slowest search)
is above the mean search.
    GANNS_LIB_PATH=ab/libganns_prof.so python tools/round_tail.py [--every 10]"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--every", type=int, default=1)
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]
X = torch.from_numpy(syn.points(cfg)).cuda()
b = g.StagedBuild(X, metric=cfg.metric, degree=cfg.degree, l_build=128, l_local=32)
S, G, dm, dx = b.info()
b.phase1(0, G)
g.profile_read(reset=True)
rows = []
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for i in range(1, G):
    lo, hi = b.group_rows(i, i + 1)
    ev0.record()
    f = b.round_search(i, lo, hi)
    ev1.record()
    p = g.profile_read(reset=True)
    if i % a.every == 0:
        tot = sum(p[k] for k in g.PROFILE_PHASES)
        rows.append({"round": i, "kernel_ms": ev0.elapsed_time(ev1), "searches": p["searches"],
                     "mean_cycles": tot / p["searches"], "max_cycles": p["max_search_cycles"],
                     "mean_iters": p["iterations"] / p["searches"],
                     "max_iters": p["max_search_iterations"]})
    b.round_apply(i, *f)
b.finish()
for r in rows[:: max(1, len(rows) // 12)]:
    print(json.dumps({k: round(v, 3) if isinstance(v, float) else v for k, v in r.items()}))
summ = {
    "rounds": len(rows),
    "kernel_ms_mean": statistics.mean(r["kernel_ms"] for r in rows),
    "max_over_mean_cycles": statistics.mean(r["max_cycles"] / r["mean_cycles"] for r in rows),
    "max_over_mean_iters": statistics.mean(r["max_iters"] / r["mean_iters"] for r in rows),
    "mean_iters": statistics.mean(r["mean_iters"] for r in rows),
    "max_iters_mean": statistics.mean(r["max_iters"] for r in rows),
    "kernel_cycles_over_max_search": statistics.mean(r["kernel_ms"] * 1.965e6 / r["max_cycles"] for r in rows),
}
print(json.dumps({k: round(v, 3) if isinstance(v, float) else v for k, v in summ.items()}))
