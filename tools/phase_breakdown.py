"""Per-phase time breakdown of the GANNS search loop (the analogue of the paper's
Fig. 7 / Fig. 10: "data structure operations" vs "distance
computation"), from a GANNS_PROFILE library build (GANNS_LIB_PATH=ab/libganns_prof.so):
the bench's search at its operating point, and the two build phases.
    GANNS_LIB_PATH=ab/libganns_prof.so python tools/phase_breakdown.py --config C2 --l 128 --e 109"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, make_workload  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--l", type=int, required=True)
ap.add_argument("--e", type=int, default=0)
a = ap.parse_args()
cfg = syn.CONFIGS[a.config]


def shares(p):
    tot = sum(p[k] for k in g.PROFILE_PHASES)
    out = {k: round(p[k] / tot, 4) for k in g.PROFILE_PHASES}
    out["data_structure_ops"] = round(1 - out["distance"] - out["explore"], 4)
    out["cycles_per_iteration"] = round(tot / max(1, p["iterations"]), 1)
    out["iterations_per_search"] = round(p["iterations"] / max(1, p["searches"]), 2)
    if p.get("gather_rounds") and p.get("spec_build"):
        out["spec_fill_cycles_per_iteration"] = round(p["gather_issue"] / max(1, p["iterations"]), 1)
        out["spec_math_cycles_per_iteration"] = round(p["gather_wait"] / max(1, p["iterations"]), 1)
        out["spec_gathered_ahead_rate"] = round(p["gather_rounds"] / max(1, p["iterations"]), 4)
    elif p.get("gather_rounds"):
        r = p["gather_rounds"]
        out["gather_issue_cycles_per_round"] = round(p["gather_issue"] / r, 1)
        out["gather_wait_cycles_per_round"] = round(p["gather_wait"] / r, 1)
        out["gather_rounds_per_iteration"] = round(r / max(1, p["iterations"]), 3)
        out["spec_hit_rate"] = round(p["spec_hits"] / max(1, p["iterations"]), 4)
    return out


X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
res = {"config": a.config, "note": "lane 0 clock64 at phase boundaries; the explore phase "
       "ends when the adjacency row is in registers"}
if cfg.name != "C4":
    g.profile_read(reset=True)
    b = g.StagedBuild(Xd, metric=cfg.metric, degree=cfg.degree, l_build=128, l_local=32)
    S, G, dm, dx = b.info()
    b.phase1(0, G)
    res["build_phase1"] = shares(dict(g.profile_read(reset=True), spec_build=True))
    for i in range(1, G):
        lo, hi = b.group_rows(i, i + 1)
        b.round_apply(i, *b.round_search(i, lo, hi))
    res["build_phase2"] = shares(dict(g.profile_read(reset=True), spec_build=True))
    gr = b.finish()
idx = BenchIndex(g, cfg, Xd, 128, 32)
g.profile_read(reset=True)
Qd = torch.from_numpy(np.concatenate(Qs)).cuda()
idx.search(Qd, cfg.k, a.l, e=a.e or a.l)
res["search"] = shares(g.profile_read(reset=True))
res["search"]["l"], res["search"]["e"] = a.l, a.e or a.l
print(json.dumps(res), flush=True)
