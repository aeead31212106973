"""Build time over group sizes for the configs whose Phase-2 rounds exceed one wave
of resident searches at the auto group size (C3: 3.84-KB rows, C4: 800-B rows, HNSW):
wall time of each build (after a warm-up), 2 reps per size (0 = auto rule).
    python tools/group_wave_sweep.py C4 0,1024,1280"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1]]
sizes = [int(x) for x in sys.argv[2].split(",")]
X = torch.from_numpy(syn.points(cfg)).cuda()
hnsw = cfg.name == "C4"
levels = syn.hnsw_levels(X.shape[0], cfg.degree // 2, 1) if hnsw else None


def build(Xs, lv, s):
    if hnsw:
        return g.build_hnsw(Xs, lv, metric=cfg.metric, degree=cfg.degree, l_build=128, group_size=s)
    return g.build(Xs, metric=cfg.metric, degree=cfg.degree, l_build=128, l_local=32, group_size=s)


build(X[:50000].contiguous(), levels[:50000] if hnsw else None, 0)
for s in sizes:
    ts = []
    for _ in range(2):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        h = build(X, levels, s)
        torch.cuda.synchronize()
        ts.append(round(time.perf_counter() - t0, 3))
        del h
    print(cfg.name, "group_size", s, "build_s", ts, flush=True)
