"""C4 HNSW probe: time hnsw_search vs a plain search of its layer 0 from vertex 0."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex  # noqa: E402
cfg = syn.CONFIGS["C4"]
X = torch.from_numpy(syn.normalize_rows(syn.points(cfg))).cuda()
Q = torch.from_numpy(syn.queries(cfg)).cuda()
idx = BenchIndex(g, cfg, X, 128)
def t(fn, reps=5):
    ts = []
    for _ in range(reps):
        torch.cuda.synchronize(); e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record(); fn(); e1.record(); e1.synchronize(); ts.append(e0.elapsed_time(e1))
    return sorted(ts)[len(ts) // 2]
l = int(sys.argv[1]) if len(sys.argv) > 1 else 320
_, _, st = g.hnsw_search(idx.idx, X, Q, 10, l, stats=True)
_, _, st0 = g.search(idx.graph, X, Q, 10, l, stats=True)
print(json.dumps({"hnsw_ms": t(lambda: g.hnsw_search(idx.idx, X, Q, 10, l)),
                  "layer0_ms": t(lambda: g.search(idx.graph, X, Q, 10, l)),
                  "hnsw_iters": float(st[:, 0].float().mean()), "layer0_iters": float(st0[:, 0].float().mean()),
                  "hnsw_comps": float(st[:, 1].float().mean()), "layer0_comps": float(st0[:, 1].float().mean()),
                  "layers": idx.idx.nlayers}))
# layer 0 in the shuffled (level-sorted) id space with permuted rows: hubs contiguous
import numpy as np  # noqa: E402
perm = idx.idx.perm()                      # perm[new] = old
inv = np.empty_like(perm); inv[perm] = np.arange(len(perm), dtype=np.int32)
base = idx.idx.layer(0)                    # original ids
nb = base[perm]                            # row of new id i = row of old perm[i]
nb = np.where(nb >= 0, inv[np.maximum(nb, 0)], -1).astype(np.int32)
gs = g.from_adjacency(nb, cfg.d, "cosine")
Xp = X[torch.from_numpy(perm.astype(np.int64)).cuda()].contiguous()
e0 = int(inv[0])
_, _, st2 = g.search(gs, Xp, Q, 10, l, entry=e0, stats=True)
print(json.dumps({"shuffled_space_ms": t(lambda: g.search(gs, Xp, Q, 10, l, entry=e0)),
                  "shuffled_iters": float(st2[:, 0].float().mean()),
                  "shuffled_entry0_ms": t(lambda: g.search(gs, Xp, Q, 10, l, entry=0))}))
# NSW over the same points for reference (id-order insertion)
gn = g.build(X, metric="cosine", degree=cfg.degree, l_build=128)
_, _, st3 = g.search(gn, X, Q, 10, l, stats=True)
print(json.dumps({"nsw_ms": t(lambda: g.search(gn, X, Q, 10, l)), "nsw_iters": float(st3[:, 0].float().mean())}))
# host-side enqueue cost of one call (no sync inside the API expected)
for name, fn in (("hnsw", lambda: g.hnsw_search(idx.idx, X, Q, 10, l)),
                 ("nsw", lambda: g.search(gn, X, Q, 10, l))):
    fn(); torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(5):
        fn()
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    print(json.dumps({name: {"enqueue_ms_per_call": round((t1 - t0) / 5 * 1e3, 3),
                             "total_ms_per_call": round((t2 - t0) / 5 * 1e3, 3)}}))
