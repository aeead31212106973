"""Build-time breakdown on a config: Phase 1 alone, then full builds over group sizes."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
lb = int(sys.argv[2]) if len(sys.argv) > 2 else 128
groups = [int(x) for x in (sys.argv[3] if len(sys.argv) > 3 else "1024,2048,4096").split(",")]
X = torch.from_numpy(syn.points(cfg)).cuda()
g.build(X[:20000].contiguous(), degree=cfg.degree, l_build=lb)   # warm-up (module load)
for s in groups:
    torch.cuda.synchronize()
    t0 = time.time()
    g.build(X, degree=cfg.degree, l_build=lb, group_size=s, stop_after_phase1=True)
    torch.cuda.synchronize()
    t1 = time.time() - t0
    t0 = time.time()
    gr = g.build(X, degree=cfg.degree, l_build=lb, group_size=s)
    torch.cuda.synchronize()
    t2 = time.time() - t0
    print(json.dumps({"group": s, "phase1_s": round(t1, 3), "total_s": round(t2, 3),
                      "phase2_s": round(t2 - t1, 3), "stats": gr.build_stats}), flush=True)
