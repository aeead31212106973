"""C2 build time vs group size (R-C14) at the bench's l_build 128 / l_local 32: GPU-clock
Phase 1 / Phase 2 (staged API, events) and wall time; median of 3 per size."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402

cfg = syn.CONFIGS["C2"]
X = torch.from_numpy(syn.points(cfg)).cuda()
a = torch.randn(8192, 8192, device="cuda")
for _ in range(20):
    a @ a
g.build(X, degree=32, l_build=128, l_local=32)
for s in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "1024,1280,1536,1792,2048,2560").split(",")]:
    walls = []
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        gr = g.build(X, degree=32, l_build=128, l_local=32, group_size=s)
        torch.cuda.synchronize()
        walls.append(time.perf_counter() - t0)
    print(json.dumps({"group": s, "build_s": round(statistics.median(walls), 4),
                      "all": [round(w, 4) for w in walls], "rounds": gr.build_stats[3]}), flush=True)
