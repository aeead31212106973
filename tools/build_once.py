"""One C2 build with the bench's parameters (l_build 128, l_local 32, auto group size),
after an untimed warm-up build -- for ncu launch lists / captures of the build kernels."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
X = torch.from_numpy(syn.points(cfg)).cuda()
g.build(X[:20000].contiguous(), degree=cfg.degree, l_build=128, l_local=32)
for _ in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gr = g.build(X, degree=cfg.degree, l_build=128, l_local=32)
    torch.cuda.synchronize()
    print("build_s", round(time.perf_counter() - t0, 4), gr.build_stats, flush=True)
