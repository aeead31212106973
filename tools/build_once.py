"""C2 builds with the bench's parameters (l_build 128, l_local 32, auto group size),
after a warm-up (GEMMs to bring the GPU out of idle clocks + one 20K-point build);
prints each build's wall time -- for A/B runs (GANNS_LIB_PATH selects the library)
and for ncu launch lists / captures of the build kernels.
    python tools/build_once.py [config] [reps]"""
import os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
cfg = syn.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C2"]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 1
X = torch.from_numpy(syn.points(cfg)).cuda()
a = torch.randn(8192, 8192, device="cuda")
for _ in range(20):
    a @ a
g.build(X[:20000].contiguous(), degree=cfg.degree, l_build=128, l_local=32)
ts = []
for _ in range(reps):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gr = g.build(X, degree=cfg.degree, l_build=128, l_local=32)
    torch.cuda.synchronize()
    ts.append(time.perf_counter() - t0)
    print("build_s", round(ts[-1], 4), gr.build_stats, flush=True)
print("median", round(statistics.median(ts), 4), "lib", g.LIB_PATH, flush=True)
