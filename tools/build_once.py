"""One C2 build (for ncu launch lists of the build kernels)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
X = torch.from_numpy(syn.points(syn.CONFIGS["C2"])).cuda()
gr = g.build(X, degree=32, l_build=128)
torch.cuda.synchronize()
print("done", gr.build_stats)
