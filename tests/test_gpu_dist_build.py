"""NEXT-2 on the GPU: the staged Algorithm-2 ABI (ganns_build_begin ... finish)
driven by dist.build_distributed.  One GPU carries several replicas: (a) one rank
== ganns_build == oracle.alg2; (b) two replicas in one process exchanging rows and
F blocks by hand; (c) two processes on cuda:0 over gloo (host staging of the
exchange).  All bit-exact against the oracle's Algorithm 2."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import ganns_synth as syn

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)
import paper_conf_icde_yuwzqzl22_b200 as g   # noqa: E402
from paper_conf_icde_yuwzqzl22_b200 import dist as gd   # noqa: E402

DEV = torch.device("cuda:0")
KW = dict(degree=16, l_build=32, l_local=16, group_size=250)


def _data(n=3000):
    return syn.points(syn.with_size(syn.CONFIGS["C1"], n=n))


def _ref(X):
    return oracle.alg2(X, 8, 16, 250, l_build=32, l_local=16)


def test_staged_one_rank_equals_build_and_oracle():
    X = _data()
    Xd = torch.from_numpy(X).to(DEV)
    gr = gd.build_distributed(g.StagedBuild(Xd, **KW))
    ref, _, st = _ref(X)
    assert (gr.adjacency() == ref).all()
    one = g.build(Xd, **KW)
    assert (one.adjacency() == ref).all()
    assert gr.build_stats[:3] == one.build_stats[:3] == tuple(int(x) for x in st)
    assert gr.build_stats[3] == one.build_stats[3] == 11


def test_staged_two_replicas_in_one_process():
    X = _data(2600)
    Xd = torch.from_numpy(X).to(DEV)
    A, B = g.StagedBuild(Xd, **KW), g.StagedBuild(Xd, **KW)
    S, G, dm, dx = A.info()
    h = G // 2
    A.phase1(0, h)
    B.phase1(h, G)
    ra, rb = A.export_rows(*A.group_rows(0, h)), B.export_rows(*B.group_rows(h, G))
    A.import_rows(*A.group_rows(h, G), rb)
    B.import_rows(*B.group_rows(0, h), ra)
    for i in range(1, G):
        lo, hi = A.group_rows(i, i + 1)
        mid = (lo + hi) // 2
        fa, fb = A.round_search(i, lo, mid), B.round_search(i, mid, hi)
        F = (torch.cat([fa[0], fb[0]]), torch.cat([fa[1], fb[1]]))
        A.round_apply(i, *F)
        B.round_apply(i, *F)
    ga, gb = A.finish(), B.finish()
    ref, _, st = oracle.alg2(X, 8, 16, 250, l_build=32, l_local=16)
    assert (ga.adjacency() == ref).all() and (gb.adjacency() == ref).all()
    assert ga.build_stats[2] + gb.build_stats[2] == int(st[2])   # searches split, not repeated


def test_staged_api_rejects_out_of_order_use():
    Xd = torch.from_numpy(_data(1200)).to(DEV)
    b = g.StagedBuild(Xd, **KW)
    with pytest.raises(g.GannsError):
        b.round_search(1, 250, 300)          # Phase 1 of groups 0..1 missing
    b.phase1(0, b.ngroups)
    with pytest.raises(g.GannsError):
        b.round_search(2, 500, 600)          # round 1 not applied
    with pytest.raises(g.GannsError):
        b.round_search(1, 100, 300)          # vertices outside P_1
    f = b.round_search(1, 250, 500)
    b.round_apply(1, *f)
    with pytest.raises(g.GannsError):
        b.phase1(0, 1)                       # Phase 1 after a round


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    X = _data()
    gr = gd.build_distributed(g.StagedBuild(torch.from_numpy(X).to(DEV), **KW))
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), adj=gr.adjacency(),
             searches=gr.build_stats[2])
    dist.destroy_process_group()


def test_staged_two_processes_gloo_on_one_gpu(tmp_path):
    mp.spawn(_worker, args=(2, _free_port(), str(tmp_path)), nprocs=2, join=True)
    ref, _, st = _ref(_data())
    res = [dict(np.load(os.path.join(tmp_path, f"r{r}.npz"))) for r in range(2)]
    for r in res:
        assert (r["adj"] == ref).all()
    assert sum(int(r["searches"]) for r in res) == int(st[2])
