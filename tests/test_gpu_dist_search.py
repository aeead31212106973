"""dist.py's GPU helpers under a real NCCL process group (world size 1 on the one
GPU this box has): gpu_replicated_search and gpu_sharded_index (two local shards,
two streams) against the oracle, bit-exact.  The multi-rank host logic is covered
by the gloo tests (test_dist_cpu.py)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

import oracle
import ganns_synth as syn

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)
import paper_conf_icde_yuwzqzl22_b200 as g   # noqa: E402
from paper_conf_icde_yuwzqzl22_b200 import dist as gd   # noqa: E402

DEV = torch.device("cuda:0")


@pytest.fixture(scope="module")
def nccl_world1():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=DEV)
    assert dist.get_backend() == "nccl"
    yield
    dist.destroy_process_group()


def test_gpu_replicated_search_nccl(nccl_world1):
    cfg = syn.with_size(syn.CONFIGS["C1"], n=4000, nq=300)
    X, Q = syn.points(cfg), syn.queries(cfg)
    nbr, _, _ = oracle.alg2(X, 8, 16, 256, l_build=32)
    graph = g.from_adjacency(nbr, X.shape[1])
    ids, dists = gd.gpu_replicated_search(graph, torch.from_numpy(X).to(DEV),
                                          torch.from_numpy(Q).to(DEV), 10, 48)
    oi, od = oracle.search(nbr, X, Q, 10, 48, threads=8)
    assert (ids.cpu().numpy() == oi).all() and (dists.cpu().numpy() == od).all()


def test_gpu_sharded_index_two_local_shards_nccl(nccl_world1):
    cfg = syn.with_size(syn.CONFIGS["C1"], n=5000, nq=200)
    X, Q = syn.points(cfg), syn.queries(cfg)
    h = len(X) // 2
    shards, parts = [], []
    for a, b in ((0, h), (h, len(X))):
        nb, _, _ = oracle.alg2(X[a:b], 8, 16, 256, l_build=32)
        shards.append((a, g.from_adjacency(nb, X.shape[1]), torch.from_numpy(X[a:b]).to(DEV)))
        i, d = oracle.search(nb, X[a:b], Q, 10, 40, threads=8)
        parts.append((np.where(i >= 0, i + a, -1), d))
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    idx = gd.gpu_sharded_index(shards, 10, 40, streams=streams)
    ids, dists = idx.search(torch.from_numpy(Q).to(DEV))
    ri, rd = oracle.merge_topk(np.stack([p[0] for p in parts]), np.stack([p[1] for p in parts]))
    assert (ids.cpu().numpy() == ri).all() and (dists.cpu().numpy() == rd).all()
