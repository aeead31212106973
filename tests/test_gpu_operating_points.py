"""Parity at the exact kernel instances and operating points bench.py measures
(VERDICT r1 "prove parity at the exact points the bench measures").

* C4: d = 200, HNSW with the greedy descent fused into K1 (search_kernel
  <NV4=2, TPL=1, L2=false, HNSW=true>), l = 288, on a 100K-point HNSW -- integer
  inner products (bit-exact: ids, dists, counters, entries) and the cosine data
  of the bench (tolerance).
* C3: d = 960, the warp-group kernel (search_group_kernel) at l = 320.
* C2: the full 1M-point build with the bench's parameters (l_build 128,
  l_local 32, auto group size 1536) bit-exact against the oracle's Algorithm 2
  (all host cores; the arithmetic is the sequential one), then the search at
  the bench's operating point (l 128, e 109) on that graph.

Cosine tolerance: |d_gpu - d_oracle| <= 1e-5 |d| + 1e-6.  The
north star's 1e-5 relative bar applies to the dot product; the distance
1 - <q, x>/||q|| is near 0 for the nearest neighbours, where the subtraction
cancels: an fp32 error of a few ulp(1.0) = 1.19e-7 in <q, x>/||q|| becomes an
absolute error of the same size in the distance.  1e-6 = 8 ulp(1.0).
"""
import numpy as np
import pytest
import torch

import oracle
import ganns_synth as syn

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)
import paper_conf_icde_yuwzqzl22_b200 as g   # noqa: E402

DEV = torch.device("cuda:0")
COS_RTOL, COS_ATOL = 1e-5, 1e-6


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def oracle_index(idx):
    """The GPU-built HNSW's layers in the oracle's format (the oracle searches the
    same graph; the build itself is checked bit-exact in test_gpu_hnsw.py)."""
    ups = {j: idx.layer(j) for j in range(1, idx.nlayers)}
    flat = np.concatenate([ups[j].reshape(-1) for j in range(1, idx.nlayers)]) if ups \
        else np.zeros(1, np.int32)
    return dict(perm=idx.perm(), layer_n=np.array(idx.layer_n, np.int64), upper=ups,
                layer0=idx.layer(0), upper_flat=flat)


def _c4_like(n, metric):
    cfg = syn.with_size(syn.CONFIGS["C4"], n=n)
    X = syn.points(cfg)
    Q = syn.queries(cfg, 2000)
    if metric == "cosine":
        X = syn.normalize_rows(X)
    return cfg, X, Q


def test_c4_instance_hnsw_fused_l288_integer_ip_bitexact():
    """Same kernel instance as the C4 bench line (d = 200, IP family, fused
    descent), integer inner products: everything bit-exact."""
    cfg, X, Q = _c4_like(100_000, "ip")
    Xd = cu(X)
    levels = syn.hnsw_levels(len(X), cfg.degree // 2, 1)
    idx = g.build_hnsw(Xd, levels, metric="ip", degree=cfg.degree, l_build=128, l_local=32)
    assert idx.nlayers >= 3
    ids, dists, st, ds = g.hnsw_search(idx, Xd, cu(Q), cfg.k, 288, stats=True,
                                       descent_stats=True)   # one launch
    torch.cuda.synchronize()
    ids, dists, st, ds = ids.cpu().numpy(), dists.cpu().numpy(), st.cpu().numpy(), ds.cpu().numpy()
    h = oracle_index(idx)
    sample = np.arange(0, len(Q), 25)
    oi, od, _, ost, ods = oracle.hnsw_search(h, X, Q[sample], cfg.k, 288, metric="ip", stats=True,
                                             descent_stats=True)
    assert (ds[sample] == ods).all()          # the descent's counters (bench bytes)
    assert (ids[sample] == oi).all()
    assert (dists[sample] == od).all()
    assert (st[sample][:, 0] == ost[:, 0]).all() and (st[sample][:, 1] == ost[:, 1]).all()
    assert (st[sample][:, 2] == ost[:, 3]).all()


def test_c4_instance_hnsw_fused_l288_cosine():
    """The bench's C4 data (unit rows, cosine) on the same instance: distances
    within the cosine tolerance, id sets >= 99.8 % equal, recall within 0.002."""
    cfg, X, Q = _c4_like(100_000, "cosine")
    Xd = cu(X)
    levels = syn.hnsw_levels(len(X), cfg.degree // 2, 1)
    idx = g.build_hnsw(Xd, levels, metric="cosine", degree=cfg.degree, l_build=128, l_local=32)
    ids, dists = g.hnsw_search(idx, Xd, cu(Q), cfg.k, 288)
    ids, dists = ids.cpu().numpy(), dists.cpu().numpy()
    h = oracle_index(idx)
    sample = np.arange(0, len(Q), 10)
    oi, od, _ = oracle.hnsw_search(h, X, Q[sample], cfg.k, 288, metric="cosine")
    np.testing.assert_allclose(dists[sample], od, rtol=COS_RTOL, atol=COS_ATOL)
    agree = np.mean([len(set(a) & set(b)) / cfg.k for a, b in zip(ids[sample], oi)])
    assert agree >= 0.998, agree
    gt, _ = oracle.bruteforce(X, Q[sample], cfg.k, metric="cosine")
    assert abs(oracle.recall(ids[sample], gt) - oracle.recall(oi, gt)) <= 0.002


def test_c3_group_kernel_l320_fullsize_sampled():
    """BASELINE configs[2] (1M x 960) in the bench's launch shape (all 1K queries in
    one launch, warp group per query) at the bench's l = 320."""
    cfg = syn.CONFIGS["C3"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    nbr = syn.random_graph(cfg.n, cfg.degree, seed=33, min_degree=cfg.degree // 2)
    graph = g.from_adjacency(nbr, cfg.d)
    ids, dists, st = g.search(graph, cu(X), cu(Q), cfg.k, 320, stats=True)
    ids, dists, st = ids.cpu().numpy(), dists.cpu().numpy(), st.cpu().numpy()
    sample = np.arange(0, cfg.nq, cfg.nq // 12)
    oi, od, ost = oracle.search(nbr, X, Q[sample], cfg.k, 320, threads=16, stats=True)
    assert (ids[sample] == oi).all() and (dists[sample] == od).all()
    assert (st[sample][:, 0] == ost[:, 0]).all() and (st[sample][:, 1] == ost[:, 1]).all()
    assert (st[sample][:, 2] == ost[:, 3]).all()


@pytest.mark.slow
def test_c2_fullsize_build_bitexact_and_operating_point():
    """BASELINE configs[1]: the bench's build (1M x 128, degree 32, l_build 128,
    l_local 32, auto group size = 1536, 651 Phase-2 rounds) == the oracle's
    Algorithm 2, adjacency and build counters; then the bench's operating point
    (l 128, e 109) searched on it in one launch, sampled queries bit-exact."""
    cfg = syn.CONFIGS["C2"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    Xd = cu(X)
    graph = g.build(Xd, degree=cfg.degree, l_build=128, l_local=32)
    adj = graph.adjacency()
    ref, _, st = oracle.alg2(X, cfg.degree // 2, cfg.degree, 1536, l_build=128, l_local=32,
                             threads=oracle.ncores())
    bad = np.argwhere((adj != ref).any(1)).ravel()
    assert len(bad) == 0, f"{len(bad)} rows differ, first {bad[:5]}"
    assert tuple(graph.build_stats[:3]) == tuple(int(x) for x in st)
    assert graph.build_stats[3] == (cfg.n + 1535) // 1536 - 1
    ids, dists, gst = g.search(graph, Xd, cu(Q), cfg.k, 128, e=109, stats=True)
    ids, dists, gst = ids.cpu().numpy(), dists.cpu().numpy(), gst.cpu().numpy()
    sample = np.arange(0, cfg.nq, 50)
    oi, od, ost = oracle.search(ref, X, Q[sample], cfg.k, 128, e=109, threads=oracle.ncores(),
                                stats=True)
    assert (ids[sample] == oi).all() and (dists[sample] == od).all()
    assert (gst[sample][:, :2] == ost[:, :2]).all() and (gst[sample][:, 2] == ost[:, 3]).all()
