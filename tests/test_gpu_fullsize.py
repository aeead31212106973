"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(one ganns_search launch over the whole query batch), checked on sampled outputs
the oracle computes one by one, plus properties that hold at any size.

Search: the graph is a seeded random fixed-degree graph (ganns_synth) -- an
input, so the oracle and the kernel see the same adjacency without the oracle
depending on the CUDA build.  Build: Phase 1 of Algorithm 2 is per-group
independent, so sampled groups of the full-size build are checked against the
oracle's sequential insertion of that group alone; the complete graph is checked
for the invariants (P7) and for recall against brute force.
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


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


@pytest.fixture(scope="module")
def c2():
    cfg = syn.CONFIGS["C2"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    return cfg, X, Q, cu(X), cu(Q)


def _sampled_search_parity(cfg, X, Q, Xd, Qd, nbr, l, sample, metric="l2", exact=True):
    graph = g.from_adjacency(nbr, X.shape[1], metric)
    ids, dists, st = g.search(graph, Xd, Qd, cfg.k, l, stats=True)   # the whole batch
    torch.cuda.synchronize()
    ids, dists, st = ids.cpu().numpy(), dists.cpu().numpy(), st.cpu().numpy()
    oi, od, os_ = oracle.search(nbr, X, Q[sample], cfg.k, l, metric=metric, threads=16, stats=True)
    if exact:
        assert (ids[sample] == oi).all()
        assert (dists[sample] == od).all()
        assert (st[sample][:, 0] == os_[:, 0]).all() and (st[sample][:, 1] == os_[:, 1]).all()
        assert (st[sample][:, 2] == os_[:, 3]).all()
    else:
        np.testing.assert_allclose(dists[sample], od, rtol=1e-5, atol=1e-6)
    # properties of every output row: ascending (dist, id), no repeats, distances true
    for q in range(0, len(Q), max(1, len(Q) // 200)):
        row = ids[q][ids[q] >= 0]
        assert len(set(row.tolist())) == len(row)
        assert all((dists[q][i], row[i]) <= (dists[q][i + 1], row[i + 1]) for i in range(len(row) - 1))
        d0 = oracle.distance(Q[q], X[row[0]], metric)
        assert abs(d0 - dists[q][0]) <= (0 if exact else 1e-5 * max(1.0, abs(d0)))
    return ids, dists


def test_c2_search_fullsize_sampled(c2):
    """BASELINE configs[1]: 1M x 128, degree 32, 10K queries in one launch, l = 128."""
    cfg, X, Q, Xd, Qd = c2
    nbr = syn.random_graph(cfg.n, cfg.degree, seed=2, min_degree=cfg.degree // 2)
    rng = np.random.default_rng(0)
    sample = np.sort(rng.choice(len(Q), 48, replace=False))
    _sampled_search_parity(cfg, X, Q, Xd, Qd, nbr, 128, sample)
    _sampled_search_parity(cfg, X, Q, Xd, Qd, nbr, 512, sample[:16])


def test_c2_build_phase1_sampled_groups(c2):
    """Phase 1 of the full-size build (auto group size) == the oracle's sequential
    NSW insertion of each sampled group on its own (Alg. 2 lines 2-8)."""
    cfg, X, Q, Xd, Qd = c2
    graph = g.build(Xd, degree=cfg.degree, l_build=64, stop_after_phase1=True)
    adj = graph.adjacency()
    S = 1536   # R-C14 auto for n = 1M: clamp(round256(1.5 sqrt(n)), 256, 8192)
    ngroups = (cfg.n + S - 1) // S
    for gi in (0, 1, ngroups // 2, ngroups - 1):
        lo, hi = gi * S, min(cfg.n, (gi + 1) * S)
        ref, _, _ = oracle.nsw_seq(X[lo:hi], cfg.degree // 2, cfg.degree, l_build=64)
        ref = np.where(ref >= 0, ref + lo, -1)
        assert (adj[lo:hi] == ref).all(), gi


def test_c2_build_full_invariants_and_recall(c2):
    cfg, X, Q, Xd, Qd = c2
    graph = g.build(Xd, degree=cfg.degree, l_build=128)
    adj = graph.adjacency()
    assert adj.shape == (cfg.n, cfg.degree)
    rng = np.random.default_rng(1)
    for v in rng.choice(cfg.n, 300, replace=False):
        row = adj[v]
        c = int((row >= 0).sum())
        assert (row[:c] >= 0).all() and (row[c:] == -1).all()       # -1 suffix
        assert c >= 1 and v not in row[:c] and len(set(row[:c].tolist())) == c
        keys = [(oracle.distance(X[v], X[u]), u) for u in row[:c]]
        assert keys == sorted(keys)                                 # sorted by (dist, id)
    # forward edges: v's d_min nearest among earlier points are approximated; the
    # build must give high recall on the bench's own metric
    ids, _ = g.search(graph, Xd, Qd[:200], cfg.k, 128)
    gt, _ = oracle.bruteforce(X, Q[:200], cfg.k)
    assert oracle.recall(ids.cpu().numpy(), gt) >= 0.93
    assert graph.build_stats[3] == (cfg.n + 1535) // 1536 - 1       # Phase-2 rounds (auto s = 1536)


def test_c4_cosine_fullsize_sampled():
    """BASELINE configs[3]: 1.18M x 200 cosine (unit rows), degree 32."""
    cfg = syn.CONFIGS["C4"]
    X = syn.normalize_rows(syn.points(cfg))
    Q = syn.queries(cfg)
    nbr = syn.random_graph(cfg.n, cfg.degree, seed=4, min_degree=cfg.degree // 2)
    sample = np.arange(0, cfg.nq, cfg.nq // 24)
    ids, _ = _sampled_search_parity(cfg, X, Q, cu(X), cu(Q), nbr, 128, sample,
                                    metric="cosine", exact=False)
    oi, _ = oracle.search(nbr, X, Q[sample], cfg.k, 128, metric="cosine", threads=16)
    agree = np.mean([len(set(a) & set(b)) / cfg.k for a, b in zip(ids[sample], oi)])
    assert agree >= 0.998


def test_c3_gist_fullsize_sampled():
    """BASELINE configs[2]: 1M x 960 (3.84 GB of vectors), degree 32, 1K queries."""
    cfg = syn.CONFIGS["C3"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    nbr = syn.random_graph(cfg.n, cfg.degree, seed=3, min_degree=cfg.degree // 2)
    sample = np.arange(0, cfg.nq, cfg.nq // 16)
    _sampled_search_parity(cfg, X, Q, cu(X), cu(Q), nbr, 64, sample)


def test_c5_shard_slice_sampled():
    """BASELINE configs[4] per-shard shape: a 1M-row slice of shard 3 of the 100M x 96
    set (ids offset to global), 10K queries, sharded top-k merge against the oracle."""
    cfg = syn.CONFIGS["C5"]
    lo = 3 * (cfg.n // cfg.shards)
    X = syn.points(cfg, lo, lo + 1_000_000)
    Q = syn.queries(cfg)
    nbr = syn.random_graph(len(X), cfg.degree, seed=5, min_degree=cfg.degree // 2)
    sub = syn.with_size(cfg, n=len(X))
    sample = np.arange(0, cfg.nq, cfg.nq // 24)
    ids, dists = _sampled_search_parity(sub, X, Q, cu(X), cu(Q), nbr, 64, sample)
    # merge two "shards" (the slice's two halves searched as separate graphs)
    half = len(X) // 2
    parts = []
    for a, b in ((0, half), (half, len(X))):
        nb = syn.random_graph(b - a, cfg.degree, seed=50 + a, min_degree=cfg.degree // 2)
        gr = g.from_adjacency(nb, X.shape[1])
        i, d = g.search(gr, cu(X[a:b]), cu(Q), cfg.k, 64)
        g.offset_ids(i, lo + a)
        oi, od = oracle.search(nb, X[a:b], Q[sample], cfg.k, 64, threads=16)
        assert (i.cpu().numpy()[sample] == np.where(oi >= 0, oi + lo + a, -1)).all()
        parts.append((i, d, np.where(oi >= 0, oi + lo + a, -1), od))
    mi, md = g.merge_topk(torch.stack([parts[0][0], parts[1][0]]),
                          torch.stack([parts[0][1], parts[1][1]]))
    ri, rd = oracle.merge_topk(np.stack([parts[0][2], parts[1][2]]),
                               np.stack([parts[0][3], parts[1][3]]))
    assert (mi.cpu().numpy()[sample] == ri).all() and (md.cpu().numpy()[sample] == rd).all()
