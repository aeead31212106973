"""GGraphCon build on the GPU (ganns_build through the C ABI) vs the oracle's
Algorithm 2 with the same partition and search parameters: the adjacency must be
bit-identical on integer-grid data."""
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


def gpu_build(X, degree, **kw):
    graph = g.build(cu(X), degree=degree, **kw)
    torch.cuda.synchronize()
    return graph, graph.adjacency()


def test_build_theorem_regime_equals_sequential_nsw():
    """d_max >= n-1 and l_build >= n: every build search is exact, so by the
    quality theorem the GPU graph equals the sequential NSW graph for
    every group size."""
    for seed in range(4):
        n = 40 + 7 * seed                      # <= 61, so degree 64 >= n - 1
        X = syn.random_int_points(n, 8, 0, 6, 900 + seed)
        ref, _, _ = oracle.nsw_seq(X, 4, 64, exact=True)
        for s in (1, 5, 16, n):
            _, adj = gpu_build(X, 64, d_min=4, l_build=n + 1, group_size=s)
            assert (adj == ref).all(), (seed, s)


@pytest.mark.parametrize("n,degree,l_build,s,metric", [
    (2000, 16, 32, 256, "l2"),
    (3000, 32, 64, 300, "l2"),
    (1500, 64, 96, 128, "l2"),
    (2000, 16, 32, 100, "ip"),
    (4000, 32, 64, 4000, "l2"),      # one group: Phase 1 only = sequential NSW
    (1200, 128, 128, 200, "l2"),
])
def test_build_parity_alg2(n, degree, l_build, s, metric):
    cfg = syn.with_size(syn.CONFIGS["C1"], n=n)
    X = syn.points(cfg)
    if metric == "ip":
        X = X - 128.0   # signed integer grid: exact inner products
    ref, _, st = oracle.alg2(X, degree // 2, degree, s, l_build=l_build, metric=metric)
    graph, adj = gpu_build(X, degree, l_build=l_build, group_size=s, metric=metric)
    assert (adj == ref).all(), np.argwhere(adj != ref)[:5]
    it, comps, searches, rounds = graph.build_stats
    assert (it, comps, searches) == tuple(int(x) for x in st)
    assert rounds == (n + s - 1) // s - 1


def test_build_phase1_and_rounds_hooks():
    cfg = syn.with_size(syn.CONFIGS["C1"], n=2500)
    X = syn.points(cfg)
    ref0, _, _ = oracle.alg2(X, 8, 16, 250, l_build=32, max_rounds=0)
    _, adj0 = gpu_build(X, 16, l_build=32, group_size=250, stop_after_phase1=True)
    assert (adj0 == ref0).all()
    ref3, _, _ = oracle.alg2(X, 8, 16, 250, l_build=32, max_rounds=3)
    _, adj3 = gpu_build(X, 16, l_build=32, group_size=250, max_rounds=3)
    assert (adj3 == ref3).all()


def test_build_deterministic():
    X = syn.points(syn.with_size(syn.CONFIGS["C1"], n=5000))
    _, a = gpu_build(X, 16, l_build=32, group_size=200)
    _, b = gpu_build(X, 16, l_build=32, group_size=200)
    assert (a == b).all()


def test_build_c1_parity_and_quality():
    """BASELINE configs[0]: 10K x 128, degree 16; graph bit-exact vs the oracle's
    Algorithm 2, then search parity and recall on the built graph."""
    cfg = syn.CONFIGS["C1"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    ref, _, _ = oracle.alg2(X, 8, 16, 256, l_build=64)
    graph, adj = gpu_build(X, 16, l_build=64, group_size=256)
    assert (adj == ref).all()
    ids, dists = g.search(graph, cu(X), cu(Q), 10, 64)
    oi, od = oracle.search(ref, X, Q, 10, 64, threads=8)
    assert (ids.cpu().numpy() == oi).all() and (dists.cpu().numpy() == od).all()
    gt, _ = oracle.bruteforce(X, Q, 10)
    assert oracle.recall(oi, gt) > 0.8


@pytest.mark.parametrize("l_local", [16, 40])
def test_build_parity_l_local(l_local):
    """Phase-1 searches at l_local < l_build (R-C13): bit-exact vs the oracle."""
    cfg = syn.with_size(syn.CONFIGS["C1"], n=4000)
    X = syn.points(cfg)
    ref, _, _ = oracle.alg2(X, 8, 16, 256, l_build=64, l_local=l_local)
    _, adj = gpu_build(X, 16, l_build=64, group_size=256, l_local=l_local)
    assert (adj == ref).all()


@pytest.mark.parametrize("d,metric,s", [(384, "l2", 300), (960, "l2", 256), (960, "ip", 500)])
def test_build_parity_wide_rows_group(d, metric, s):
    """d > 256: the build searches run on a warp group (warp 0 the GANNS loop, all
    four warps the column slices of the bulk distance, search_group.cuh) -- Phase 1
    and Phase 2 equal the oracle's Algorithm 2 (adjacency and counters)."""
    cfg = syn.with_size(syn.CONFIGS["C3"], n=2500)
    X = np.ascontiguousarray(syn.points(cfg)[:, :d])
    if metric == "ip":
        X = X - 8.0   # signed integer grid: exact inner products
    ref, _, st = oracle.alg2(X, 16, 32, s, l_build=64, l_local=32, metric=metric)
    graph, adj = gpu_build(X, 32, l_build=64, l_local=32, group_size=s, metric=metric)
    assert (adj == ref).all(), np.argwhere(adj != ref)[:5]
    assert tuple(graph.build_stats[:3]) == tuple(int(x) for x in st)


@pytest.mark.parametrize("n,d,degree,l_build,l_local,s,metric", [
    (1800, 24, 16, 48, 16, 200, "l2"),     # d4 = 6: masked tail chunks (S = 8)
    (1800, 100, 32, 64, 32, 300, "l2"),    # d4 = 25
    (1500, 200, 32, 96, 32, 256, "ip"),    # d4 = 50 (S = 16, masked), C4's row width
    (1500, 256, 32, 64, 24, 250, "l2"),    # d4 = 64 (S = 16, full)
    (1200, 128, 24, 40, 40, 128, "l2"),    # d_max 24 < 32: partial adjacency rows
    (1600, 128, 32, 128, 32, 1600, "l2"),  # one group: Phase 1 only
    (2000, 128, 32, 32, 16, 64, "l2"),     # many small rounds
])
def test_build_parity_cpasync_speculation_shapes(n, d, degree, l_build, l_local, s, metric):
    """The build searches' cp.async four-row fill (full and masked rows), the
    speculative gather of the next candidate, and programmatic dependent launch
    across many rounds: adjacency and counters equal the oracle's Algorithm 2."""
    rng = np.random.default_rng(n + d)
    X = rng.integers(0, 16, size=(n, d)).astype(np.float32)
    if metric == "ip":
        X = X - 8.0
    ref, _, st = oracle.alg2(X, degree // 2, degree, s, l_build=l_build, l_local=l_local,
                             metric=metric, threads=4)
    graph, adj = gpu_build(X, degree, l_build=l_build, l_local=l_local, group_size=s,
                           metric=metric)
    assert (adj == ref).all(), np.argwhere(adj != ref)[:5]
    assert tuple(graph.build_stats[:3]) == tuple(int(x) for x in st)
