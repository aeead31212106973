"""CUDA path (libganns.so through its C ABI) vs the CPU oracle, on the same seeded
inputs.  Integer-grid data makes every fp32 distance exact, so ids, distances and
per-query counters must be bit-identical (DESIGN.md
"Parity bar").  Cosine data (non-integer) is compared to 1e-5 relative with
recall within 0.002 (BASELINE.json north_star).
"""
import numpy as np
import pytest
import torch

import oracle
import ganns_synth as syn

pytestmark = pytest.mark.gpu

g = pytest.importorskip("paper_conf_icde_yuwzqzl22_b200") if torch.cuda.is_available() else None
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to(DEV)


def gpu_search(graph, X, Q, k, l, e=0, entry=0):
    ids, dists, st = g.search(graph, cu(X), cu(Q), k, l, e=e, entry=entry, stats=True)
    torch.cuda.synchronize()
    return ids.cpu().numpy(), dists.cpu().numpy(), st.cpu().numpy()


def assert_search_parity(nbr, X, Q, k, l, e=0, entry=0, metric="l2"):
    graph = g.from_adjacency(nbr, X.shape[1], metric)
    gi, gd, gs = gpu_search(graph, X, Q, k, l, e, entry)
    oi, od, os_ = oracle.search(nbr, X, Q, k, l, e=e, entry=entry, metric=metric, threads=8,
                                stats=True)
    assert (gi == oi).all(), np.argwhere(gi != oi)[:5]
    assert (gd == od).all()
    assert (gs[:, 0] == os_[:, 0]).all() and (gs[:, 1] == os_[:, 1]).all()
    assert (gs[:, 2] == os_[:, 3]).all()
    return gi, gd


# ------------------------------------------------------------- worked example
def test_example2_through_abi(g1):
    """Example 2 on the GPU: result v12, v9, v8, v10; 5 iterations,
    17 distance computations."""
    graph = g.from_adjacency(g1["nbr"], 4)
    ids, dists, st = gpu_search(graph, g1["X"], g1["q"][None], k=4, l=4, e=4)
    assert ids[0].tolist() == g1["ex2"]["result"]
    assert dists[0].tolist() == g1["ex2"]["dists"]
    assert st[0].tolist() == [5, 17, 7]


# -------------------------------------------------- search parity, imported graphs
@pytest.fixture(scope="module")
def c1():
    cfg = syn.CONFIGS["C1"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    nbr, _, _ = oracle.alg2(X, 8, 16, 256, l_build=32)
    return X, Q, nbr


@pytest.mark.parametrize("l", [10, 31, 32, 33, 64, 100, 256, 1024])
def test_search_parity_c1_oracle_graph(c1, l):
    X, Q, nbr = c1
    assert_search_parity(nbr, X, Q, k=10, l=l)


@pytest.mark.parametrize("e", [1, 5, 40, 64])
def test_search_parity_explore_budget(c1, e):
    X, Q, nbr = c1
    assert_search_parity(nbr, X, Q, k=10, l=64, e=e)


def test_search_parity_entry_and_k(c1):
    X, Q, nbr = c1
    assert_search_parity(nbr, X, Q, k=1, l=16, entry=777)
    assert_search_parity(nbr, X, Q, k=64, l=64, entry=9999)
    assert_search_parity(nbr, X, Q, k=100, l=300)


@pytest.mark.parametrize("d,d_max,metric", [
    (4, 8, "l2"), (96, 32, "l2"), (128, 16, "ip"), (200, 32, "l2"), (384, 48, "l2"),
    (960, 32, "l2"), (128, 64, "l2"), (128, 128, "ip"), (256, 100, "l2"),
])
def test_search_parity_shapes(d, d_max, metric):
    """Every template family (float4/lane 1,2,4,8 x keys/lane 1,2,4 x L2/IP) on a
    ragged random graph (degrees U[d_max/2, d_max], -1 suffix)."""
    n = 3000
    X = syn.random_int_points(n, d, 0, 15 if d > 256 else 40, d + d_max)
    Q = syn.random_int_points(40, d, 0, 15 if d > 256 else 40, 7 * d)
    nbr = syn.random_graph(n, d_max, seed=d_max + d, min_degree=d_max // 2)
    for l in (16, 100):
        assert_search_parity(nbr, X, Q, k=10, l=l, metric=metric)


def test_search_edge_cases():
    X = syn.random_int_points(50, 8, 0, 5, 3)
    Q = syn.random_int_points(5, 8, 0, 5, 4)
    # isolated entry: N = [entry], output padded with (-1, +inf) (R-C8)
    nbr = np.full((50, 4), -1, np.int32)
    gi, gd = assert_search_parity(nbr, X, Q, k=3, l=8)
    assert (gi[:, 1:] == -1).all() and np.isinf(gd[:, 1:]).all()
    # self loops and a chain: every vertex reachable, l >= n => exact (P3)
    nbr = np.stack([[v, (v + 1) % 50, -1, -1] for v in range(50)]).astype(np.int32)
    gi, gd = assert_search_parity(nbr, X, Q, k=7, l=64)
    bi, bd = oracle.bruteforce(X, Q, 7)
    assert (gi == bi).all() and (gd == bd).all()
    # nq = 0 is a no-op
    graph = g.from_adjacency(nbr, 8)
    ids, dists = g.search(graph, cu(X), cu(Q[:0]), 3, 8)
    assert ids.shape == (0, 3)


def test_search_cosine_tolerance():
    """Non-integer data: distances within 1e-5 relative + 1e-6 absolute (the
    cancellation in 1 - <q,x>/||q|| near 0: 8 ulp(1.0), derived in DESIGN.md §4 and
    test_gpu_operating_points.py), recall within 0.002."""
    cfg = syn.with_size(syn.CONFIGS["C4"], n=8000, nq=200)
    X = syn.normalize_rows(syn.points(cfg))
    Q = syn.queries(cfg)
    nbr = syn.random_graph(len(X), 32, seed=11, min_degree=16)
    graph = g.from_adjacency(nbr, X.shape[1], "cosine")
    gi, gd, _ = gpu_search(graph, X, Q, 10, 128)
    oi, od = oracle.search(nbr, X, Q, 10, 128, metric="cosine", threads=8)
    np.testing.assert_allclose(gd, od, rtol=1e-5, atol=1e-6)
    gt, _ = oracle.bruteforce(X, Q, 10, metric="cosine")
    assert abs(oracle.recall(gi, gt) - oracle.recall(oi, gt)) <= 0.002
    # every returned distance is the true distance of the returned id
    for qi in range(0, 200, 37):
        for j in range(10):
            assert abs(oracle.distance(Q[qi], X[gi[qi, j]], "cosine") - gd[qi, j]) <= 1e-5 * max(1, abs(gd[qi, j]))


def test_search_deterministic_and_host_path(c1):
    X, Q, nbr = c1
    graph = g.from_adjacency(nbr, X.shape[1])
    a = gpu_search(graph, X, Q, 10, 64)
    b = gpu_search(graph, X, Q, 10, 64)
    assert all((x == y).all() for x, y in zip(a, b))
    hi, hd = g.search_host(graph, cu(X), torch.from_numpy(Q).pin_memory(), 10, 64)
    assert (hi.numpy() == a[0]).all() and (hd.numpy() == a[1]).all()


def test_search_host_async_two_streams(c1):
    """ganns_search_host_async: consecutive batches alternating over two streams
    (the bench's pipeline) give the oracle's results, bit-exact, for every batch."""
    X, Q, nbr = c1
    graph = g.from_adjacency(nbr, X.shape[1])
    Xd = cu(X)
    k, l, nq = 10, 64, 25
    batches = [torch.from_numpy(np.ascontiguousarray(Q[i * nq:(i + 1) * nq])).pin_memory()
               for i in range(len(Q) // nq)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    outs = []
    for i, qh in enumerate(batches):
        scratch = (torch.empty((nq, X.shape[1]), dtype=torch.float32, device=DEV),
                   torch.empty((nq, k), dtype=torch.int32, device=DEV),
                   torch.empty((nq, k), dtype=torch.float32, device=DEV))
        hout = (torch.empty((nq, k), dtype=torch.int32).pin_memory(),
                torch.empty((nq, k), dtype=torch.float32).pin_memory())
        g.search_host_async(graph, Xd, qh, k, l, scratch, hout, stream=streams[i % 2])
        outs.append((scratch, hout))
    torch.cuda.synchronize()
    oi, od = oracle.search(nbr, X, Q[:nq * len(batches)], k, l, threads=8)
    for i, (_, (hi, hd)) in enumerate(outs):
        assert (hi.numpy() == oi[i * nq:(i + 1) * nq]).all()
        assert (hd.numpy() == od[i * nq:(i + 1) * nq]).all()
    with pytest.raises(TypeError):   # queries must be pinned host memory
        g.search_host_async(graph, Xd, torch.from_numpy(Q[:nq]), k, l, outs[0][0], outs[0][1])


def test_abi_errors(c1):
    X, Q, nbr = c1
    graph = g.from_adjacency(nbr, X.shape[1])
    Xd, Qd = cu(X), cu(Q)
    for k, l in ((0, 10), (10, 5), (10, 1025)):
        with pytest.raises(g.GannsError):
            g.search(graph, Xd, Qd, k, l)
    with pytest.raises(g.GannsError):
        g.search(graph, Xd, Qd, 10, 64, e=65)
    with pytest.raises(g.GannsError):
        g.search(graph, Xd, Qd, 10, 64, entry=len(X))
    bad = nbr.copy()
    bad[3, 1] = bad[3, 0]
    with pytest.raises(g.GannsError):
        g.from_adjacency(bad, X.shape[1])
    with pytest.raises(g.GannsError):
        g.build(Xd, degree=1)
    with pytest.raises(g.GannsError):
        g.build(Xd, degree=16, l_build=4)


def test_graph_save_load(c1, tmp_path):
    X, Q, nbr = c1
    graph = g.from_adjacency(nbr, X.shape[1])
    p = str(tmp_path / "g.bin")
    graph.save(p)
    g2 = g.Graph.load(p)
    assert (g2.adjacency() == nbr).all() and g2.d == X.shape[1] and g2.d_max == 16


# ----------------------------------------------------------------- K6 merge
@pytest.mark.parametrize("W,k", [(1, 10), (2, 10), (8, 10), (8, 100), (3, 7)])
def test_merge_topk_parity(W, k):
    rng = np.random.default_rng(W * 100 + k)
    nq = 333
    ids = np.stack([np.sort(rng.choice(10_000, size=(nq, k), replace=True)) + s * 10_000
                    for s in range(W)]).astype(np.int32)
    dists = rng.integers(0, 50, size=(W, nq, k)).astype(np.float32)   # ties across shards
    dists = np.sort(dists, axis=2)
    ids[:, ::7, k // 2:] = -1
    dists[ids < 0] = np.inf
    # ids must be unique within a query: make them so
    for s in range(W):
        for q in range(nq):
            row = ids[s, q]
            valid = row[row >= 0]
            ids[s, q, :len(valid)] = s * 10_000 + np.arange(len(valid)) * 3 + q % 3
    oi, od = oracle.merge_topk(ids, dists)
    gi, gd = g.merge_topk(cu(ids), cu(dists))
    assert (gi.cpu().numpy() == oi).all() and (gd.cpu().numpy() == od).all()


def test_offset_ids():
    a = np.array([0, 5, -1, 7], np.int32)
    t = cu(a)
    g.offset_ids(t, 1000)
    assert t.cpu().numpy().tolist() == [1000, 1005, -1, 1007]


# ------------------------------------- wide form (d > 256): rows per TMA round
_WIDE_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, {root!r})
import oracle, ganns_synth as syn, paper_conf_icde_yuwzqzl22_b200 as g
cases = [(960, 32, "l2", 300), (384, 48, "ip", 300), (512, 100, "l2", 300), (960, 32, "l2", 3000)]
for d, d_max, metric, nq in cases:
    X = syn.random_int_points(2000, d, 0, 15, d + d_max)
    Q = syn.random_int_points(nq, d, 0, 15, 7 * d)
    nbr = syn.random_graph(2000, d_max, seed=d_max + d, min_degree=d_max // 2)
    nbr[5:2000:3] = -1          # empty rows: explorations with no neighbour
    graph = g.from_adjacency(nbr, d, metric)
    for l in (16, 64):
        ids, dists, st = g.search(graph, torch.from_numpy(X).cuda(), torch.from_numpy(Q).cuda(),
                                  10, l, stats=True)
        oi, od, os_ = oracle.search(nbr, X, Q, 10, l, metric=metric, threads=8, stats=True)
        assert (ids.cpu().numpy() == oi).all(), (d, d_max, l)
        assert (dists.cpu().numpy() == od).all(), (d, d_max, l)
        assert (st.cpu().numpy()[:, :2] == os_[:, :2]).all(), (d, d_max, l)
print("ok")
"""


@pytest.mark.parametrize("group", ["1", "0"])
@pytest.mark.parametrize("rows", [1, 3, 5, 7, 8])
def test_search_parity_wide_rows_per_round(group, rows):
    """Wide rows (d > 256) run on a warp group per query (GANNS_WIDE_GROUP=1, the
    default) or one warp (=0), staging R rows per TMA round (the launcher lowers R
    so a small batch fits one wave).  Every form and R in 1..8 must give the
    oracle's results bit for bit, including explorations of empty rows and
    several queries per persistent CTA.  Knobs are read once, so each
    combination runs in a child process."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, GANNS_WIDE_ROWS=str(rows), GANNS_WIDE_GROUP=group)
    r = subprocess.run([sys.executable, "-c", _WIDE_CHILD.format(root=root)], env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and r.stdout.strip().endswith("ok"), r.stderr[-3000:]
