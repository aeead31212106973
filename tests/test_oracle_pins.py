"""Pins of the CPU oracle against the paper and the mathematics (no GPU).

Each test names what it pins.
None of these retypes an oracle formula: they compare it with values the paper
prints for its worked examples, closed forms, an independent library routine
(numpy lexsort) on tiny inputs, brute force, the paper's quality theorem, and
invariants that any correct implementation satisfies.
"""
import itertools

import numpy as np
import pytest

import oracle
import ganns_synth as syn


# ----------------------------------------------------------------- O1 (R-C9)
def test_distance_closed_forms():
    # hand-computed: (1-4)^2 + (2-6)^2 = 25
    assert oracle.distance([1, 2, 3, 4], [4, 6, 3, 4], "l2") == 25.0
    # -<(1,2,3,4),(2,0,-1,1)> = -(2 + 0 - 3 + 4) = -3
    assert oracle.distance([1, 2, 3, 4], [2, 0, -1, 1], "ip") == -3.0
    # 1 - <(3,4,0,0),(1,0,0,0)> / 5 = 0.4
    assert abs(oracle.distance([3, 4, 0, 0], [1, 0, 0, 0], "cosine") - 0.4) < 1e-7
    # orthogonal IP is +0.0, never -0.0 (total order on keys)
    z = oracle.distance([1, 0, 0, 0], [0, 1, 0, 0], "ip")
    assert z == 0.0 and np.signbit(np.float32(z)) == False  # noqa: E712


def test_distance_matches_numpy_float64():
    rng = np.random.default_rng(1)
    for metric in ("l2", "ip", "cosine"):
        for d in (4, 8, 128, 960):
            q = rng.standard_normal(d).astype(np.float32)
            x = rng.standard_normal(d).astype(np.float32)
            q64, x64 = q.astype(np.float64), x.astype(np.float64)
            ref = {"l2": ((q64 - x64) ** 2).sum(), "ip": -(q64 @ x64),
                   "cosine": 1 - (q64 @ x64) / np.linalg.norm(q64)}[metric]
            assert oracle.distance(q, x, metric) == np.float32(ref)


# ----------------------------------------------------------- P1: Example 2
def test_example2_trace(g1):
    """GANNS on Fig. 1: T of iteration 1 sorts v8,v7,v2,v5,v3; path
    v1->v8->v10->v12->v9; iteration 5 explores v9 (the only unexplored point) and
    leaves N unchanged; returns v12, v9, v8, v10."""
    ex = g1["ex2"]
    tr = oracle.search_trace(g1["nbr"], g1["X"], g1["q"], k=4, l=4, e=4, entry=0)
    assert tr["explored"].tolist() == [it["explore"] for it in ex["its"]]
    for i, it in enumerate(ex["its"]):
        assert tr["N"][i].tolist() == it["N"], f"iteration {i + 1}"
        assert tr["flags"][i].tolist() == it["flags"], f"iteration {i + 1}"
        t = tr["T"][i]
        assert t[t >= 0].tolist() == it["tsorted"], f"iteration {i + 1}"
    assert tr["ids"].tolist() == ex["result"]
    assert tr["dists"].tolist() == ex["dists"]
    assert tr["stats"][:3].tolist() == ex["stats"]
    # merged entries, read off the N states above: 3 + 1 + 2 + 1 + 0
    assert int(tr["stats"][3]) == 7
    # iteration 5 leaves N unchanged
    assert tr["N"][4].tolist() == tr["N"][3].tolist()


def test_example2_literal_dup_reading_is_rejected(g1):
    """R-C1: the oracle drops duplicates; its result equals the paper's list.  The
    alternative reading ("keep duplicates, flag them explored") would return v12
    twice -- a contradiction with P:214 -- so the oracle must never emit a repeated id."""
    ids, _ = oracle.search(g1["nbr"], g1["X"], g1["q"][None], k=4, l=4)
    assert len(set(ids[0].tolist())) == 4


# ----------------------------------------------------------- P2: Example 1
def test_example1_trace(g1):
    """Algorithm 1 on Fig. 1: pops v1, v8, v10, v12, v9; then C's closest
    is v4, worse than v10; returns v12, v9, v8, v10."""
    ex = g1["ex1"]
    r = oracle.alg1(g1["nbr"], g1["X"], g1["q"], k=4, entry=0)
    assert r["pops"].tolist() == ex["pops"]
    assert r["cmin"] == ex["cmin"][0]
    assert r["ids"].tolist() == ex["result"]
    assert r["dist_comps"] == ex["dist_comps"][0]


def test_g1_is_nsw_with_dmin2(g1):
    """G1 is an NSW graph with d_min = 2: v7's neighbours are v1, v5
    (forward) and v8 (backward).  Checks the fixture, not the oracle."""
    nbr = g1["nbr"]
    assert sorted(nbr[6][nbr[6] >= 0].tolist()) == [0, 4, 7]
    for v in range(12):
        row = set(nbr[v][nbr[v] >= 0].tolist())
        for u in row:
            assert v in set(nbr[u][nbr[u] >= 0].tolist())   # bidirectional links
        fwd = [u for u in row if u < v]
        assert len(fwd) == min(2, v) or len(fwd) >= 2


# ---------------------------------------------------- P4: brute force (O6)
@pytest.mark.parametrize("metric", ["l2", "ip"])
def test_bruteforce_matches_lexsort(metric):
    for seed in range(20):
        X = syn.random_int_points(60, 5, 0, 3, seed)        # heavy ties
        Q = syn.random_int_points(7, 5, 0, 3, 100 + seed)
        ids, dists = oracle.bruteforce(X, Q, k=9, metric=metric, threads=2)
        for qi in range(len(Q)):
            diff = X.astype(np.int64) - Q[qi].astype(np.int64)
            dd = (diff ** 2).sum(1) if metric == "l2" else -(X.astype(np.int64) @ Q[qi].astype(np.int64))
            order = np.lexsort((np.arange(len(X)), dd))[:9]
            assert ids[qi].tolist() == order.tolist()
            assert dists[qi].tolist() == dd[order].astype(np.float32).tolist()


# ------------------------------------- P3: search == brute force when l >= n
def _strongly_connected_graph(n, d_max, seed):
    adj = syn.random_graph(n, d_max, seed, min_degree=1)
    # a Hamiltonian cycle in slot 0 makes every vertex reachable from any entry
    for v in range(n):
        row = [u for u in adj[v].tolist() if u >= 0 and u != (v + 1) % n]
        row = [(v + 1) % n] + row
        adj[v] = (row + [-1] * d_max)[:d_max]
    return adj


@pytest.mark.parametrize("metric", ["l2", "ip"])
def test_search_exact_when_l_ge_n(metric):
    for seed in range(30):
        n = 20 + seed % 17
        X = syn.random_int_points(n, 4, 0, 4, seed)
        Q = syn.random_int_points(3, 4, 0, 4, 500 + seed)
        nbr = _strongly_connected_graph(n, 4, seed)
        l = n + seed % 3
        for k in (1, 5, n - 1):
            ids, dists = oracle.search(nbr, X, Q, k=k, l=l, entry=seed % n, metric=metric)
            gi, gd = oracle.bruteforce(X, Q, k=k, metric=metric, threads=1)
            assert (ids == gi).all() and (dists == gd).all()


# --------------------------------------------------- P5: search invariants
def test_search_invariants_tie_heavy():
    """Per-iteration invariants on 1500 tie-heavy random digraphs."""
    rng = np.random.default_rng(5)
    checked = 0
    for seed in range(1500):
        n = int(rng.integers(3, 30))
        d_max = int(rng.integers(1, 6))
        X = syn.random_int_points(n, 2, 0, 2, seed)          # distances in 0..8
        q = syn.random_int_points(1, 2, 0, 2, 10_000 + seed)[0]
        nbr = syn.random_graph(n, min(d_max, n - 1), seed, min_degree=0)
        l = int(rng.integers(1, 17))
        e = int(rng.integers(1, l + 1))
        k = int(rng.integers(1, l + 1))
        entry = int(rng.integers(0, n))
        tr = oracle.search_trace(nbr, X, q, k=k, l=l, e=e, entry=entry)
        dist = ((X.astype(np.int64) - q.astype(np.int64)) ** 2).sum(1)
        explored = tr["explored"].tolist()
        assert len(explored) == len(set(explored))              # never explored twice
        assert len(explored) <= n
        prev_worst = None
        prev_N, prev_F = [entry], [0]
        comps = 1
        for i, v in enumerate(explored):
            # v was the first unexplored entry among the first e of the previous N
            cand = [u for u, f in zip(prev_N[:e], prev_F[:e]) if not f]
            assert cand and cand[0] == v
            N = [u for u in tr["N"][i].tolist() if u >= 0]
            F = tr["flags"][i][:len(N)].tolist()
            keys = [(dist[u], u) for u in N]
            assert keys == sorted(keys) and len(set(N)) == len(N) and len(N) <= l
            if len(N) == l:
                if prev_worst is not None:
                    assert keys[-1] <= prev_worst                 # l-th key never increases
                prev_worst = keys[-1]
            # explored flags survive; new entries are unexplored
            for u, f in zip(N, F):
                was = u == v or (u in prev_N and prev_F[prev_N.index(u)] == 1)
                assert f == int(was)
            # N is the l smallest of prev_N ∪ valid neighbours (a set)
            row = [u for u in nbr[v].tolist() if u >= 0]
            comps += len(row)
            union = sorted(set(prev_N) | set(row), key=lambda u: (dist[u], u))[:l]
            assert N == union
            prev_N, prev_F = N, F
        # termination: no unexplored entry among the first e
        assert explored and all(prev_F[:e])
        assert int(tr["stats"][0]) == len(explored)
        assert int(tr["stats"][1]) == comps
        out = [u for u in tr["ids"].tolist() if u >= 0]
        assert out == prev_N[:k]
        checked += 1
    assert checked == 1500


# -------------------------------------------- NSW definition
def test_nsw_seq_exact_definition():
    """Sequential NSW with exact NN: v's forward edges are its d_min nearest among
    earlier points (all of them if fewer), links are bidirectional; checked with
    an independent numpy lexsort."""
    for seed in range(10):
        n, d_min = 25, 3
        X = syn.random_int_points(n, 3, 0, 3, seed)
        ids, dists, _ = oracle.nsw_seq(X, d_min, n - 1, exact=True)
        D = ((X[:, None, :].astype(np.int64) - X[None].astype(np.int64)) ** 2).sum(-1)
        for v in range(n):
            fwd = np.lexsort((np.arange(v), D[v, :v]))[:d_min].tolist() if v else []
            row = ids[v][ids[v] >= 0].tolist()
            assert set(fwd) <= set(row)
            expect = set(fwd) | {w for w in range(v + 1, n)
                                 if v in np.lexsort((np.arange(w), D[w, :w]))[:d_min]}
            assert set(row) == expect
            keys = [(D[v, u], u) for u in row]
            assert keys == sorted(keys)
            assert dists[v][:len(row)].tolist() == [float(D[v, u]) for u in row]


# ----------------------------------- P6: quality theorem
@pytest.mark.parametrize("metric", ["l2", "ip"])
def test_alg2_equals_sequential_nsw_exact(metric):
    rng = np.random.default_rng(3)
    for seed in range(30):
        n = int(rng.integers(20, 91))
        d = int(rng.integers(2, 7))
        d_min = int(rng.integers(2, 5))
        d_max = 2 * d_min
        X = syn.random_int_points(n, d, 0, 4, 300 + seed)
        ref_i, ref_d, _ = oracle.nsw_seq(X, d_min, d_max, exact=True, metric=metric)
        for s in (1, 3, 7, 16, n):
            gi, gd, _ = oracle.alg2(X, d_min, d_max, s, exact=True, metric=metric)
            assert (gi == ref_i).all(), (seed, s)
            assert (gd == ref_d).all(), (seed, s)


def test_alg2_equals_sequential_nsw_search_regime():
    """Without an exact-NN hook: d_max >= n-1 (no truncation => connected) and
    l_build >= n make every build search exact (P3), so the theorem applies to the
    search-driven builds too.  This is the regime the GPU build is checked in."""
    for seed in range(12):
        n = 40 + seed
        X = syn.random_int_points(n, 4, 0, 6, 700 + seed)
        ref_i, _, _ = oracle.nsw_seq(X, 4, n - 1, exact=True)
        seq_i, _, _ = oracle.nsw_seq(X, 4, n - 1, l_build=n + 1)
        assert (seq_i == ref_i).all()
        for s in (5, 16, n):
            gi, _, _ = oracle.alg2(X, 4, n - 1, s, l_build=n + 1)
            assert (gi == ref_i).all(), (seed, s)


# ------------------------------------------------ P7: graph invariants
def _check_graph_invariants(ids, dists, X, d_max, metric="l2"):
    n = ids.shape[0]
    for v in range(n):
        row = ids[v].tolist()
        c = sum(1 for u in row if u >= 0)
        assert all(u >= 0 for u in row[:c]) and all(u == -1 for u in row[c:])  # -1 suffix
        assert c <= d_max and v not in row[:c] and len(set(row[:c])) == c
        keys = [(dists[v][j], row[j]) for j in range(c)]
        assert keys == sorted(keys)
        for j in range(0, c, max(1, c // 3)):
            assert dists[v][j] == oracle.distance(X[v], X[row[j]], metric)


def test_alg2_approx_invariants_and_groups():
    X = syn.points(syn.with_size(syn.CONFIGS["C1"], n=1500))
    for s in (64, 300, 1500):
        ids, dists, st = oracle.alg2(X, 8, 16, s, l_build=32)
        _check_graph_invariants(ids, dists, X, 16)
        sizes = [min(s, 1500 - g) for g in range(0, 1500, s)]
        assert st[2] == sum(z - 1 for z in sizes) + (1500 - sizes[0])   # searches run


def test_alg2_max_rounds_zero_is_union_of_local_graphs():
    X = syn.points(syn.with_size(syn.CONFIGS["C1"], n=900))
    ids, _, _ = oracle.alg2(X, 8, 16, 300, l_build=32, max_rounds=0)
    for g in range(3):
        sub, _, _ = oracle.nsw_seq(X[g * 300:(g + 1) * 300], 8, 16, l_build=32)
        sub = np.where(sub >= 0, sub + g * 300, -1)
        assert (ids[g * 300:(g + 1) * 300] == sub).all()


def test_alg2_l_local_is_phase1_only():
    """l_local (R-C13) sets the list length of the Phase-1 searches only: (1) with
    max_rounds = 0 the result is each group's sequential NSW at list length l_local;
    (2) once l_local >= the group size every local search is exhaustive (l >= |G_i|,
    connected local graph: pin P3), so any such l_local gives the same graph; (3) a
    short l_local still changes the local graphs (the parameter is live)."""
    X = syn.points(syn.with_size(syn.CONFIGS["C1"], n=900))
    ids, _, _ = oracle.alg2(X, 8, 16, 300, l_build=64, max_rounds=0, l_local=16)
    for g in range(3):
        sub, _, _ = oracle.nsw_seq(X[g * 300:(g + 1) * 300], 8, 16, l_build=16)
        sub = np.where(sub >= 0, sub + g * 300, -1)
        assert (ids[g * 300:(g + 1) * 300] == sub).all()
    a, _, _ = oracle.alg2(X, 8, 16, 60, l_build=96, l_local=64)
    b, _, _ = oracle.alg2(X, 8, 16, 60, l_build=96, l_local=96)
    assert (a == b).all()
    c, _, _ = oracle.alg2(X, 8, 16, 300, l_build=64, l_local=8)
    d, _, _ = oracle.alg2(X, 8, 16, 300, l_build=64)
    assert (c != d).any()
    with pytest.raises(Exception):
        oracle.alg2(X, 8, 16, 300, l_build=64, l_local=128)   # l_local > l_build


# ------------------------------------- P8: Fig. 12 quality (statistical)
def test_alg2_quality_matches_sequential_nsw():
    """Fig. 12: GGraphCon's graph is as good as the sequential NSW
    graph; GNaiveParallel's is worse."""
    cfg = syn.with_size(syn.CONFIGS["C1"], n=4000, nq=100)
    X, Q = syn.points(cfg), syn.queries(cfg)
    gt, _ = oracle.bruteforce(X, Q, 10)
    seq, _, _ = oracle.nsw_seq(X, 8, 16, l_build=32)
    a2, _, _ = oracle.alg2(X, 8, 16, 128, l_build=32)
    nv, _ = oracle.naive_parallel(X, 8, 16, 500, l_build=32)
    rec = {}
    for name, g in (("seq", seq), ("alg2", a2), ("naive", nv)):
        ids, _ = oracle.search(g, X, Q, k=10, l=32, threads=4)
        rec[name] = oracle.recall(ids, gt)
    assert abs(rec["alg2"] - rec["seq"]) <= 0.03, rec
    assert rec["naive"] < rec["alg2"] - 0.02, rec


@pytest.mark.parametrize("batch", [1, 2, 5])
def test_naive_parallel_exact_regime_definition(batch):
    """GNaiveParallel with l_build >= n and d_max >= n - 1, checked
    against its definition written out with BFS + numpy lexsort: every point of a
    batch takes the d_min nearest of the points reachable from entry 0 in the
    graph as it stood before the batch (an l >= n search returns exactly the
    reachable set, P3), and the batch's links are added afterwards, both ways."""
    for seed in range(8):
        n, d_min = 23, 3
        X = syn.random_int_points(n, 3, 0, 4, 700 + seed)
        ids, dists = oracle.naive_parallel(X, d_min, n - 1, batch, l_build=n + 1)
        D = ((X[:, None, :].astype(np.int64) - X[None].astype(np.int64)) ** 2).sum(-1)
        adj = [set() for _ in range(n)]
        for b0 in range(0, n, batch):
            b1 = min(b0 + batch, n)
            reach = set()
            if b0 > 0:
                reach, todo = {0}, [0]
                while todo:
                    u = todo.pop()
                    for w in adj[u]:
                        if w not in reach:
                            reach.add(w)
                            todo.append(w)
            cand = np.array(sorted(reach), np.int64)
            new = []
            for v in range(b0, b1):
                if len(cand):
                    f = cand[np.lexsort((cand, D[v, cand]))[:d_min]]
                    new += [(v, int(u)) for u in f]
            for v, u in new:
                adj[v].add(u)
                adj[u].add(v)
        for v in range(n):
            row = ids[v][ids[v] >= 0].tolist()
            assert sorted(row, key=lambda u: (D[v, u], u)) == row, (seed, v)
            assert set(row) == adj[v], (seed, v)
            assert dists[v][:len(row)].tolist() == [float(D[v, u]) for u in row]


# ------------------------------- shard merge == global brute force
@pytest.mark.parametrize("W", [1, 2, 3, 8])
def test_merge_topk_of_exact_shards_is_global_bruteforce(W):
    """If every shard returns its exact top-k, the merged top-k is the exact
    top-k of the whole base set (Def. 1 on the union)."""
    X = syn.random_int_points(400, 4, 0, 3, 41 + W)     # tie-heavy
    Q = syn.random_int_points(9, 4, 0, 3, 99)
    k = 12
    bounds = np.linspace(0, len(X), W + 1).astype(int)
    sid, sd = [], []
    for a, b in zip(bounds[:-1], bounds[1:]):
        i, d = oracle.bruteforce(X[a:b], Q, k, threads=1)
        sid.append(np.where(i >= 0, i + a, -1))
        sd.append(d)
    mi, md = oracle.merge_topk(np.stack(sid), np.stack(sd))
    gi, gd = oracle.bruteforce(X, Q, k, threads=1)
    assert (mi == gi).all() and (md == gd).all()


# ------------------------------------------------ HNSW, NEXT-1
def test_hnsw_levels_are_geometric():
    lv = syn.hnsw_levels(200_000, 16, 1)
    for j in (1, 2, 3):
        frac = (lv >= j).mean()
        assert abs(frac - 16.0 ** -j) < 4 * np.sqrt(16.0 ** -j / 200_000) + 1e-4


def test_hnsw_layers_are_id_prefixes_and_exact_regime_is_sequential_nsw():
    """With exact searches (l_build >= n, d_max >= n-1) every layer equals the
    sequential NSW of its points taken in shuffled order (quality theorem per
    layer), upper layers only reference ids of their prefix, and layer 0 is
    that graph relabelled to the original ids (P:373 steps 1-3)."""
    for seed in range(6):
        n = 40 + seed * 3
        X = syn.random_int_points(n, 4, 0, 6, 40 + seed)
        levels = np.zeros(n, np.int8)
        rng = np.random.default_rng(seed)
        levels[rng.choice(n, 12, replace=False)] = 1
        levels[rng.choice(np.nonzero(levels)[0], 4, replace=False)] = 2
        h = oracle.hnsw_build(X, levels, 3, 64, group_size=7, l_build=n + 1)
        perm, ln = h["perm"], h["layer_n"]
        # perm: stable by level descending
        order = sorted(range(n), key=lambda v: (-levels[v], v))
        assert perm.tolist() == order
        assert ln.tolist() == [n, 12, 4]
        Xp = X[perm]
        for j in (1, 2):
            up = h["upper"][j]
            assert up.max() < ln[j]
            ref, _, _ = oracle.nsw_seq(Xp[:ln[j]], 3, 64, exact=True)
            assert (up == ref).all()
        ref0, _, _ = oracle.nsw_seq(Xp, 3, 64, exact=True)
        relab = np.full_like(ref0, -1)
        for v in range(n):
            row = ref0[v]
            relab[perm[v]] = np.where(row >= 0, perm[np.maximum(row, 0)], -1)
        assert (h["layer0"] == relab).all()
        # search: exact layer 0 search whatever the entry; the descent entry is the
        # nearest top-layer point (greedy on complete upper layers)
        Q = syn.random_int_points(5, 4, 0, 6, 90 + seed)
        ids, dists, ent = oracle.hnsw_search(h, X, Q, 5, n + 1)
        gi, gd = oracle.bruteforce(X, Q, 5)
        assert (ids == gi).all() and (dists == gd).all()


def test_hnsw_quality_at_least_nsw():
    cfg = syn.with_size(syn.CONFIGS["C1"], n=4000, nq=100)
    X, Q = syn.points(cfg), syn.queries(cfg)
    gt, _ = oracle.bruteforce(X, Q, 10)
    lv = syn.hnsw_levels(len(X), 8, 3)
    h = oracle.hnsw_build(X, lv, 8, 16, group_size=128, l_build=32)
    nsw, _, _ = oracle.alg2(X, 8, 16, 128, l_build=32)
    ih, _, _ = oracle.hnsw_search(h, X, Q, 10, 32)
    inn, _ = oracle.search(nsw, X, Q, 10, 32)
    assert oracle.recall(ih, gt) >= oracle.recall(inn, gt) - 0.02


# --------------------------------------- KNN graph, NN-Descent form (NEXT-4)
def _exact_knn_lists(X, K):
    gi, gd = oracle.bruteforce(X, X, K + 1)
    ids = np.array([[u for u in r if u != i][:K] for i, r in enumerate(gi)], np.int32)
    return ids


def test_knn_exact_init_is_a_fixed_point():
    """If every list already holds the exact K nearest, no proposal can enter:
    one iteration, nothing changes ("terminates when ... cease to change")."""
    X = syn.random_int_points(300, 6, 0, 50, 4)
    ex = _exact_knn_lists(X, 8)
    ids, dists, it, ch = oracle.knn_descent(X, ex, 8, 10)
    assert it == 1 and ch == 0
    assert (ids == ex).all()


def test_knn_lists_only_improve_and_converge():
    cfg = syn.with_size(syn.CONFIGS["C1"], n=1200)
    X = syn.points(cfg)
    init = syn.random_graph(len(X), 12, seed=9)
    prev = None
    for t in range(0, 6):
        ids, dists, it, ch = oracle.knn_descent(X, init, 12, t)
        if prev is not None:
            assert (dists <= prev + 0).all()          # element-wise non-increasing
        prev = dists
        for v in range(0, len(X), 97):              # rows sorted, distinct, no self loop
            row = ids[v][ids[v] >= 0]
            assert v not in row and len(set(row.tolist())) == len(row)
            assert all(dists[v][i] <= dists[v][i + 1] for i in range(len(row) - 1))
            assert dists[v][0] == oracle.distance(X[v], X[row[0]])
    ids, dists, it, ch = oracle.knn_descent(X, init, 12, 50)
    assert ch == 0 and it < 50
    assert oracle.recall(ids, _exact_knn_lists(X, 12)) > 0.9


def test_knn_complete_lists_are_exact():
    """K = n - 1: every list holds all other points, sorted = the exact lists."""
    X = syn.random_int_points(20, 3, 0, 9, 6)
    init = syn.random_graph(20, 19, seed=1)
    ids, dists, it, ch = oracle.knn_descent(X, init, 19, 3)
    assert (ids == _exact_knn_lists(X, 19)).all()
