"""Pins of the oracle's HNSW descent / HNSW build and of its KNN-graph join step
(no GPU).  None of these retypes the oracle's C: they compare it with

* the nearest point of a layer (greedy descent on complete upper layers is exact);
* a hand-built 3-layer fixture whose greedy path is worked out by hand below;
* a Python restatement of Algorithm 2 + the HNSW construction order
  (R-H1, R-H2) written with plain lists and sorts, using only the
  oracle's O2 search (pinned by Example 2, brute force and invariants in
  test_oracle_pins.py) as a library step;
* one neighbours-of-neighbours iteration (R-K1, R-K2) written with numpy
  sets and lexsort.
"""
import numpy as np
import pytest

import oracle
import ganns_synth as syn


def _l2(a, b):
    """Exact squared L2 on integer-grid rows (int64), as fp32 (R-C18)."""
    diff = a.astype(np.int64) - b.astype(np.int64)
    return np.float32((diff * diff).sum(-1))


# ------------------------------------------------------------ HNSW descent
def test_hnsw_descent_on_complete_upper_layers_is_the_nearest_layer1_point():
    """Upper layers with at most d_min + 1 points are complete graphs (each point
    links to every earlier one, backward links complete the rest), so the greedy
    descent (GANNS with l = e = 1, R-H1) ends at the layer-1 point nearest to q by
    (dist, shuffled id) -- the upper layers live in shuffled ids (P:373 step 1);
    the layer-0 entry is that point's ORIGINAL id (perm lookup)."""
    d_min = 3
    for seed in range(8):
        n = 50
        X = syn.random_int_points(n, 4, 0, 9, 300 + seed)
        rng = np.random.default_rng(seed)
        levels = np.zeros(n, np.int8)
        l1 = rng.choice(n, 4, replace=False)          # layer 1: 4 = d_min + 1 points
        levels[l1] = 1
        levels[l1[:2]] = 2                             # layer 2: 2 points
        h = oracle.hnsw_build(X, levels, d_min, 8, group_size=9, l_build=16)
        perm = h["perm"]
        assert h["layer_n"].tolist() == [n, 4, 2]
        for j, m in ((1, 4), (2, 2)):                  # complete: every other point
            up = h["upper"][j]
            for v in range(m):
                assert sorted(up[v][up[v] >= 0].tolist()) == [u for u in range(m) if u != v]
        Q = syn.random_int_points(25, 4, 0, 9, 400 + seed)
        _, _, ent = oracle.hnsw_search(h, X, Q, 5, 16)
        for qi, q in enumerate(Q):
            sh = np.arange(4)                          # layer-1 points, shuffled ids
            dd = np.array([_l2(q, X[perm[s]]) for s in sh])
            best = sh[np.lexsort((sh, dd))[0]]
            assert ent[qi] == perm[best], (seed, qi)


def test_hnsw_descent_handbuilt_fixture():
    """Points on a line (x, 0, 0, 0); shuffled id s sits at x = XS[s]; perm maps
    shuffled -> original ids.  q at x = 3.1.

    layer 2 (ids 0, 1):       0 -> [1], 1 -> [0]
    layer 1 (ids 0..3):       0 -> [2], 1 -> [0, 2, 3], 2 -> [1], 3 -> [0]
    XS = [0, 5, 10, 2]

    Greedy by hand: layer 2 from 0 (d 9.61): T = {1 (3.61)} -> 1; explore 1:
    T = {0} -> stays 1.  Layer 1 from 1 (3.61): T = {0 (9.61), 2 (47.61),
    3 (1.21)} -> 3; explore 3: T = {0} -> stays 3.  Entry = perm[3].
    Skipping layer 2 would stay at 0 (0's only neighbour 2 is farther); reading
    layer 2's rows as layer 1 would return 1 -- both differ."""
    XS = [0.0, 5.0, 10.0, 2.0, 7.0, 12.0]       # shuffled ids 0..5 (4, 5: layer 0 only)
    perm = np.array([4, 2, 0, 5, 1, 3], np.int32)   # shuffled -> original
    n, d_max = 6, 3
    X = np.zeros((n, 4), np.float32)
    for s, x in enumerate(XS):
        X[perm[s], 0] = x
    up1 = np.array([[2, -1, -1], [0, 2, 3], [1, -1, -1], [0, -1, -1]], np.int32)
    up2 = np.array([[1, -1, -1], [0, -1, -1]], np.int32)
    # layer 0 (original ids): two components, {perm[3], perm[0]} and the rest, so
    # the result depends on the entry
    a, b = perm[3], perm[0]
    layer0 = np.full((n, d_max), -1, np.int32)
    layer0[a] = [b, -1, -1]
    layer0[b] = [a, -1, -1]
    rest = [v for v in range(n) if v not in (a, b)]
    for v in rest:
        layer0[v, :len(rest) - 1] = [u for u in rest if u != v]
    h = dict(perm=perm, layer_n=np.array([n, 4, 2], np.int64), upper={1: up1, 2: up2},
             layer0=layer0, upper_flat=np.concatenate([up1.reshape(-1), up2.reshape(-1)]))
    q = np.array([[3.1, 0, 0, 0]], np.float32)
    ids, dists, ent, st, ds = oracle.hnsw_search(h, X, q, 2, 2, stats=True, descent_stats=True)
    assert ent.tolist() == [perm[3]]
    # the descent's counters, by hand: layer 2 -- entry 0 (1 distance), explore 0
    # (T = {1}), explore 1 (T = {0}, not in N = [1]: recomputed) = 2 iterations, 3
    # distances; layer 1 -- entry 1 (1), explore 1 (T = {0, 2, 3}), explore 3
    # (T = {0}) = 2 iterations, 5 distances
    assert ds.tolist() == [[4, 8]]
    # layer-0 search from perm[3] (x = 2): its component {x=2, x=0}
    assert ids[0].tolist() == [perm[3], perm[0]]
    assert np.allclose(dists[0], [(3.1 - 2) ** 2, 3.1 ** 2])


# ---------------------------------- HNSW build == Python restatement (R-H2)
def _search1(nbr, Y, q, k, l, e, entry):
    ids, dists = oracle.search(nbr, Y, q[None], k, l, e=e, entry=entry)
    return [(float(dd), int(i)) for dd, i in zip(dists[0], ids[0]) if i >= 0]


def _alg2_restated(Y, d_min, d_max, S, l_b, entry_of, l_loc=0):
    """Algorithm 2 in plain Python lists: Phase 1 local graphs with
    sorted truncated back-insertion, searched at list length l_loc (0 = l_b,
    R-C13); Phase 2 rounds: search G_0 from entry_of(v, lo), first d_min of
    (S u N'(v)) (R-C16), v's row replaced (R-C15), E sorted by (u, dist, v) (R-C17)
    merged into u's row keeping d_max."""
    l_p1 = l_loc or l_b
    n = len(Y)
    rows = [[] for _ in range(n)]                 # sorted (dist, id) lists

    def adj():
        a = np.full((n, d_max), -1, np.int32)
        for v, r in enumerate(rows):
            a[v, :len(r)] = [u for _, u in r]
        return a

    gp = [[] for _ in range(n)]
    ng = (n + S - 1) // S
    for g in range(ng):
        lo, hi = g * S, min(n, (g + 1) * S)
        for v in range(lo, hi):
            F = [] if v == lo else _search1(adj(), Y, Y[v], d_min, l_p1, 0, lo)[:d_min]
            rows[v] = list(F)
            gp[v] = list(F)
            for dist, u in F:
                rows[u] = sorted(rows[u] + [(dist, v)])[:d_max]
    for g in range(1, ng):
        lo, hi = g * S, min(n, (g + 1) * S)
        A = adj()                                  # all searches see G_0 before the round
        new, E = {}, []
        for v in range(lo, hi):
            Sv = _search1(A, Y, Y[v], d_min, l_b, 0, entry_of(v, lo))[:d_min]
            F = sorted(Sv + gp[v])[:d_min]
            new[v] = F
            E += [(u, dist, v) for dist, u in F]
        for v, F in new.items():
            rows[v] = list(F)
        E.sort()
        for u in sorted({e[0] for e in E}):
            seg = [(dist, v) for uu, dist, v in E if uu == u]
            merged = sorted(rows[u] + seg)
            assert len({i for _, i in merged}) == len(merged)
            rows[u] = merged[:d_max]
    return adj()


@pytest.mark.parametrize("l_loc", [0, 3])
def test_hnsw_build_matches_restated_algorithm2_with_descent_entries(l_loc):
    """Non-exact regime (l_build = 6 << n).  Layers are built top-down; a Phase-2
    search of layer j enters at the greedy descent of the finished layers above
    (l = e = 1 from shuffled id 0), or at vertex 0 when that vertex is not yet in
    G_0 (R-H2).  Both branches occur in this instance.  l_loc: every layer's Phase 1
    at list length 3 (R-C13), which changes the index."""
    n, d_min, d_max, S, l_b = 420, 3, 6, 40, 6
    X = syn.random_int_points(n, 8, 0, 15, 77)
    levels = syn.hnsw_levels(n, d_min, 5)
    h = oracle.hnsw_build(X, levels, d_min, d_max, group_size=S, l_build=l_b, l_local=l_loc)
    if l_loc:
        h0 = oracle.hnsw_build(X, levels, d_min, d_max, group_size=S, l_build=l_b)
        assert (h["layer0"] != h0["layer0"]).any()
    perm = h["perm"]
    assert perm.tolist() == sorted(range(n), key=lambda v: (-levels[v], v))
    L = int(levels.max()) + 1
    sizes = [int((levels >= j).sum()) for j in range(L)]
    assert sizes[1] > 2 * S                        # layers 0 and 1 have Phase-2 rounds
    Xp = X[perm]
    built = {}
    used = {"fallback": 0, "descent": 0}
    for j in range(L - 1, -1, -1):
        def entry_of(v, lo, j=j):
            if j == L - 1:
                return 0
            cur = 0
            for jj in range(L - 1, j, -1):         # greedy: GANNS with k = l = e = 1
                cur = _search1(built[jj], Xp[:sizes[jj]], Xp[v], 1, 1, 1, cur)[0][1]
            if cur >= lo:
                used["fallback"] += 1
                return 0
            used["descent"] += cur != 0
            return cur
        built[j] = _alg2_restated(Xp[:sizes[j]], d_min, d_max, S, l_b, entry_of, l_loc)
        if j >= 1:
            assert (h["upper"][j] == built[j]).all(), f"layer {j}"
    assert used["fallback"] > 0 and used["descent"] > 0, used
    relab = np.full((n, d_max), -1, np.int32)
    for v in range(n):
        row = built[0][v]
        relab[perm[v]] = np.where(row >= 0, perm[np.maximum(row, 0)], -1)
    assert (h["layer0"] == relab).all()


# ------------------------------------------ KNN join step (R-K1, R-K2)
def _knn_iteration(X, lists, K, cap_reverse=True):
    """One neighbours-of-neighbours iteration from `lists` (int [n, K], rows
    sorted by (dist, id)): S(v) = list(v) u R(v), R(v) = the K nearest (dist, w)
    with v in list(w) (uncapped if not cap_reverse); every ordered pair a != b of
    S(v) proposes b to a; a keeps the K smallest distinct (dist, id) of its list
    and its proposals."""
    n = len(X)
    D = np.array([[_l2(X[a], X[b]) for b in range(n)] for a in range(n)], np.float64)
    rev = [[] for _ in range(n)]
    for w in range(n):
        for v in lists[w]:
            rev[v].append(w)
    R = []
    for v in range(n):
        ws = np.array(rev[v], np.int64)
        if len(ws):
            ws = ws[np.lexsort((ws, D[v, ws]))]
        R.append(ws[:K].tolist() if cap_reverse else ws.tolist())
    prop = [set() for _ in range(n)]
    for v in range(n):
        Sv = set(lists[v].tolist()) | set(R[v])
        for a in Sv:
            prop[a] |= Sv - {a}
    out = np.empty_like(lists)
    for a in range(n):
        cand = np.array(sorted(set(lists[a].tolist()) | prop[a]), np.int64)
        out[a] = cand[np.lexsort((cand, D[a, cand]))][:K]
    return out, max(len(r) for r in rev)


def test_knn_iterations_match_definition_and_reverse_cap_matters():
    n, K = 36, 4
    X = syn.random_int_points(n, 3, 0, 5, 21)        # tie-heavy
    init = syn.random_graph(n, K, seed=3, min_degree=K)
    D = np.array([[_l2(X[a], X[b]) for b in range(n)] for a in range(n)], np.float64)
    lists = np.array([r[np.lexsort((r, D[v, r]))] for v, r in enumerate(init.astype(np.int64))])
    for t in (1, 2, 3):
        nxt, max_in = _knn_iteration(X, lists, K)
        ids, dists, it, ch = oracle.knn_descent(X, init, K, t)
        assert it == t
        assert (ids == nxt).all(), f"iteration {t}"
        assert (dists == D[np.arange(n)[:, None], nxt].astype(np.float32)).all()
        assert ch == int((nxt != lists).any(1).sum())
        if t == 1:
            # the reverse cap is exercised here and changes the result
            assert max_in > K
            unc, _ = _knn_iteration(X, lists, K, cap_reverse=False)
            assert (unc != nxt).any()
        lists = nxt
