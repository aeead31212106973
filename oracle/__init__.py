"""CPU oracle for GANNS search / GGraphCon construction -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline (and
``--impl reference``) leg may import this package.  The product path
(paper_conf_icde_yuwzqzl22_b200) never imports it and shares no code with it.

This module is argument marshalling (ctypes + numpy) around the plain C
implementation in ``ganns_oracle.c``; see that file for the per-function
citations of PAPER.md and for what pins each function.
"""
from __future__ import annotations

import ctypes as ct
import os
import subprocess
import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ganns_oracle.c")
_LIB = os.path.join(_HERE, "libganns_oracle.so")

METRICS = {"l2": 0, "ip": 1, "cosine": 2}


def build(force: bool = False) -> str:
    """Compile the oracle with plain gcc -O2 (no intrinsics, no OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".{os.getpid()}.tmp"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fPIC", "-shared", "-Wall",
                               "-o", tmp, _SRC, "-lm", "-lpthread"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = ct.CDLL(build())
        P = ct.c_void_p
        i32, i64 = ct.c_int, ct.c_int64
        _lib.ora_distance.restype = ct.c_float
        _lib.ora_distance.argtypes = [i32, P, P, i32]
        _lib.ora_search_one.argtypes = [P, i64, i32, P, i32, i32, P, i32, i32, i32, i64,
                                        P, P, P, P, i32]
        _lib.ora_search_batch.argtypes = [P, i64, i32, P, i32, i32, P, i64, i32, i32, i32,
                                          i64, P, P, P, i32]
        _lib.ora_alg1.argtypes = [P, i64, i32, P, i32, i32, P, i32, i64, P, P, P, i32, P, P, P]
        _lib.ora_bruteforce.argtypes = [P, i64, i32, i32, P, i64, i32, P, P, i32]
        _lib.ora_nsw_seq.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i32, P, P, P]
        _lib.ora_alg2.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i64, i32, i32, P, P, P]
        _lib.ora_alg2_ex.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i32, i64, i32, i32, P,
                                     P, P]
        _lib.ora_alg2_mt.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i32, i64, i32, i32, P,
                                     P, P, i32]
        _lib.ora_naive_parallel.argtypes = [P, i64, i32, i32, i32, i32, i32, i32, i64, P, P]
        _lib.ora_merge_topk.argtypes = [P, P, i32, i64, i32, P, P]
        _lib.ora_knn_descent.argtypes = [P, i64, i32, i32, i32, P, i32, P, P, P]
        _lib.ora_knn_descent.restype = ct.c_int
        _lib.ora_hnsw_build.argtypes = [P, i64, i32, i32, P, i32, i32, i32, i32, i32, i64, P, P,
                                        P, P, P]
        _lib.ora_hnsw_search.argtypes = [P, P, i32, P, P, i64, i32, P, i32, i32, P, i64, i32,
                                         i32, i32, P, P, P, P, P]
        for f in ("ora_hnsw_build", "ora_hnsw_search", "ora_merge_topk", "ora_search_one", "ora_search_batch", "ora_alg1", "ora_bruteforce",
                  "ora_nsw_seq", "ora_alg2", "ora_alg2_ex", "ora_alg2_mt",
                  "ora_naive_parallel"):
            getattr(_lib, f).restype = ct.c_int
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ct.c_void_p)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _check(rc):
    if rc != 0:
        raise ValueError(f"oracle returned {rc}")


def ncores() -> int:
    return len(os.sched_getaffinity(0))


def distance(q, x, metric="l2") -> float:
    q, x = _f32(q), _f32(x)
    return float(lib().ora_distance(METRICS[metric], _p(q), _p(x), q.shape[-1]))


def search(nbr, X, Q, k, l, e=0, entry=0, metric="l2", threads=1, stats=False):
    """O2 over a batch of queries.  Returns ids [nq,k], dists [nq,k] (+ stats [nq,4]:
    iterations, distance computations, lazy-check drops, merged entries)."""
    nbr, X, Q = _i32(nbr), _f32(X), _f32(np.atleast_2d(Q))
    nq = Q.shape[0]
    ids = np.empty((nq, k), np.int32)
    dists = np.empty((nq, k), np.float32)
    st = np.empty((nq, 4), np.uint32) if stats else None
    _check(lib().ora_search_batch(_p(nbr), nbr.shape[0], nbr.shape[1], _p(X), X.shape[1],
                                  METRICS[metric], _p(Q), nq, k, l, e, entry, _p(ids),
                                  _p(dists), _p(st), threads))
    return (ids, dists, st) if stats else (ids, dists)


def search_trace(nbr, X, q, k, l, e=0, entry=0, metric="l2", max_iters=None):
    """O2 for one query with the per-iteration trace.

    Returns dict(ids, dists, stats, explored=[v per iteration],
    N=[[ids after the update]], flags=[[explored flags]], T=[[sorted T ids]])."""
    nbr, X, q = _i32(nbr), _f32(X), _f32(q).reshape(-1)
    max_iters = max_iters or (nbr.shape[0] + 2)
    dm = nbr.shape[1]
    tr = np.full((max_iters, 1 + 2 * l + dm), -7, np.int32)
    ids = np.empty(k, np.int32)
    dists = np.empty(k, np.float32)
    st = np.empty(4, np.uint32)
    _check(lib().ora_search_one(_p(nbr), nbr.shape[0], nbr.shape[1], _p(X), X.shape[1],
                                METRICS[metric], _p(q), k, l, e, entry, _p(ids), _p(dists),
                                _p(st), _p(tr), max_iters))
    it = int(st[0])
    tr = tr[:min(it, max_iters)]
    return dict(ids=ids, dists=dists, stats=st, explored=tr[:, 0].copy(),
                N=tr[:, 1:1 + l].copy(), flags=tr[:, 1 + l:1 + 2 * l].copy(),
                T=tr[:, 1 + 2 * l:].copy())


def alg1(nbr, X, q, k, entry=0, metric="l2"):
    """O3 (Algorithm 1).  Returns dict(ids, dists, pops, cmin, dist_comps)."""
    nbr, X, q = _i32(nbr), _f32(X), _f32(q).reshape(-1)
    n = nbr.shape[0]
    ids = np.empty(k, np.int32)
    dists = np.empty(k, np.float32)
    pops = np.empty(n, np.int32)
    npops, cmin, comps = ct.c_int(), ct.c_int32(), ct.c_uint32()
    _check(lib().ora_alg1(_p(nbr), n, nbr.shape[1], _p(X), X.shape[1], METRICS[metric],
                          _p(q), k, entry, _p(ids), _p(dists), _p(pops), n,
                          ct.byref(npops), ct.byref(cmin), ct.byref(comps)))
    return dict(ids=ids, dists=dists, pops=pops[:npops.value].copy(), cmin=cmin.value,
                dist_comps=comps.value)


def bruteforce(X, Q, k, metric="l2", threads=None):
    """O6 exact kNN by (dist, id).  Returns ids [nq,k], dists [nq,k]."""
    X, Q = _f32(X), _f32(np.atleast_2d(Q))
    nq = Q.shape[0]
    ids = np.empty((nq, k), np.int32)
    dists = np.empty((nq, k), np.float32)
    _check(lib().ora_bruteforce(_p(X), X.shape[0], X.shape[1], METRICS[metric], _p(Q), nq,
                                k, _p(ids), _p(dists), threads or ncores()))
    return ids, dists


def recall(ids, gt) -> float:
    """O7: mean over queries of |X ∩ N(q)| / k."""
    ids, gt = np.asarray(ids), np.asarray(gt)
    k = gt.shape[1]
    hit = 0
    for a, b in zip(ids, gt):
        hit += len(set(a[a >= 0].tolist()) & set(b.tolist()))
    return hit / (k * len(gt))


def nsw_seq(X, d_min, d_max, l_build=64, e_build=0, exact=False, metric="l2"):
    """O4 sequential NSW.  Returns (ids [n,d_max], dists [n,d_max], stats[3])."""
    X = _f32(X)
    n = X.shape[0]
    ids = np.empty((n, d_max), np.int32)
    dists = np.empty((n, d_max), np.float32)
    st = np.zeros(3, np.uint64)
    _check(lib().ora_nsw_seq(_p(X), n, X.shape[1], METRICS[metric], d_min, d_max, l_build,
                             e_build, int(exact), _p(ids), _p(dists), _p(st)))
    return ids, dists, st


def alg2(X, d_min, d_max, group_size, l_build=64, e_build=0, exact=False, metric="l2",
         max_rounds=-1, l_local=0, threads=1):
    """O5 Algorithm 2.  Returns (ids [n,d_max], dists [n,d_max], stats[3]).  l_local
    (0 = l_build): list length of the Phase-1 searches on the local graphs (R-C13).
    threads > 1 splits the units the paper runs in parallel (Phase-1 groups, the
    searches of a Phase-2 round) over POSIX threads; the result does not depend on it."""
    X = _f32(X)
    n = X.shape[0]
    ids = np.empty((n, d_max), np.int32)
    dists = np.empty((n, d_max), np.float32)
    st = np.zeros(3, np.uint64)
    _check(lib().ora_alg2_mt(_p(X), n, X.shape[1], METRICS[metric], d_min, d_max, l_build,
                             e_build, l_local, group_size, int(exact), max_rounds, _p(ids),
                             _p(dists), _p(st), max(1, int(threads))))
    return ids, dists, st


def naive_parallel(X, d_min, d_max, batch, l_build=64, e_build=0, metric="l2"):
    """GNaiveParallel ablation.  Returns (ids, dists)."""
    X = _f32(X)
    n = X.shape[0]
    ids = np.empty((n, d_max), np.int32)
    dists = np.empty((n, d_max), np.float32)
    _check(lib().ora_naive_parallel(_p(X), n, X.shape[1], METRICS[metric], d_min, d_max,
                                    l_build, e_build, batch, _p(ids), _p(dists)))
    return ids, dists


def merge_topk(ids, dists):
    """k smallest (dist, id) of W per-shard lists [W, nq, k] -> [nq, k]."""
    ids, dists = _i32(ids), _f32(dists)
    W, nq, k = ids.shape
    oi = np.empty((nq, k), np.int32)
    od = np.empty((nq, k), np.float32)
    _check(lib().ora_merge_topk(_p(ids), _p(dists), W, nq, k, _p(oi), _p(od)))
    return oi, od


def hnsw_build(X, levels, d_min, d_max, group_size, l_build=64, e_build=0, metric="l2",
               l_local=0):
    """HNSW (Section IV-D).  Returns dict(perm, layer_n, upper, layer0):
    perm[new] = old; layer_n[j] = |layer j|; upper[j] (j >= 1) = [n_j, d_max] adjacency
    in shuffled ids; layer0 = [n, d_max] adjacency in original ids.  l_local (0 =
    l_build): list length of every layer's Phase-1 searches (R-C13)."""
    X = _f32(X)
    levels = np.ascontiguousarray(levels, dtype=np.int8)
    n = X.shape[0]
    L = int(levels.max()) + 1
    perm = np.empty(n, np.int32)
    layer_n = np.zeros(L, np.int64)
    nl = ct.c_int()
    cnt = [int((levels >= j).sum()) for j in range(L)]
    upper = np.empty(max(1, sum(cnt[1:]) * d_max), np.int32)
    layer0 = np.empty((n, d_max), np.int32)
    _check(lib().ora_hnsw_build(_p(X), n, X.shape[1], METRICS[metric], _p(levels), d_min, d_max,
                                l_build, e_build, l_local, group_size, _p(perm), _p(layer_n),
                                ct.byref(nl), _p(upper), _p(layer0)))
    ups, off = {}, 0
    for j in range(1, nl.value):
        ups[j] = upper[off:off + cnt[j] * d_max].reshape(cnt[j], d_max).copy()
        off += cnt[j] * d_max
    return dict(perm=perm, layer_n=layer_n, upper=ups, layer0=layer0, upper_flat=upper)


def hnsw_search(h, X, Q, k, l, e=0, metric="l2", stats=False, descent_stats=False):
    """Greedy descent through the upper layers, then GANNS on layer 0.
    Returns ids, dists, entries (+ stats [nq,4]) (+ descent stats [nq,2]: iterations,
    distance computations of the descent, summed over the upper layers)."""
    X, Q = _f32(X), _f32(np.atleast_2d(Q))
    nq = Q.shape[0]
    ids = np.empty((nq, k), np.int32)
    dists = np.empty((nq, k), np.float32)
    ent = np.empty(nq, np.int32)
    st = np.empty((nq, 4), np.uint32) if stats else None
    ds = np.empty((nq, 2), np.uint32) if descent_stats else None
    layer0 = h["layer0"]
    _check(lib().ora_hnsw_search(_p(h["perm"]), _p(h["layer_n"]), len(h["layer_n"]),
                                 _p(h["upper_flat"]), _p(layer0), layer0.shape[0],
                                 layer0.shape[1], _p(X), X.shape[1], METRICS[metric], _p(Q), nq,
                                 k, l, e, _p(ids), _p(dists), _p(st), _p(ent), _p(ds)))
    res = (ids, dists, ent, st) if stats else (ids, dists, ent)
    return res + (ds,) if descent_stats else res


def knn_descent(X, init, K, max_iters=30, metric="l2"):
    """KNN graph by neighbours-of-neighbours iterations.
    Returns (ids [n,K], dists [n,K], iterations, changed_in_last_iteration)."""
    X = _f32(X)
    init = _i32(init)
    n = X.shape[0]
    ids = np.full((n, K), -1, np.int32)
    dists = np.empty((n, K), np.float32)
    ch = ct.c_int64()
    it = lib().ora_knn_descent(_p(X), n, X.shape[1], METRICS[metric], K, _p(init), max_iters,
                               _p(ids), _p(dists), ct.byref(ch))
    if it < 0:
        raise ValueError(f"oracle returned {it}")
    return ids, dists, it, ch.value
