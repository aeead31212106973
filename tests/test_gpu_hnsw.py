"""HNSW extension (NEXT-1; Section IV-D) on the GPU vs the oracle:
permutation, layer sizes, every layer's adjacency and the search bit-exact on
integer-grid data."""
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


@pytest.mark.parametrize("n,degree,l_build,s,metric,seed,l_local", [
    (3000, 16, 32, 128, "l2", 1, 0),
    (2500, 32, 64, 256, "l2", 2, 0),
    (2000, 16, 32, 100, "ip", 3, 0),
    (2500, 32, 64, 256, "l2", 4, 24),    # every layer's Phase 1 at l_local (R-C13)
    (2000, 16, 48, 100, "ip", 5, 16),
])
def test_hnsw_build_and_search_parity(n, degree, l_build, s, metric, seed, l_local):
    cfg = syn.with_size(syn.CONFIGS["C1"], n=n, nq=100)
    X, Q = syn.points(cfg), syn.queries(cfg)
    if metric == "ip":
        X, Q = X - 128.0, Q - 128.0
    levels = syn.hnsw_levels(n, degree // 2, seed)
    ref = oracle.hnsw_build(X, levels, degree // 2, degree, s, l_build=l_build, metric=metric,
                            l_local=l_local)
    idx = g.build_hnsw(cu(X), levels, metric=metric, degree=degree, l_build=l_build, group_size=s,
                       l_local=l_local)
    torch.cuda.synchronize()
    assert idx.nlayers == len(ref["layer_n"]) and idx.layer_n == ref["layer_n"].tolist()
    assert (idx.perm() == ref["perm"]).all()
    for j in range(1, idx.nlayers):
        assert (idx.layer(j) == ref["upper"][j]).all(), j
    assert (idx.layer(0) == ref["layer0"]).all()
    ids, dists, st = g.hnsw_search(idx, cu(X), cu(Q), 10, 48, stats=True)
    oi, od, _, ost = oracle.hnsw_search(ref, X, Q, 10, 48, metric=metric, stats=True)
    assert (ids.cpu().numpy() == oi).all() and (dists.cpu().numpy() == od).all()
    st = st.cpu().numpy()
    assert (st[:, 0] == ost[:, 0]).all() and (st[:, 1] == ost[:, 1]).all()


def test_hnsw_theorem_regime():
    n = 50
    X = syn.random_int_points(n, 8, 0, 6, 77)
    levels = np.zeros(n, np.int8)
    levels[::4] = 1
    levels[::16] = 2
    idx = g.build_hnsw(cu(X), levels, degree=64, d_min=4, l_build=n + 1, group_size=7)
    ref = oracle.hnsw_build(X, levels, 4, 64, 7, l_build=n + 1)
    for j in range(idx.nlayers):
        assert (idx.layer(j) == (ref["layer0"] if j == 0 else ref["upper"][j])).all()


def test_hnsw_c2_recall_beats_or_matches_nsw():
    """Full C2 size: HNSW (same degree, d_min, l_build) reaches at least the NSW
    graph's recall at the same (l, e) and needs fewer layer-0 iterations."""
    cfg = syn.CONFIGS["C2"]
    X, Q = syn.points(cfg), syn.queries(cfg)
    Xd, Qd = cu(X), cu(Q[:2000])
    levels = syn.hnsw_levels(cfg.n, cfg.degree // 2, 1)
    idx = g.build_hnsw(Xd, levels, degree=cfg.degree, l_build=64)
    nsw = g.build(Xd, degree=cfg.degree, l_build=64)
    gt, _ = oracle.bruteforce(X, Q[:2000], 10)
    hi, _, hs = g.hnsw_search(idx, Xd, Qd, 10, 64, stats=True)
    ni, _, ns = g.search(nsw, Xd, Qd, 10, 64, stats=True)
    rh, rn = oracle.recall(hi.cpu().numpy(), gt), oracle.recall(ni.cpu().numpy(), gt)
    assert rh >= rn - 0.005, (rh, rn)
    assert hs[:, 0].float().mean() <= ns[:, 0].float().mean() + 1.0


def test_hnsw_wide_rows_entry_kernel_path():
    """d > 256: the search takes the separate entry-kernel path (the descent is fused
    into K1 only for d <= 256); bit-exact vs the oracle as well."""
    n, d = 1500, 384
    X = syn.random_int_points(n, d, 0, 15, 11)
    Q = syn.random_int_points(60, d, 0, 15, 12)
    levels = syn.hnsw_levels(n, 8, 5)
    ref = oracle.hnsw_build(X, levels, 8, 16, 128, l_build=32)
    idx = g.build_hnsw(cu(X), levels, degree=16, l_build=32, group_size=128)
    assert (idx.layer(0) == ref["layer0"]).all()
    ids, dists, st = g.hnsw_search(idx, cu(X), cu(Q), 10, 40, stats=True)
    oi, od, _, ost = oracle.hnsw_search(ref, X, Q, 10, 40, stats=True)
    assert (ids.cpu().numpy() == oi).all() and (dists.cpu().numpy() == od).all()
    assert (st.cpu().numpy()[:, 0] == ost[:, 0]).all()


def test_hnsw_search_host_async():
    """ganns_hnsw_search_host_async (H2D, search, D2H on a stream) == hnsw_search."""
    cfg = syn.with_size(syn.CONFIGS["C1"], n=3000, nq=64)
    X, Q = syn.points(cfg), syn.queries(cfg)
    levels = syn.hnsw_levels(3000, 8, 2)
    idx = g.build_hnsw(cu(X), levels, degree=16, l_build=32, group_size=128)
    Xd = cu(X)
    ids, dists = g.hnsw_search(idx, Xd, cu(Q), 10, 48)
    scratch = (torch.empty((64, X.shape[1]), dtype=torch.float32, device=DEV),
               torch.empty((64, 10), dtype=torch.int32, device=DEV),
               torch.empty((64, 10), dtype=torch.float32, device=DEV))
    hout = (torch.empty((64, 10), dtype=torch.int32).pin_memory(),
            torch.empty((64, 10), dtype=torch.float32).pin_memory())
    s = torch.cuda.Stream()
    g.search_host_async(idx, Xd, torch.from_numpy(Q).pin_memory(), 10, 48, scratch, hout, stream=s)
    s.synchronize()
    assert (hout[0] == ids.cpu()).all() and (hout[1] == dists.cpu()).all()
