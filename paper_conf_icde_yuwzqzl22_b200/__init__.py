"""B200-native GANNS search and GGraphCon NSW construction (Yu et al., ICDE 2022).

Thin Python binding over the C ABI of ``libganns.so`` (include/ganns.h):
argument marshalling only -- every step of the search and of the build runs in
the library's sm_100a kernels.  PyTorch supplies device memory and streams.
There is no CPU fallback: if the library is missing, importing this package
raises.  Build it with ``__graft_entry__.build()`` (or ``python
paper_conf_icde_yuwzqzl22_b200/_build.py``).
"""
from __future__ import annotations

import ctypes as ct
import os

import numpy as np
import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GANNS_LIB_PATH") or os.path.join(_HERE, "libganns.so")

METRICS = {"l2": 0, "ip": 1, "cosine": 2}
_METRIC_NAMES = {v: k for k, v in METRICS.items()}


class GannsError(RuntimeError):
    pass


class _BuildParams(ct.Structure):
    _fields_ = [("d_min", ct.c_int), ("l_build", ct.c_int), ("e_build", ct.c_int),
                ("group_size", ct.c_int64), ("max_rounds", ct.c_int),
                ("stop_after_phase1", ct.c_int), ("stats", ct.POINTER(ct.c_uint64)),
                ("l_local", ct.c_int)]


class _SearchParams(ct.Structure):
    _fields_ = [("e", ct.c_int), ("entry", ct.c_int64), ("stats", ct.c_void_p),
                ("descent_stats", ct.c_void_p)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing; build it with __graft_entry__.build() "
                          "(there is no CPU fallback)")
    lib = ct.CDLL(LIB_PATH)
    P, i32, i64 = ct.c_void_p, ct.c_int, ct.c_int64
    sig = {
        "ganns_build": [P, i64, i32, i32, i32, ct.POINTER(_BuildParams), P, ct.POINTER(P)],
        "ganns_search": [P, P, P, i64, i32, i32, P, P, P],
        "ganns_search_ex": [P, P, P, i64, i32, i32, ct.POINTER(_SearchParams), P, P, P],
        "ganns_search_host": [P, P, P, i64, i32, i32, ct.POINTER(_SearchParams), P, P, P],
        "ganns_search_host_async": [P, P, P, i64, i32, i32, ct.POINTER(_SearchParams), P, P, P,
                                    P, P, P],
        "ganns_hnsw_search_host_async": [P, P, P, i64, i32, i32, ct.POINTER(_SearchParams), P, P,
                                         P, P, P, P],
        "ganns_merge_topk": [P, P, i32, i64, i32, P, P, P],
        "ganns_offset_ids": [P, i64, i64, P],
        "ganns_graph_from_adjacency": [P, i64, i32, i32, i32, i32, ct.POINTER(P)],
        "ganns_graph_adjacency": [P, P],
        "ganns_graph_device_ptr": [P, ct.POINTER(P)],
        "ganns_graph_info": [P, ct.POINTER(i64), ct.POINTER(i32), ct.POINTER(i32), ct.POINTER(i32)],
        "ganns_graph_save": [P, ct.c_char_p],
        "ganns_graph_load": [ct.c_char_p, i32, ct.POINTER(P)],
        "ganns_build_hnsw": [P, i64, i32, i32, i32, P, ct.POINTER(_BuildParams), P, ct.POINTER(P)],
        "ganns_hnsw_search": [P, P, P, i64, i32, i32, ct.POINTER(_SearchParams), P, P, P],
        "ganns_hnsw_info": [P, ct.POINTER(i32), P],
        "ganns_hnsw_layer": [P, i32, P],
        "ganns_hnsw_perm": [P, P],
        "ganns_hnsw_base": [P, ct.POINTER(P)],
        "ganns_build_knn": [P, i64, i32, i32, i32, P, i32, P, ct.POINTER(P), ct.POINTER(i32),
                            ct.POINTER(i64)],
        "ganns_build_begin": [P, i64, i32, i32, i32, ct.POINTER(_BuildParams), P, ct.POINTER(P)],
        "ganns_build_info": [P, ct.POINTER(i64), ct.POINTER(i64), ct.POINTER(i32), ct.POINTER(i32)],
        "ganns_build_phase1": [P, i64, i64, P],
        "ganns_build_rows": [P, i64, i64, P, P, P, P, i32, P],
        "ganns_build_round_search": [P, i64, i64, i64, P, P, P],
        "ganns_build_round_apply": [P, i64, P, P, P],
        "ganns_build_finish": [P, P, P, ct.POINTER(P)],
    }
    for name, args in sig.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = ct.c_int
    lib.ganns_graph_free.argtypes = [P]
    lib.ganns_graph_free.restype = None
    lib.ganns_hnsw_free.argtypes = [P]
    lib.ganns_hnsw_free.restype = None
    lib.ganns_build_abort.argtypes = [P]
    lib.ganns_build_abort.restype = None
    lib.ganns_last_error.argtypes = []
    lib.ganns_last_error.restype = ct.c_char_p
    lib.ganns_kernel_launches.argtypes = []
    lib.ganns_kernel_launches.restype = ct.c_uint64
    lib.ganns_profile_read.argtypes = [P, i32]
    lib.ganns_profile_read.restype = ct.c_int
    lib.ganns_profile_read_n.argtypes = [P, i32, i32]
    lib.ganns_profile_read_n.restype = ct.c_int
    return lib


_lib = _load()

# exported symbol list (include/ganns.h) -- checked by the CPU tests
ABI_SYMBOLS = ("ganns_build", "ganns_search", "ganns_search_ex", "ganns_search_host",
               "ganns_search_host_async", "ganns_hnsw_search_host_async",
               "ganns_merge_topk", "ganns_offset_ids", "ganns_graph_from_adjacency",
               "ganns_graph_adjacency", "ganns_graph_device_ptr", "ganns_graph_info",
               "ganns_graph_save", "ganns_graph_load", "ganns_graph_free", "ganns_last_error",
               "ganns_kernel_launches", "ganns_build_hnsw", "ganns_hnsw_search",
               "ganns_hnsw_info", "ganns_hnsw_layer", "ganns_hnsw_perm", "ganns_hnsw_base",
               "ganns_hnsw_free", "ganns_build_knn", "ganns_build_begin", "ganns_build_info",
               "ganns_build_phase1", "ganns_build_rows", "ganns_build_round_search",
               "ganns_build_round_apply", "ganns_build_finish", "ganns_build_abort",
               "ganns_profile_read", "ganns_profile_read_n")


def lib():
    return _lib


def _check(rc: int):
    if rc != 0:
        msg = _lib.ganns_last_error().decode(errors="replace")
        raise GannsError(f"ganns error {rc}: {msg}")


def _stream(stream) -> ct.c_void_p:
    if stream is None:
        stream = torch.cuda.current_stream()
    return ct.c_void_p(stream.cuda_stream)


def _check_buf(t, shape, dtype, cuda: bool, name: str):
    """Output / scratch buffers are written by the library through raw pointers:
    refuse anything that is not exactly the expected contiguous layout."""
    if not (isinstance(t, torch.Tensor) and tuple(t.shape) == tuple(shape) and t.dtype == dtype
            and t.is_cuda == cuda and t.is_contiguous()):
        where = "CUDA" if cuda else "host"
        raise TypeError(f"{name} must be a contiguous {where} {dtype} tensor of shape {tuple(shape)}")


def _check_out(out, nq: int, k: int, device):
    ids, dists = out
    _check_buf(ids, (nq, k), torch.int32, True, "out[0] (ids)")
    _check_buf(dists, (nq, k), torch.float32, True, "out[1] (dists)")
    if ids.device != device or dists.device != device:
        raise TypeError("out tensors must be on the queries' device")
    return ids, dists


def _dev_f32(t: torch.Tensor, name: str) -> torch.Tensor:
    if not (isinstance(t, torch.Tensor) and t.is_cuda and t.dtype == torch.float32 and t.dim() == 2):
        raise TypeError(f"{name} must be a 2-D float32 CUDA tensor")
    return t.contiguous()


def _check_index_inputs(graph, points: torch.Tensor, queries: torch.Tensor):
    """The kernels read points through a tensor map / row pointers built from the
    graph's (n, d) and queries (device or host) as [nq][d]: refuse any other shape
    (an out-of-bounds access otherwise) and device queries on another device."""
    if tuple(points.shape) != (graph.n, graph.d):
        raise ValueError(f"points must be [{graph.n}, {graph.d}] (the graph's n and d), "
                         f"got {list(points.shape)}")
    if queries.shape[1] != graph.d:
        raise ValueError(f"queries must have d = {graph.d} columns, got {queries.shape[1]}")
    if queries.is_cuda and points.device != queries.device:
        raise ValueError("points and queries must be on the same device")


def kernel_launches() -> int:
    """Kernels launched by libganns.so in this process."""
    return int(_lib.ganns_kernel_launches())


PROFILE_PHASES = ("locate", "explore", "distance", "lazy_check", "sort", "merge")


def profile_read(reset: bool = True):
    """Per-phase cycle counters of a GANNS_PROFILE library build (ganns_profile_read):
    dict(phase -> cycles, iterations, searches).  Raises on a normal build."""
    out = (ct.c_uint64 * 14)()
    _check(_lib.ganns_profile_read_n(ct.cast(out, ct.c_void_p), 14, int(reset)))
    d = {k: int(out[i]) for i, k in enumerate(PROFILE_PHASES)}
    d["iterations"], d["searches"] = int(out[6]), int(out[7])
    d["gather_issue"], d["gather_wait"], d["gather_rounds"] = int(out[8]), int(out[9]), int(out[10])
    d["spec_hits"] = int(out[11])
    d["max_search_cycles"], d["max_search_iterations"] = int(out[12]), int(out[13])
    return d


class Graph:
    """Fixed-degree proximity graph (int32 [n][d_max] adjacency in device memory)."""

    def __init__(self, handle: ct.c_void_p, owned: bool = True):
        self._h = handle
        self._owned = owned
        n, d, dm, m = ct.c_int64(), ct.c_int(), ct.c_int(), ct.c_int()
        _check(_lib.ganns_graph_info(handle, ct.byref(n), ct.byref(d), ct.byref(dm), ct.byref(m)))
        self.n, self.d, self.d_max, self.metric = n.value, d.value, dm.value, _METRIC_NAMES[m.value]
        self.build_stats = None

    @property
    def handle(self):
        return self._h

    def adjacency(self) -> np.ndarray:
        out = np.empty((self.n, self.d_max), np.int32)
        _check(_lib.ganns_graph_adjacency(self._h, out.ctypes.data_as(ct.c_void_p)))
        return out

    def device_adjacency(self) -> int:
        p = ct.c_void_p()
        _check(_lib.ganns_graph_device_ptr(self._h, ct.byref(p)))
        return p.value

    def save(self, path: str):
        _check(_lib.ganns_graph_save(self._h, path.encode()))

    @staticmethod
    def load(path: str, device: int = 0) -> "Graph":
        h = ct.c_void_p()
        _check(_lib.ganns_graph_load(path.encode(), device, ct.byref(h)))
        return Graph(h)

    def free(self):
        if self._h and self._owned:
            _lib.ganns_graph_free(self._h)
        self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def from_adjacency(nbr: np.ndarray, d: int, metric: str = "l2", device: int = 0) -> Graph:
    nbr = np.ascontiguousarray(nbr, dtype=np.int32)
    h = ct.c_void_p()
    _check(_lib.ganns_graph_from_adjacency(nbr.ctypes.data_as(ct.c_void_p), nbr.shape[0],
                                           nbr.shape[1], d, METRICS[metric], device, ct.byref(h)))
    return Graph(h)


def build(points: torch.Tensor, metric: str = "l2", degree: int = 32, d_min: int = 0,
          l_build: int = 0, e_build: int = 0, group_size: int = 0, max_rounds: int = 0,
          stop_after_phase1: bool = False, l_local: int = 0, stream=None) -> Graph:
    """GGraphCon NSW construction (Algorithm 2).  ``points`` [n, d] float32 CUDA
    (unit rows for metric="cosine").  Returns a Graph; ``graph.build_stats`` =
    (search iterations, distance computations, searches, rounds)."""
    points = _dev_f32(points, "points")
    st = (ct.c_uint64 * 4)()
    p = _BuildParams(d_min, l_build, e_build, group_size, max_rounds, int(stop_after_phase1),
                     ct.cast(st, ct.POINTER(ct.c_uint64)), l_local)
    h = ct.c_void_p()
    with torch.cuda.device(points.device):
        _check(_lib.ganns_build(ct.c_void_p(points.data_ptr()), points.shape[0], points.shape[1],
                                METRICS[metric], degree, ct.byref(p), _stream(stream), ct.byref(h)))
    g = Graph(h)
    g.build_stats = tuple(int(x) for x in st)
    return g


class StagedBuild:
    """Algorithm 2 one step at a time (ganns_build_begin ... ganns_build_finish; the
    multi-GPU construction of dist.build_distributed).  Same parameters as build().
    Every method enqueues on `stream` (default: the current stream)."""

    def __init__(self, points: torch.Tensor, metric: str = "l2", degree: int = 32, d_min: int = 0,
                 l_build: int = 0, e_build: int = 0, group_size: int = 0, l_local: int = 0,
                 stream=None):
        self.points = _dev_f32(points, "points")
        self.device = self.points.device
        self.stream = stream
        self.n, self.d = self.points.shape
        p = _BuildParams(d_min, l_build, e_build, group_size, 0, 0, None, l_local)
        h = ct.c_void_p()
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_begin(ct.c_void_p(self.points.data_ptr()), self.n, self.d,
                                          METRICS[metric], degree, ct.byref(p),
                                          _stream(stream), ct.byref(h)))
        self._h = h
        s, t, dm, dx = ct.c_int64(), ct.c_int64(), ct.c_int(), ct.c_int()
        _check(_lib.ganns_build_info(h, ct.byref(s), ct.byref(t), ct.byref(dm), ct.byref(dx)))
        self.group_size, self.ngroups, self.d_min, self.d_max = s.value, t.value, dm.value, dx.value

    def _p(self, t):
        return ct.c_void_p(t.data_ptr())

    def info(self):
        return self.group_size, self.ngroups, self.d_min, self.d_max

    def group_rows(self, g0: int, g1: int):
        """Vertex range [v0, v1) of groups [g0, g1)."""
        return min(g0 * self.group_size, self.n), min(g1 * self.group_size, self.n)

    def phase1(self, g0: int, g1: int):
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_phase1(self._h, g0, g1, _stream(self.stream)))

    def export_rows(self, v0: int, v1: int):
        """(ids [m, d_max], dists, pids [m, d_min], pdists) of vertices [v0, v1)."""
        m = v1 - v0
        kw = dict(device=self.device)
        out = (torch.empty((m, self.d_max), dtype=torch.int32, **kw),
               torch.empty((m, self.d_max), dtype=torch.float32, **kw),
               torch.empty((m, self.d_min), dtype=torch.int32, **kw),
               torch.empty((m, self.d_min), dtype=torch.float32, **kw))
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_rows(self._h, v0, v1, *(self._p(t) for t in out), 0,
                                         _stream(self.stream)))
        return out

    def import_rows(self, v0: int, v1: int, rows):
        m = v1 - v0
        shapes = ((m, self.d_max), (m, self.d_max), (m, self.d_min), (m, self.d_min))
        dts = (torch.int32, torch.float32, torch.int32, torch.float32)
        for t, shp, dt, nm in zip(rows, shapes, dts, ("ids", "dists", "pids", "pdists")):
            _check_buf(t, shp, dt, True, nm)
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_rows(self._h, v0, v1, *(self._p(t) for t in rows), 1,
                                         _stream(self.stream)))

    def round_search(self, i: int, v0: int, v1: int):
        """New forward rows F of vertices [v0, v1) of P_i: (ids, dists) [v1-v0, d_min]."""
        f = (torch.empty((v1 - v0, self.d_min), dtype=torch.int32, device=self.device),
             torch.empty((v1 - v0, self.d_min), dtype=torch.float32, device=self.device))
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_round_search(self._h, i, v0, v1, self._p(f[0]), self._p(f[1]),
                                                 _stream(self.stream)))
        return f

    def round_apply(self, i: int, f_ids: torch.Tensor, f_dists: torch.Tensor):
        lo, hi = self.group_rows(i, i + 1)
        _check_buf(f_ids, (hi - lo, self.d_min), torch.int32, True, "f_ids")
        _check_buf(f_dists, (hi - lo, self.d_min), torch.float32, True, "f_dists")
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_round_apply(self._h, i, self._p(f_ids), self._p(f_dists),
                                                _stream(self.stream)))

    def finish(self) -> Graph:
        st = (ct.c_uint64 * 4)()
        h = ct.c_void_p()
        with torch.cuda.device(self.device):
            _check(_lib.ganns_build_finish(self._h, _stream(self.stream),
                                           ct.cast(st, ct.POINTER(ct.c_uint64)), ct.byref(h)))
        self._h = None
        g = Graph(h)
        g.build_stats = tuple(int(x) for x in st)
        return g

    def __del__(self):
        try:
            if self._h:
                _lib.ganns_build_abort(self._h)
        except Exception:
            pass


def search(graph: Graph, points: torch.Tensor, queries: torch.Tensor, k: int, l: int,
           e: int = 0, entry: int = 0, stats: bool = False, out=None, stream=None):
    """Batched GANNS search.  Returns (ids int32 [nq,k], dists float32 [nq,k]) on the
    queries' device, plus per-query stats int32 [nq,3] (iterations, distance
    computations, merged entries) when ``stats``."""
    points = _dev_f32(points, "points")
    queries = _dev_f32(queries, "queries")
    _check_index_inputs(graph, points, queries)
    nq = queries.shape[0]
    if out is None:
        ids = torch.empty((nq, k), dtype=torch.int32, device=queries.device)
        dists = torch.empty((nq, k), dtype=torch.float32, device=queries.device)
    else:
        ids, dists = _check_out(out, nq, k, queries.device)
    st = torch.empty((nq, 3), dtype=torch.int32, device=queries.device) if stats else None
    p = _SearchParams(e, entry, ct.c_void_p(st.data_ptr()) if stats else None, None)
    with torch.cuda.device(queries.device):
        _check(_lib.ganns_search_ex(graph.handle, ct.c_void_p(points.data_ptr()),
                                    ct.c_void_p(queries.data_ptr()), nq, k, l, ct.byref(p),
                                    ct.c_void_p(ids.data_ptr()), ct.c_void_p(dists.data_ptr()),
                                    _stream(stream)))
    return (ids, dists, st) if stats else (ids, dists)


def search_host(graph: Graph, points: torch.Tensor, queries: torch.Tensor, k: int, l: int,
                e: int = 0, entry: int = 0, out=None, stream=None):
    """End-to-end search from host memory: ``queries`` is a CPU float32 tensor
    (pin it for copy/compute overlap); results come back in CPU tensors."""
    points = _dev_f32(points, "points")
    if queries.is_cuda or queries.dtype != torch.float32 or queries.dim() != 2:
        raise TypeError("queries must be a 2-D float32 CPU tensor")
    queries = queries.contiguous()
    _check_index_inputs(graph, points, queries)
    nq = queries.shape[0]
    if out is None:
        ids = torch.empty((nq, k), dtype=torch.int32, pin_memory=True)
        dists = torch.empty((nq, k), dtype=torch.float32, pin_memory=True)
    else:
        ids, dists = out
        _check_buf(ids, (nq, k), torch.int32, False, "out[0] (ids)")
        _check_buf(dists, (nq, k), torch.float32, False, "out[1] (dists)")
    p = _SearchParams(e, entry, None, None)
    with torch.cuda.device(points.device):
        _check(_lib.ganns_search_host(graph.handle, ct.c_void_p(points.data_ptr()),
                                      ct.c_void_p(queries.data_ptr()), nq, k, l, ct.byref(p),
                                      ct.c_void_p(ids.data_ptr()), ct.c_void_p(dists.data_ptr()),
                                      _stream(stream)))
    return ids, dists


def search_host_async(index, points: torch.Tensor, queries_host: torch.Tensor, k: int, l: int,
                      scratch, out_host, e: int = 0, stream=None):
    """One batch end to end from pinned HOST buffers, enqueued on ``stream`` without
    synchronising (ganns_search_host_async / ganns_hnsw_search_host_async): H2D of
    the queries into ``scratch[0]`` (device [nq, d]), the search into ``scratch[1:3]``
    (device ids/dists [nq, k]), D2H into ``out_host`` (pinned ids/dists [nq, k]).
    ``index`` is a Graph or an Hnsw.  No buffer may be touched until ``stream``
    has passed the call."""
    points = _dev_f32(points, "points")
    if queries_host.is_cuda or queries_host.dtype != torch.float32 or not queries_host.is_pinned():
        raise TypeError("queries_host must be a pinned float32 CPU tensor")
    ids_h, dists_h = out_host
    if not (ids_h.is_pinned() and dists_h.is_pinned()):
        raise TypeError("out_host must be pinned CPU tensors")
    qd, ids_d, dists_d = scratch
    nq = queries_host.shape[0]
    if queries_host.dim() != 2 or not queries_host.is_contiguous():
        raise TypeError("queries_host must be a contiguous 2-D tensor")
    base = index.base if isinstance(index, Hnsw) else index
    _check_index_inputs(base, points, queries_host)
    d = base.d      # the library copies nq * graph.d floats
    _check_buf(qd, (nq, d), torch.float32, True, "scratch[0] (queries)")
    _check_buf(ids_d, (nq, k), torch.int32, True, "scratch[1] (ids)")
    _check_buf(dists_d, (nq, k), torch.float32, True, "scratch[2] (dists)")
    _check_buf(ids_h, (nq, k), torch.int32, False, "out_host[0] (ids)")
    _check_buf(dists_h, (nq, k), torch.float32, False, "out_host[1] (dists)")
    p = _SearchParams(e, 0, None, None)
    fn = _lib.ganns_hnsw_search_host_async if isinstance(index, Hnsw) else _lib.ganns_search_host_async
    with torch.cuda.device(points.device):
        _check(fn(index.handle, ct.c_void_p(points.data_ptr()),
                  ct.c_void_p(queries_host.data_ptr()), nq, k, l, ct.byref(p),
                  ct.c_void_p(qd.data_ptr()), ct.c_void_p(ids_d.data_ptr()),
                  ct.c_void_p(dists_d.data_ptr()), ct.c_void_p(ids_h.data_ptr()),
                  ct.c_void_p(dists_h.data_ptr()), _stream(stream)))
    return out_host


def merge_topk(shard_ids: torch.Tensor, shard_dists: torch.Tensor, stream=None):
    """K6: [W, nq, k] per-shard lists with GLOBAL ids -> global top-k [nq, k]."""
    W, nq, k = shard_ids.shape
    ids = torch.empty((nq, k), dtype=torch.int32, device=shard_ids.device)
    dists = torch.empty((nq, k), dtype=torch.float32, device=shard_ids.device)
    with torch.cuda.device(shard_ids.device):
        _check(_lib.ganns_merge_topk(ct.c_void_p(shard_ids.contiguous().data_ptr()),
                                     ct.c_void_p(shard_dists.contiguous().data_ptr()), W, nq, k,
                                     ct.c_void_p(ids.data_ptr()), ct.c_void_p(dists.data_ptr()),
                                     _stream(stream)))
    return ids, dists


def offset_ids(ids: torch.Tensor, offset: int, stream=None) -> torch.Tensor:
    """In place: id -> id + offset for every id >= 0."""
    with torch.cuda.device(ids.device):
        _check(_lib.ganns_offset_ids(ct.c_void_p(ids.data_ptr()), ids.numel(), offset,
                                     _stream(stream)))
    return ids


class Hnsw:
    """HNSW index (Section IV-D): upper layers in shuffled ids + layer 0."""

    def __init__(self, handle: ct.c_void_p):
        self._h = handle
        nl = ct.c_int()
        ln = (ct.c_int64 * 16)()
        _check(_lib.ganns_hnsw_info(handle, ct.byref(nl), ct.cast(ln, ct.c_void_p)))
        self.nlayers = nl.value
        self.layer_n = [int(ln[j]) for j in range(nl.value)]
        b = ct.c_void_p()
        _check(_lib.ganns_hnsw_base(handle, ct.byref(b)))
        self.base = Graph(b, owned=False)
        self.build_stats = None

    @property
    def handle(self):
        return self._h

    def layer(self, j: int) -> np.ndarray:
        out = np.empty((self.layer_n[j], self.base.d_max), np.int32)
        _check(_lib.ganns_hnsw_layer(self._h, j, out.ctypes.data_as(ct.c_void_p)))
        return out

    def perm(self) -> np.ndarray:
        out = np.empty(self.layer_n[0], np.int32)
        _check(_lib.ganns_hnsw_perm(self._h, out.ctypes.data_as(ct.c_void_p)))
        return out

    def free(self):
        if self._h:
            self.base._h = None
            _lib.ganns_hnsw_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def build_hnsw(points: torch.Tensor, levels: np.ndarray, metric: str = "l2", degree: int = 32,
               d_min: int = 0, l_build: int = 0, e_build: int = 0, group_size: int = 0,
               stream=None, l_local: int = 0) -> Hnsw:
    """HNSW construction: Algorithm 2 per layer, top-down.  `levels`
    int8 [n] (e.g. ganns_synth.hnsw_levels).  l_local (0 = l_build): list length of
    every layer's Phase-1 searches (R-C13)."""
    points = _dev_f32(points, "points")
    levels = np.ascontiguousarray(levels, dtype=np.int8)
    st = (ct.c_uint64 * 4)()
    p = _BuildParams(d_min, l_build, e_build, group_size, 0, 0, ct.cast(st, ct.POINTER(ct.c_uint64)),
                     l_local)
    h = ct.c_void_p()
    with torch.cuda.device(points.device):
        _check(_lib.ganns_build_hnsw(ct.c_void_p(points.data_ptr()), points.shape[0],
                                     points.shape[1], METRICS[metric], degree,
                                     levels.ctypes.data_as(ct.c_void_p), ct.byref(p),
                                     _stream(stream), ct.byref(h)))
    idx = Hnsw(h)
    idx.build_stats = tuple(int(x) for x in st)
    return idx


def hnsw_search(index: Hnsw, points: torch.Tensor, queries: torch.Tensor, k: int, l: int,
                e: int = 0, stats: bool = False, out=None, stream=None,
                descent_stats: bool = False):
    """Greedy descent of the upper layers, then the GANNS search on layer 0.  With
    ``stats``: layer-0 counters [nq, 3]; with ``descent_stats`` as well: the
    descent's (iterations, distance computations) [nq, 2] appended to the result."""
    points = _dev_f32(points, "points")
    queries = _dev_f32(queries, "queries")
    _check_index_inputs(index.base, points, queries)
    nq = queries.shape[0]
    if out is None:
        ids = torch.empty((nq, k), dtype=torch.int32, device=queries.device)
        dists = torch.empty((nq, k), dtype=torch.float32, device=queries.device)
    else:
        ids, dists = _check_out(out, nq, k, queries.device)
    st = torch.empty((nq, 3), dtype=torch.int32, device=queries.device) if stats else None
    ds = torch.empty((nq, 2), dtype=torch.int32, device=queries.device) if descent_stats else None
    p = _SearchParams(e, 0, ct.c_void_p(st.data_ptr()) if stats else None,
                      ct.c_void_p(ds.data_ptr()) if descent_stats else None)
    with torch.cuda.device(queries.device):
        _check(_lib.ganns_hnsw_search(index.handle, ct.c_void_p(points.data_ptr()),
                                      ct.c_void_p(queries.data_ptr()), nq, k, l, ct.byref(p),
                                      ct.c_void_p(ids.data_ptr()), ct.c_void_p(dists.data_ptr()),
                                      _stream(stream)))
    res = (ids, dists, st) if stats else (ids, dists)
    return res + (ds,) if descent_stats else res


def build_knn(points: torch.Tensor, init: np.ndarray, K: int, metric: str = "l2",
              max_iters: int = 30, stream=None):
    """KNN graph by neighbours-of-neighbours iterations.  `init` int32
    [n, K] random lists (e.g. ganns_synth.random_graph(n, K, seed)).  Returns
    (Graph, iterations, lists changed in the last iteration)."""
    points = _dev_f32(points, "points")
    init = np.ascontiguousarray(init, dtype=np.int32)
    h = ct.c_void_p()
    it, ch = ct.c_int(), ct.c_int64()
    with torch.cuda.device(points.device):
        _check(_lib.ganns_build_knn(ct.c_void_p(points.data_ptr()), points.shape[0],
                                    points.shape[1], METRICS[metric], K,
                                    init.ctypes.data_as(ct.c_void_p), max_iters, _stream(stream),
                                    ct.byref(h), ct.byref(it), ct.byref(ch)))
    return Graph(h), it.value, ch.value
