#!/usr/bin/env python
"""bench.py -- queries/sec at recall@10 = 0.95 on SIFT1M-shaped data (BASELINE.json
configs[1]), plus GGraphCon NSW build seconds, on N B200s.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl ours|reference]

One step = one ganns_search launch over a whole 10K-query batch at the fastest
(l, e) of the sweep whose recall@10 >= 0.95 -- the whole hot path (candidate
locating, adjacency gather, bulk distance, lazy check, sort, merge, top-k out)
in one fused kernel.  Steps are back-to-back batches issued alternately on two
CUDA streams (the streamed multi-batch pipeline), so the
drain tail of one batch overlaps the start of the next.  They rotate over
--batches distinct query batches (no step re-reads its predecessor's queries'
rows from L2); the working set (vectors + graph) is larger than the 126 MB L2, so
L2 is not flushed.  Inputs are resident in HBM when the timed region starts.
Under torchrun each rank builds the same deterministic graph; by default
each step's fixed 10K-query batch is split over the ranks (strong scaling through
dist.search_replicated, no data-path collective); --scaling weak gives every rank its
own batches.  Time = max over ranks.

--impl reference times the CPU oracle (oracle/, plain C, all host cores) on a
bounded sample of the same queries, same graph, same l.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import ganns_synth as syn  # noqa: E402

L_SWEEP = [32, 40, 48, 56, 64, 72, 80, 88, 96, 104, 112, 120, 128, 144, 160, 192, 224, 256, 288,
           320, 352, 384, 448, 512]


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--target", type=float, default=0.95)
    ap.add_argument("--l-build", type=int, default=128,
                    help="candidate-list length of the build searches (P:222: 32/64/128)")
    ap.add_argument("--l-local", type=int, default=32,
                    help="list length of the Phase-1 (local graph) build searches, <= l_build "
                         "(R-C13; 0 = l_build); not used by the HNSW config")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--json-out", default=None)
    ap.add_argument("--batches", type=int, default=4,
                    help="distinct query batches the steps rotate over")
    ap.add_argument("--streams", type=int, default=2,
                    help="CUDA streams the steps alternate over (1 = serialised launches)")
    ap.add_argument("--shard-rows", type=int, default=0,
                    help="C5 only: rows per shard (default: n / shards = 12.5M)")
    ap.add_argument("--scaling", default="strong", choices=["weak", "strong"],
                    help="strong (default, SURVEY 8(e)): each step's fixed 10K batch is split "
                         "over the ranks (dist.search_replicated / query_slice); weak: every "
                         "rank searches its own batches")
    ap.add_argument("--proxy-worlds", default="2,4,8",
                    help="N=1 only: strong-scaling proxy -- time each of the W slices of the "
                         "fixed batch alone on this GPU (max over slices), per W")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            m = json.load(f)
        return float(m["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """SM clock + throttle reasons sampled through NVML every ~2 ms while the timed
    region runs (the recipe's nvidia-smi clocks line, at a rate that resolves a
    region of tens of milliseconds)."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "sw_power_cap": 0x4}

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.stop = threading.Event()
        self.max_mhz = None

    def sample_now(self):
        """One sample from the calling thread (bench loops call it between timed
        steps, so a short timed region still has samples)."""
        if getattr(self, "h", None) is None:
            return
        import pynvml as nv
        try:
            sm = float(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
            rs = int(nv.nvmlDeviceGetCurrentClocksEventReasons(self.h))
        except Exception:
            return
        self.samples.append((sm, rs))

    def _run(self):
        fails = 0
        while not self.stop.is_set() and fails < 100:
            n = len(self.samples)
            self.sample_now()
            fails += len(self.samples) == n   # a failed NVML read: retry, give up after 100
            time.sleep(0.002)

    def __enter__(self):
        self.h, self.t = None, None
        try:
            import pynvml as nv
            nv.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            if vis:
                self.index = int(vis.split(",")[self.index])
            self.h = nv.nvmlDeviceGetHandleByIndex(self.index)
            self.max_mhz = float(nv.nvmlDeviceGetMaxClockInfo(self.h, nv.NVML_CLOCK_SM))
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception:
            self.t = None
        return self

    def __exit__(self, *a):
        self.stop.set()
        if self.t:
            self.t.join(timeout=2)

    def summary(self):
        sm = [s for s, _ in self.samples]
        reasons = sorted({n for _, r in self.samples for n, bit in self.REASONS.items() if r & bit})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_mhz,
                "reasons": reasons, "samples": len(sm)}


SHAPES = {"C1": "SIFT-shaped", "C2": "SIFT1M-shaped", "C3": "GIST1M-shaped",
          "C4": "GloVe-200-shaped", "C5": "DEEP-shaped"}


def workload_name(cfg, kind):
    return (f"{cfg.name}: {SHAPES[cfg.name]} {cfg.n}x{cfg.d} {cfg.metric}, {kind} degree "
            f"{cfg.degree}")


def make_workload(cfg, rank: int, batches: int = 1):
    """Points and `batches` query batches of cfg.nq for this rank; rank 0's first
    batch is the config's query set (the operating point and the oracle's sample
    use it)."""
    X = syn.points(cfg)
    if cfg.metric == "cosine":
        X = syn.normalize_rows(X)   # input preparation: unit rows (Table I "Cosine")
    # every rank draws its own batches of nq queries (weak scaling)
    first = rank * batches
    Qall = syn.queries(cfg, cfg.nq * (first + batches))
    Qs = [np.ascontiguousarray(Qall[(first + b) * cfg.nq:(first + b + 1) * cfg.nq])
          for b in range(batches)]
    return (X, Qs[0]) if batches == 1 else (X, Qs)


def ground_truth(torch, Xd, Qd, k, metric="l2", with_dist=False):
    """Exact top-k by (dist, id) on the GPU in fp64 (bench-side measurement only).
    L2 on integer-grid data: every fp64 term is an exact integer, and the key
    dist * 2^21 + id (exact below 2^53) breaks ties by id.  IP / cosine (unit
    rows): ranking by -<q, x>."""
    n = Xd.shape[0]
    Xd64, Qd64 = Xd.double(), Qd.double()
    best_k = best_i = None
    shift = float(1 << max(21, int(n - 1).bit_length()))   # > every id: exact (dist, id) key
    for a in range(0, n, 65536):
        b = min(n, a + 65536)
        dot = Qd64 @ Xd64[a:b].T
        if metric == "l2":
            D = (Qd64 ** 2).sum(1)[:, None] + (Xd64[a:b] ** 2).sum(1)[None, :] - 2.0 * dot
            key = D * shift + torch.arange(a, b, device=Xd.device, dtype=torch.float64)[None, :]
        else:
            key = -dot
        kk, ki = torch.topk(key, k, dim=1, largest=False, sorted=True)
        ki = ki + a
        if best_k is None:
            best_k, best_i = kk, ki
        else:
            ck, ci = torch.cat([best_k, kk], 1), torch.cat([best_i, ki], 1)
            best_k, pos = torch.topk(ck, k, dim=1, largest=False, sorted=True)
            best_i = torch.gather(ci, 1, pos)
    if with_dist:
        dist = torch.floor(best_k / shift) if metric == "l2" else best_k
        return best_i.int(), dist
    return best_i.int()


class BenchIndex:
    """The index a config is benchmarked on: the NSW graph of Algorithm 2, or --
    for the GloVe-shaped config (BASELINE configs[3]) -- the HNSW-style graph of
    Section IV-D with seeded levels."""

    def __init__(self, g, cfg, Xd, l_build, l_local=0):
        self.g, self.cfg, self.Xd = g, cfg, Xd
        self.hnsw = cfg.name == "C4"
        if self.hnsw:
            levels = syn.hnsw_levels(Xd.shape[0], cfg.degree // 2, 1)
            self.idx = g.build_hnsw(Xd, levels, metric=cfg.metric, degree=cfg.degree,
                                    l_build=l_build, l_local=min(l_local, l_build))
            self.graph = self.idx.base
            self.build_stats = self.idx.build_stats
        else:
            self.idx = None
            self.graph = g.build(Xd, metric=cfg.metric, degree=cfg.degree, l_build=l_build,
                                 l_local=min(l_local, l_build))
            self.build_stats = self.graph.build_stats
        self.kind = "HNSW-style (Section IV-D)" if self.hnsw else "NSW (Algorithm 2)"

    def search(self, Q, k, l, e=0, stats=False, out=None):
        if self.hnsw:
            return self.g.hnsw_search(self.idx, self.Xd, Q, k, l, e=e, stats=stats, out=out)
        return self.g.search(self.graph, self.Xd, Q, k, l, e=e, stats=stats, out=out)

    def search_host(self, torch, Qh, k, l, e, out):
        """End to end from pinned host buffers through the public API."""
        if not self.hnsw:
            return self.g.search_host(self.graph, self.Xd, Qh, k, l, e=e, out=out)
        Qd = Qh.to(self.Xd.device, non_blocking=True)
        ids, dists = self.search(Qd, k, l, e=e)
        out[0].copy_(ids, non_blocking=True)
        out[1].copy_(dists, non_blocking=True)
        torch.cuda.current_stream().synchronize()
        return out

    def oracle_search(self, X, Q, k, l, e, threads):
        """The oracle on the same graph: (ids, dists, stats [iters, comps, drops,
        merged]).  The HNSW oracle search is single-threaded."""
        import oracle
        if not self.hnsw:
            if not hasattr(self, "_adj"):
                self._adj = self.graph.adjacency()
            return oracle.search(self._adj, X, Q, k, l, e=e, metric=self.cfg.metric,
                                 threads=threads, stats=True)
        h = self._oracle_index()
        ids, dists, _, st = oracle.hnsw_search(h, X, Q, k, l, e=e, metric=self.cfg.metric,
                                               stats=True)
        return ids, dists, st

    def descent_stats(self, Qd, k, l, e):
        """HNSW: per query (iterations, distance computations) of the greedy descent
        through the upper layers (R-H1), counted by the fused kernel itself."""
        return self.g.hnsw_search(self.idx, self.Xd, Qd, k, l, e=e, stats=True,
                                  descent_stats=True)[3]

    def _oracle_index(self):
        if not hasattr(self, "_oi"):
            import numpy as _np
            ups = {j: self.idx.layer(j) for j in range(1, self.idx.nlayers)}
            flat = _np.concatenate([ups[j].reshape(-1) for j in range(1, self.idx.nlayers)]) \
                if ups else _np.zeros(1, _np.int32)
            self._oi = dict(perm=self.idx.perm(), layer_n=_np.array(self.idx.layer_n, _np.int64),
                            upper=ups, layer0=self.idx.layer(0), upper_flat=flat)
        return self._oi


class Pipeline:
    """Back-to-back search steps, step i on stream i % S over batch i % B (the
    streamed multi-batch pipeline): the drain tail of a batch overlaps
    the start of the next one.  Device-timed with CUDA events bracketing all
    streams."""

    def __init__(self, torch, index, Qds, k, nstreams, lo=0, hi=None, replicated=False):
        """replicated: the steps go through dist.search_replicated (each rank searches
        its query_slice of the full batch); otherwise the [lo, hi) slice directly."""
        self.torch, self.index, self.k = torch, index, k
        hi = Qds[0].shape[0] if hi is None else hi
        self.replicated = replicated
        self.Qds = Qds if replicated else [q[lo:hi] for q in Qds]   # this rank's slice
        nq = hi - lo
        dev = Qds[0].device
        self.streams = [torch.cuda.Stream(device=dev) for _ in range(max(1, nstreams))]
        self.outs = [(torch.empty((nq, k), dtype=torch.int32, device=dev),
                      torch.empty((nq, k), dtype=torch.float32, device=dev))
                     for _ in self.streams]

    def _bracket(self, body, clk=None):
        torch = self.torch
        cur = torch.cuda.current_stream()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(cur)
        for st in self.streams:
            st.wait_event(e0)
        body()
        for st in self.streams:
            ev = torch.cuda.Event()
            ev.record(st)
            cur.wait_event(ev)
        e1.record(cur)
        while clk is not None and not e1.query():
            clk.sample_now()   # the steps are running on the device
            time.sleep(0.001)
        e1.synchronize()
        return e0.elapsed_time(e1) / 1e3

    def run(self, steps, l, e, clk=None):
        """Seconds for `steps` steps (device time, all streams)."""
        torch, S = self.torch, len(self.streams)

        def body():
            for i in range(steps):
                with torch.cuda.stream(self.streams[i % S]):
                    out = self.outs[i % S]
                    if self.replicated:
                        from paper_conf_icde_yuwzqzl22_b200 import dist as gdist
                        gdist.search_replicated(
                            lambda q: self.index.search(q, self.k, l, e=e, out=out),
                            self.Qds[i % len(self.Qds)], gather=False)
                    else:
                        self.index.search(self.Qds[i % len(self.Qds)], self.k, l, e=e, out=out)
        return self._bracket(body, clk)

    def run_host(self, g, Xd, Qhs, steps, l, e):
        """Wall seconds for `steps` end-to-end steps through ganns_search_host_async:
        H2D of the batch from pinned host memory, search, D2H of ids + dists, each
        step on its stream; synchronised at the end."""
        torch, S = self.torch, len(self.streams)
        if not hasattr(self, "scratch"):
            nq, d = Qhs[0].shape
            dev = Xd.device
            self.scratch = [(torch.empty((nq, d), dtype=torch.float32, device=dev),
                             torch.empty((nq, self.k), dtype=torch.int32, device=dev),
                             torch.empty((nq, self.k), dtype=torch.float32, device=dev))
                            for _ in range(S)]
            self.hout = [(torch.empty((nq, self.k), dtype=torch.int32).pin_memory(),
                          torch.empty((nq, self.k), dtype=torch.float32).pin_memory())
                         for _ in range(S)]
        obj = self.index.idx if self.index.hnsw else self.index.graph
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for i in range(steps):
            g.search_host_async(obj, Xd, Qhs[i % len(Qhs)], self.k, l, self.scratch[i % S],
                                self.hout[i % S], e=e, stream=self.streams[i % S])
        for st in self.streams:
            st.synchronize()
        return time.perf_counter() - t0


def recall_at(ids, gt):
    k = gt.shape[1]
    hit = (ids[:, :, None] == gt[:, None, :]).any(2).sum()
    return float(hit) / (k * gt.shape[0])


def select_operating_point(torch, index, Qd, gt, k, target, timer):
    """(l, e) sweep: recall@10 of every pair over the queries Qd; among the pairs
    reaching `target` the fastest (timer(l, e) -> seconds) is the operating point.
    e (explore budget) is the paper's fine-grained speed/accuracy knob."""
    sweep, chosen, feasible = [], {}, []
    timed = timer

    for l in L_SWEEP:
        best_r = 0.0
        es = {l, max(k, int(round(0.92 * l))), max(k, int(round(0.85 * l))),
              max(k, int(round(0.7 * l)))}
        if len(feasible) >= 6:
            es = {l}   # only looking for the 0.99 operating point now
        for e in sorted(es, reverse=True):
            ids, _ = index.search(Qd, k, l, e=e)
            r = recall_at(ids, gt)
            sweep.append((l, e, round(r, 5)))
            best_r = max(best_r, r)
            for tgt in (0.9, 0.95, 0.99):
                if r >= tgt and tgt not in chosen:
                    chosen[tgt] = (l, e)
            if r >= target:
                feasible.append((l, e))
        if best_r >= 0.99 or (len(feasible) >= 6 and 0.99 in chosen):
            break
    # per recall target, the cheapest pair reaching it (fewest explorations e, then l)
    for tgt in list(chosen):
        _, l_c, e_c = min((e_, l_, e_) for l_, e_, r_ in sweep if r_ >= tgt)
        chosen[tgt] = (l_c, e_c)
    if not feasible:
        return L_SWEEP[-1], L_SWEEP[-1], sweep, chosen
    _, l_star, e_star = min((timed(l, e), l, e) for l, e in feasible[:6])
    chosen[target] = (l_star, e_star)
    return l_star, e_star, sweep, chosen


def dram_counters_usable():
    """The CUPTI profiler cannot be shared with ncu / nsys, which inject themselves
    through CUDA_INJECTION64_PATH (e.g. the launch-list pass under ncu)."""
    return not os.environ.get("CUDA_INJECTION64_PATH")


def measure_dram(run, device):
    """DRAM traffic of run() (which enqueues work and synchronises) from the
    hardware counters: CUPTI range profiler, one pass, user range (tools/dramprof),
    so the kernels run exactly as in the timed pass -- concurrent streams included."""
    if not dram_counters_usable():
        return {"error": "another profiler is attached (CUDA_INJECTION64_PATH)"}
    from tools.dramprof import DramRegion
    with DramRegion(device) as r:
        secs = run()
    if r.read_bytes is None:
        return {"error": r.error}
    return {"read": r.read_bytes, "write": r.write_bytes,
            "l2_read": r.l2_read_sectors * 32.0, "seconds": secs}


def read_peak_gbps(torch, dev, gib=2):
    """Read-only DRAM bandwidth of a torch reduction over `gib` GiB (context for the
    copy peak of MEASURED_PEAKS.json, which mixes reads and writes; the search
    traffic is > 99.9 % reads)."""
    x = torch.ones((gib << 28,), dtype=torch.float32, device=dev)
    best = None
    for _ in range(6):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        x.sum()
        e1.record()
        e1.synchronize()
        t = e0.elapsed_time(e1) / 1e3
        best = t if best is None else min(best, t)
    gbps = x.numel() * 4 / best / 1e9
    del x
    torch.cuda.empty_cache()
    return round(gbps, 1)


def roofline(alg_bytes, launch_s, dram, launches, peak, peak_kind, kernel, duration):
    """The line's roofline object.  `achieved` / `frac` / `traffic` are DRAM bytes
    measured by the hardware counters over `launches` launches of the timed
    configuration, per launch, over the launch duration of the timed pass.  The
    SURVEY §8(d) algorithmic bytes (every gathered row, lazy-check re-reads
    included) are reported beside them: rows served by the 126 MB L2 count
    there too, so alg_frac is an L2-level figure and can exceed 1."""
    alg = alg_bytes / launch_s / 1e9
    r = {"bound": "hbm", "peak": peak, "unit": "GB/s", "peak_kind": peak_kind, "kernel": kernel,
         "duration": duration, "alg_bytes_per_launch": int(alg_bytes), "alg_GBps": round(alg, 1),
         "alg_frac": round(alg / peak, 4),
         "alg_note": "SURVEY 8(d) algorithmic bytes incl. lazy-check re-reads (P:191); "
                     "L2-served rows count, so this is an L2-level figure"}
    if "error" not in dram:
        per = (dram["read"] + dram["write"]) / launches
        ach = per / launch_s / 1e9
        r.update(achieved=round(ach, 1), frac=round(ach / peak, 4), traffic=int(per),
                 traffic_read=int(dram["read"] / launches),
                 traffic_write=int(dram["write"] / launches),
                 l2_read_bytes_per_launch=int(dram["l2_read"] / launches),
                 dram_over_alg=round(per / alg_bytes, 4),
                 achieved_kind="measured DRAM bytes per launch / launch duration",
                 traffic_source=(f"hardware counters dram__bytes_read.sum + dram__bytes_write.sum "
                                 f"(CUPTI range profiler, one pass) over {launches} launches of "
                                 f"the timed configuration in this run"),
                 profiled_pass_s=round(dram["seconds"], 6))
    else:
        r.update(achieved=round(alg, 1), frac=round(alg / peak, 4), traffic=None,
                 achieved_kind=f"algorithmic (DRAM counters unavailable: {dram['error']})")
    # also against the B200 HBM3e specification (~8 TB/s)
    r["frac_of_spec_8TBps"] = round(r["achieved"] / 8000.0, 4)
    return r


def build_phase_split(torch, g, cfg, Xd, l_build, l_local):
    """Phase 1 and the serial Phase-2 rounds of Algorithm 2 timed apart on
    the GPU clock -- one extra build through the staged ABI (ganns_build_begin ...,
    the same kernels; a round's searches then write F and an apply kernel writes the
    rows), CUDA events around Phase 1 and around all rounds."""
    b = g.StagedBuild(Xd, metric=cfg.metric, degree=cfg.degree, l_build=l_build,
                      l_local=min(l_local, l_build))
    _, G, _, _ = b.info()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    ev[0].record()
    b.phase1(0, G)
    ev[1].record()
    for i in range(1, G):
        v0, v1 = b.group_rows(i, i + 1)
        b.round_apply(i, *b.round_search(i, v0, v1))
    ev[2].record()
    ev[2].synchronize()
    gr = b.finish()
    del gr
    p1, p2 = ev[0].elapsed_time(ev[1]) / 1e3, ev[1].elapsed_time(ev[2]) / 1e3
    return {"phase1_s": round(p1, 4), "phase2_s": round(p2, 4), "rounds": G - 1,
            "round_ms_mean": round(p2 / max(1, G - 1) * 1e3, 4),
            "method": "staged ABI, CUDA events on the build's stream (GPU clock)"}


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def parity_report(gpu, ora, exact, gt=None):
    """Element-by-element comparison of the GPU's results with the oracle's on the
    same queries, graph and (l, e).  gpu = (ids, dists, stats[iters, comps,
    merged]); ora = (ids, dists, stats[iters, comps, drops, merged]).  exact
    (integer grid): ids, dists and counters bit-identical.  Otherwise (cosine):
    |d_gpu - d_ora| <= 1e-5 |d| + 1e-6, id sets >= 99.8 % equal and
    recall within 0.002 (BASELINE north star)."""
    gi, gd, gs = gpu
    oi, od, os_ = ora
    fin = np.isfinite(od) & np.isfinite(gd)
    diff = np.abs(gd.astype(np.float64) - od.astype(np.float64))
    rel = np.where(fin, diff / np.maximum(np.abs(od.astype(np.float64)), 1e-30), 0.0)
    same_inf = (np.isfinite(od) == np.isfinite(gd)).all()
    agree = float(np.mean([len(set(a.tolist()) & set(b.tolist())) / len(a) for a, b in zip(gi, oi)]))
    rep = {"queries": int(len(gi)), "ids_equal": bool((gi == oi).all()),
           "dists_equal": bool((gd == od).all()),
           "max_rel_err": float(rel.max()) if rel.size else 0.0,
           "counters_equal": bool(gs is not None and os_ is not None and
                                  (gs[:, 0] == os_[:, 0]).all() and (gs[:, 1] == os_[:, 1]).all()
                                  and (gs[:, 2] == os_[:, 3]).all()),
           "id_agreement": round(agree, 6)}
    if gt is not None:
        rg, ro = recall_at_np(gi, gt), recall_at_np(oi, gt)
        rep.update(recall_gpu=round(rg, 5), recall_oracle=round(ro, 5),
                   recall_diff=round(abs(rg - ro), 5))
    if exact:
        rep["bar"] = "bit-exact ids, dists and counters (integer grid, R-C18)"
        rep["ok"] = rep["ids_equal"] and rep["dists_equal"] and rep["counters_equal"]
    else:
        tol_ok = bool(same_inf and (diff[fin] <= 1e-5 * np.abs(od[fin]) + 1e-6).all())
        rep["bar"] = "|dd| <= 1e-5|d| + 1e-6, id agreement >= 0.998, recall within 0.002"
        rep["dists_within_tol"] = tol_ok
        rep["ok"] = tol_ok and agree >= 0.998 and rep.get("recall_diff", 0.0) <= 0.002
    return rep


def recall_at_np(ids, gt):
    k = gt.shape[1]
    return float((ids[:, :, None] == gt[:, None, :]).any(2).sum()) / (k * gt.shape[0])


def gt_check(X, Q, gt, k, metric, nq):
    """K8: the bench's fp64 GPU ground truth against the oracle's
    brute force (O6, pinned by numpy lexsort) on the first nq queries."""
    import oracle
    t0 = time.perf_counter()
    oi, _ = oracle.bruteforce(X, Q[:nq], k, metric=metric, threads=oracle.ncores())
    g = gt[:nq]
    return {"queries": int(nq), "ids_equal": bool((oi == g).all()),
            "ids_equal_frac": round(float((oi == g).mean()), 6),
            "oracle_s": round(time.perf_counter() - t0, 2),
            "note": "exact on the integer grid (L2); cosine ranks by -<q,x> in fp64 vs the "
                    "oracle's fp32 distance, so near-ties may order differently"}


def streams_for(nq_rank, base):
    """Streams for back-to-back batches of nq_rank queries: enough batches in flight
    to cover the resident warp slots (~3.5K per B200 at d <= 128) twice."""
    return max(base, min(8, -(-2 * 3552 // max(1, nq_rank))))


def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_icde_yuwzqzl22_b200 as g
    from paper_conf_icde_yuwzqzl22_b200 import dist as gdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    distributed = "RANK" in os.environ          # launched by torchrun (any world size)
    if distributed:
        torch.cuda.set_device(local)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    cfg = syn.CONFIGS[args.config]
    k = cfg.k
    strong = args.scaling == "strong"

    B = max(1, args.batches)
    # weak: every rank draws its own batches; strong: every rank sees the same global
    # batches and searches its slice of each (dist.query_slice)
    X, Qs = make_workload(cfg, 0 if strong else rank, B)
    Qs = Qs if isinstance(Qs, list) else [Qs]
    Q = Qs[0]
    nq = Q.shape[0]
    lo, hi = gdist.query_slice(nq, rank, world) if strong else (0, nq)
    Xd = torch.from_numpy(X).to(dev)
    Qd_all = torch.from_numpy(np.concatenate(Qs)).to(dev)
    Qds = [Qd_all[b * nq:(b + 1) * nq] for b in range(B)]
    torch.cuda.synchronize()

    # exact ground truth first: it also brings the GPU out of its idle clocks before
    # the timed build
    gt = ground_truth(torch, Xd, Qd_all, k, cfg.metric)
    # untimed warm-up build on a 20K-point prefix (loads the build kernels' modules)
    BenchIndex(g, cfg, Xd[:20000].contiguous(), args.l_build, args.l_local)
    torch.cuda.synchronize()

    # ---- GGraphCon build (wall clock on device-resident points; median of 3 builds,
    # the builds are deterministic, the last one is searched)
    build_all = []
    for _ in range(3):
        index = None
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        index = BenchIndex(g, cfg, Xd, args.l_build, args.l_local)
        torch.cuda.synchronize()
        build_all.append(time.perf_counter() - t0)
    build_s = statistics.median(build_all)
    b_iters, b_comps, b_searches, b_rounds = index.build_stats
    phase_split = None if index.hnsw else build_phase_split(torch, g, cfg, Xd, args.l_build,
                                                            args.l_local)

    # ---- (l, e) operating point over every query the timed steps search (see
    # select_operating_point); candidates timed as the steps are (pipelined)
    nstreams = streams_for(hi - lo, args.streams) if strong else args.streams
    pipe = Pipeline(torch, index, Qds, k, nstreams, lo, hi, replicated=strong and distributed)
    l_star, e_star, sweep, chosen = select_operating_point(
        torch, index, Qd_all, gt, k, args.target,
        lambda l, e: min(pipe.run(3 * B, l, e) for _ in range(3)))
    ids, dists, st = index.search(Qd_all, k, l_star, e=e_star, stats=True)
    rec = recall_at(ids, gt)
    st = st.long()
    d = cfg.d
    # algorithmic bytes: query + per iteration the adjacency row + every
    # computed distance's vector row (entry and lazy-check re-computations) +
    # the top-k written; HNSW adds the descent's rows (the kernel's descent counters)
    per_q = 4 * d + 4 * cfg.degree * st[:, 0] + 4 * d * st[:, 1] + 8 * k
    if index.hnsw:   # + the descent's adjacency rows and the permuted rows it gathers
        ds = index.descent_stats(Qd_all, k, l_star, e_star).long()
        per_q = per_q + 4 * cfg.degree * ds[:, 0] + 4 * d * ds[:, 1]
    # per step = the mean over the batches of this rank's slice
    sl = torch.cat([per_q[b * nq + lo:b * nq + hi] for b in range(B)])
    alg_bytes = int(sl.sum().item()) // B
    iters_mean = float(st[:, 0].float().mean())

    # ---- timed steps: device-resident inputs, back-to-back batches on the streams
    pipe.run(args.warmup, l_star, e_star)
    torch.cuda.synchronize()
    launches0 = g.kernel_launches()
    if distributed:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_total = pipe.run(args.steps, l_star, e_star, clk)
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    launches = g.kernel_launches() - launches0
    t_max = torch.tensor([t_total], dtype=torch.float64, device=dev)
    if distributed:
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
    t_total = float(t_max.item())
    total_queries = nq * args.steps * (1 if strong else world)
    qps = total_queries / t_total
    ms_per_step = t_total / args.steps * 1e3
    launch_s = t_total / args.steps

    # ---- DRAM bytes of the same steps (hardware counters, untimed second pass)
    dram = measure_dram(lambda: pipe.run(args.steps, l_star, e_star), local)

    # ---- the other recall targets of SURVEY §8(d) (0.9, 0.99): same pipelined steps
    at_recall = {}
    for tgt in (0.9, 0.95, 0.99):
        le = chosen.get(tgt)
        if le is None:
            at_recall[str(tgt)] = None
            continue
        if tgt == args.target:
            le, tq = (l_star, e_star), qps
        else:
            tq = total_queries / pipe.run(args.steps, le[0], le[1])
        rr = next(r for l_, e_, r in sweep if (l_, e_) == tuple(le))
        at_recall[str(tgt)] = {"l": le[0], "e": le[1], "recall": rr, "qps": round(tq, 1)}

    # ---- strong-scaling proxy on one GPU (replicated graph): the time
    # of K steps over each rank's slice of the fixed batch, max over the W slices
    proxy = None
    if world == 1 and args.proxy_worlds:
        proxy = {}
        for W in [int(w) for w in args.proxy_worlds.split(",") if w]:
            ts = []
            for r in range(W):
                a, b = gdist.query_slice(nq, r, W)
                pw = Pipeline(torch, index, Qds, k, streams_for(b - a, args.streams), a, b)
                pw.run(args.warmup, l_star, e_star)
                ts.append(pw.run(args.steps, l_star, e_star))
            tq = nq * args.steps / max(ts)
            proxy[str(W)] = {"queries_per_gpu": nq // W, "streams": streams_for(nq // W, args.streams),
                             "implied_qps": round(tq, 1),
                             "per_gpu_efficiency": round(tq / (W * qps), 4)}

    # ---- end to end through the public API (ganns_search_host_async) from pinned
    # host buffers: every step copies its batch (slice) in and its ids + dists out
    Qhs = [torch.from_numpy(np.ascontiguousarray(q[lo:hi])).pin_memory() for q in Qs]
    pipe.run_host(g, Xd, Qhs, max(2, args.warmup), l_star, e_star)
    e2e_t = torch.tensor([pipe.run_host(g, Xd, Qhs, args.steps, l_star, e_star)],
                         dtype=torch.float64, device=dev)
    if distributed:
        dist.all_reduce(e2e_t, op=dist.ReduceOp.MAX)
    e2e_qps = total_queries / float(e2e_t.item())

    peak, peak_kind = peaks()
    line = {
        "metric": "queries/sec at recall@10=0.95",
        "value": round(qps, 1),
        "unit": "queries/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(ms_per_step, 4),
        "higher_is_better": True,
        "scaling": "strong" if strong else "weak",
        "vs_baseline": None,
        "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": workload_name(cfg, index.kind) + (
                       f", {nq} queries per step split over {world} GPU(s), k={k}" if strong else
                       f", {nq} queries/GPU, k={k}"),
                   "l": l_star, "e": e_star, "recall_at_10": round(rec, 5),
                   "recall_over": f"all {B * nq} queries of the {B} batches",
                   "selection": "fastest (l, e) with recall@10 >= target among the sweep",
                   "le_for_recall": {str(t): chosen.get(t) for t in (0.9, 0.95, 0.99)},
                   "le_sweep_recall": sweep, "mean_iterations": round(iters_mean, 2),
                   "qps_at_recall": at_recall,
                   "batches": B, "streams": len(pipe.streams),
                   "l2": (f"not flushed: inputs larger than L2 ({(X.nbytes + cfg.n * cfg.degree * 4) >> 20}"
                          f" MiB vectors + graph vs 126 MB); steps rotate over {B} distinct "
                          f"{nq}-query batches"),
                   "parallelism": (f"replicated graph, fixed batch split over {world} rank(s)"
                                   if strong else f"replicated graph, query data-parallel x{world}")},
        "build_seconds": round(build_s, 4),
        "build_seconds_all": [round(x, 4) for x in build_all],
        "build_params": {"degree": cfg.degree, "d_min": cfg.degree // 2, "l_build": args.l_build,
                         "l_local": min(args.l_local, args.l_build) or args.l_build,
                         "group_size": "auto"},
        "build": {"iterations": b_iters, "distance_computations": b_comps,
                  "searches": b_searches, "rounds": b_rounds,
                  "alg_GBps": round((4 * d * b_comps + 4 * cfg.degree * b_iters) / build_s / 1e9, 1),
                  "phase_split": phase_split},
        "e2e": {"value": round(e2e_qps, 1), "unit": "queries/s",
                "h2d_bytes_per_step": int(Qhs[0].numel() * 4),
                "d2h_bytes_per_step": int((hi - lo) * k * 8),
                "api": "ganns_search_host_async, steps alternating over the streams, wall clock"},
        "gpu_launches": int(launches),
        "roofline": roofline(alg_bytes, launch_s, dram, args.steps, peak, peak_kind,
                             f"ganns::search_kernel (d={cfg.d}, d_max={cfg.degree}, {cfg.metric}"
                             f"{', HNSW descent fused' if index.hnsw else ''})",
                             "timed region / steps (consecutive launches overlap on the streams)"),
        "clocks": clk.summary(),
    }
    if proxy is not None:
        line["config"]["strong_scaling_proxy"] = proxy
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["roofline"]["read_peak_torch_sum_GBps"] = read_peak_gbps(torch, dev)
        gpu_q = (ids[:nq].cpu().numpy(), dists[:nq].cpu().numpy(), st[:nq].cpu().numpy())
        gt_np = gt[:nq].cpu().numpy()
        line["cpu_baseline"], line["parity"] = cpu_baseline(
            index, X, Q, k, l_star, e_star, args.cpu_seconds, gpu_q, gt_np,
            exact=cfg.metric != "cosine")
        line["gt_check"] = gt_check(X, Q, gt_np, k, cfg.metric, 100 if cfg.d <= 256 else 40)
        if not index.hnsw:
            line["cpu_build_baseline"] = cpu_build_baseline(torch, g, cfg, X, args.l_build,
                                                            min(args.l_local, args.l_build))
    if rank == 0:
        s = json.dumps(line)
        print(s, flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(s + "\n")
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


def run_sharded(args):
    """BASELINE configs[4] (DEEP100M-shaped, 100M x 96, 8 shards): every shard is an
    independent NSW (Algorithm 2) over its rows; every query is searched on every
    shard (K1), shard-local ids become global (id offset kernel), the per-shard
    [nq, k] lists are exchanged with one NCCL all_gather_into_tensor and merged by
    K6 (ganns_merge_topk) -- all through dist.ShardedIndex.  Rank r owns the shards
    s = r, r + N, ...; one step = the whole sharded search of the 10K-query batch
    (strong scaling: the total work is fixed)."""
    import torch
    import torch.distributed as dist
    import paper_conf_icde_yuwzqzl22_b200 as g
    from paper_conf_icde_yuwzqzl22_b200 import dist as gdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    distributed = "RANK" in os.environ
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if distributed:
        dist.init_process_group("nccl", device_id=dev)
    cfg = syn.CONFIGS[args.config]
    if args.shard_rows:
        cfg = syn.with_size(cfg, n=args.shard_rows * cfg.shards)
    k, W = cfg.k, cfg.shards
    if W % world != 0:
        raise SystemExit(f"{W} shards do not split evenly over {world} ranks")
    per = cfg.n // W
    mine = [s for s in range(W) if s % world == rank]
    Q = syn.queries(cfg)
    Qd = torch.from_numpy(Q).to(dev)
    nsub = min(1000, len(Q))                 # recall measured on a fixed query subset
    shards, build_s, gt_parts = [], 0.0, []
    # untimed warm-up build (module load, GPU out of idle clocks)
    g.build(torch.from_numpy(syn.points(cfg, 0, 20000)).to(dev), metric=cfg.metric,
            degree=cfg.degree, l_build=args.l_build, l_local=min(args.l_local, args.l_build))
    torch.cuda.synchronize()
    for s in mine:
        Xs = torch.from_numpy(syn.points(cfg, s * per, (s + 1) * per)).to(dev)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        gr = g.build(Xs, metric=cfg.metric, degree=cfg.degree, l_build=args.l_build,
                     l_local=min(args.l_local, args.l_build))
        torch.cuda.synchronize()
        build_s = max(build_s, time.perf_counter() - t0)
        gi_s, gd_s = ground_truth(torch, Xs, Qd[:nsub], k, cfg.metric, with_dist=True)
        gt_parts.append((gi_s.long() + s * per, gd_s))
        shards.append((s, Xs, gr))
    # exact top-k over all shards for the subset: each shard's exact top-k (fp64
    # distances, exact on the integer grid) gathered and merged by (dist, global id)
    cid = torch.cat([p for p, _ in gt_parts], 1)
    cdd = torch.cat([d for _, d in gt_parts], 1)
    if distributed:
        ai = torch.empty((world,) + tuple(cid.shape), dtype=cid.dtype, device=dev)
        ad = torch.empty((world,) + tuple(cdd.shape), dtype=cdd.dtype, device=dev)
        dist.all_gather_into_tensor(ai, cid.contiguous())
        dist.all_gather_into_tensor(ad, cdd.contiguous())
        cid = torch.cat(list(ai), 1)
        cdd = torch.cat(list(ad), 1)
    key = cdd * float(1 << 27) + cid.double()
    kk = torch.topk(key, k, dim=1, largest=False, sorted=True).values
    gt = (kk - torch.floor(kk / float(1 << 27)) * float(1 << 27)).round().int()

    # the shard searches of a step alternate over the streams (their drain tails
    # overlap the next shard's search); the all-gather + merge wait for all of them
    streams = [torch.cuda.Stream(device=dev) for _ in range(max(1, args.streams))]

    def index_at(l):
        return gdist.gpu_sharded_index([(s * per, gr, Xs) for s, Xs, gr in shards], k, l, e=l,
                                       streams=streams)

    chosen, sweep = None, []
    for l in L_SWEEP:
        ids, _ = index_at(l).search(Qd)
        r = recall_at(ids[:nsub], gt)
        sweep.append((l, round(r, 5)))
        if r >= args.target:
            chosen = l
            break
    l_star = chosen or L_SWEEP[-1]
    sidx = index_at(l_star)

    def steps_run(n):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(n):
            out = sidx.search(Qd)
        e1.record()
        e1.synchronize()
        return e0.elapsed_time(e1) / 1e3, out

    steps_run(args.warmup)
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    torch.cuda.synchronize()
    launches0 = g.kernel_launches()
    with ClockSampler(local) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            ids, dists = sidx.search(Qd)
        e1.record()
        while not e1.query():
            clk.sample_now()
            time.sleep(0.002)
        e1.synchronize()
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    launches = g.kernel_launches() - launches0
    t = torch.tensor([e0.elapsed_time(e1) / 1e3], dtype=torch.float64, device=dev)
    if distributed:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    t_total = float(t.item())
    rec = recall_at(ids[:nsub], gt)
    qps = len(Q) * args.steps / t_total
    # DRAM bytes of the same steps (hardware counters, untimed second pass; a
    # collective inside a profiled range is fine -- it is one pass, no replay).  Two
    # steps (16 shard launches): the profiler's stop failed on a 10-step range (0.55 s)
    dsteps = min(2, args.steps)
    dram = measure_dram(lambda: steps_run(dsteps)[0], local)
    # roofline of K1 on the shards (untimed stats pass: the kernel's own counters)
    # per shard launch: the timed region over the launches (they overlap pairwise)
    search_s = t_total / args.steps / max(1, len(shards))
    alg = 0
    for s, Xs, gr in shards:
        _, _, st = g.search(gr, Xs, Qd, k, l_star, e=l_star, stats=True)
        st = st.long()
        alg += int((4 * cfg.d + 4 * cfg.degree * st[:, 0] + 4 * cfg.d * st[:, 1]).sum()) + 8 * k * len(Q)
    alg_per_launch = alg // max(1, len(shards))
    peak, peak_kind = peaks()
    # end to end: queries from pinned host memory, results back to pinned host
    # memory, inside the timed region (the all-gather and merge included)
    Qh = torch.from_numpy(Q).pin_memory()
    Qin = torch.empty_like(Qd)
    hid = torch.empty((len(Q), k), dtype=torch.int32).pin_memory()
    hdd = torch.empty((len(Q), k), dtype=torch.float32).pin_memory()
    e2e = []
    for it in range(args.warmup + args.steps):
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
        t0 = time.perf_counter()
        Qin.copy_(Qh, non_blocking=True)
        i_, d_ = sidx.search(Qin)
        hid.copy_(i_, non_blocking=True)
        hdd.copy_(d_, non_blocking=True)
        torch.cuda.current_stream().synchronize()
        if it >= args.warmup:
            e2e.append(time.perf_counter() - t0)
    te = torch.tensor([sum(e2e)], dtype=torch.float64, device=dev)
    if distributed:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_qps = len(Q) * args.steps / float(te.item())
    line = {
        "metric": "queries/sec at recall@10=0.95", "value": round(qps, 1), "unit": "queries/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(t_total / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": f"{cfg.name}: DEEP-shaped {cfg.n}x{cfg.d} {cfg.metric}, {W} shards x "
                               f"NSW degree {cfg.degree}, {len(Q)} queries, k={k}",
                   "l": l_star, "e": l_star, "recall_at_10": round(rec, 5),
                   "recall_subset": nsub, "l_sweep_recall": sweep,
                   "shards_per_gpu": len(mine),
                   "parallelism": (f"base set sharded, {world} rank(s), dist.ShardedIndex: "
                                   "NCCL all_gather_into_tensor + K6 merge"),
                   "streams": len(streams),
                   "l2": (f"not flushed: inputs larger than L2 ({cfg.n * cfg.d * 4 >> 20} MiB of "
                          "vectors); a shard is re-searched only after the other shards")},
        "build_seconds": round(build_s, 3), "build_note": "max over this run's shards (each built alone)",
        "gpu_launches": int(launches), "clocks": clk.summary(),
        "e2e": {"value": round(e2e_qps, 1), "unit": "queries/s",
                "h2d_bytes_per_step": int(Q.nbytes), "d2h_bytes_per_step": int(len(Q) * k * 8)},
        "roofline": roofline(alg_per_launch, search_s, dram, dsteps * max(1, len(shards)), peak,
                             peak_kind,
                             f"ganns::search_kernel on one {per}-row shard (d={cfg.d}, "
                             f"d_max={cfg.degree}, {cfg.metric}); mean over the shard launches",
                             "timed region / (steps x shards on this GPU)"),
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        line["cpu_baseline"], line["parity"] = sharded_cpu_baseline(
            torch, g, shards, per, Q, k, l_star, args.cpu_seconds, cfg.metric,
            (ids.cpu().numpy(), dists.cpu().numpy()), gt.cpu().numpy())
    if rank == 0:
        print(json.dumps(line), flush=True)
        if args.json_out:
            with open(args.json_out, "w") as f:
                f.write(json.dumps(line) + "\n")
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


def sharded_cpu_baseline(torch, g, shards, per, Q, k, l, seconds, metric, gpu, gt):
    """The oracle's sharded search on a bounded query sample: every shard searched by
    the oracle (plain C, one pthread per host core, same graph and l), then the
    oracle's merge by (dist, global id); compared element by element with the GPU's
    merged result for the same queries.  Host copies of the shards (not timed)."""
    import oracle
    cores = oracle.ncores()
    m = 0
    for s, Xs, gr in shards[:1]:   # calibrate the sample on the first shard
        Xh, A = Xs.cpu().numpy(), gr.adjacency()
        t0 = time.perf_counter()
        oracle.search(A, Xh, Q[:32], k, l, e=l, metric=metric, threads=cores)
        dt = time.perf_counter() - t0
        m = int(min(len(Q), max(32, 32 * seconds / max(dt * len(shards), 1e-3))))
        del Xh, A
    tot, parts = 0.0, []
    for s, Xs, gr in shards:
        Xh, A = Xs.cpu().numpy(), gr.adjacency()
        t0 = time.perf_counter()
        ids, dd = oracle.search(A, Xh, Q[:m], k, l, e=l, metric=metric, threads=cores)
        tot += time.perf_counter() - t0
        parts.append((np.where(ids >= 0, ids + s * per, -1).astype(np.int32), dd))
        del Xh, A
    t0 = time.perf_counter()
    mi, md = oracle.merge_topk(np.stack([p[0] for p in parts]), np.stack([p[1] for p in parts]))
    tot += time.perf_counter() - t0
    gi, gd = gpu
    mm = min(m, len(gt))
    par = parity_report((gi[:m], gd[:m], None), (mi, md, None), exact=True,
                        gt=gt[:mm] if mm == m else None)
    par["counters_equal"] = None   # the merged lists carry no per-shard counters
    par["ok"] = par["ids_equal"] and par["dists_equal"]
    par["bar"] = "bit-exact merged ids and dists (per-shard oracle search + oracle merge)"
    return ({"value": round(m / tot, 1), "unit": "queries/s", "cores": cores, "kind": "oracle",
             "cpu_model": cpu_model(),
             "sample": f"first {m} of the {len(Q)} queries on all {len(shards)} shards "
                       f"(same graphs, l={l}) + merge, {tot:.1f} s"}, par)


def cpu_baseline(index, X, Q, k, l, e, seconds, gpu, gt, exact):
    """The oracle's search (plain C) on a bounded sample of the same queries and
    graph: all host cores (one pthread per core) and one thread (the paper's CPU
    baselines are single-threaded).  Returns (cpu_baseline, parity): the
    oracle's results on the all-core sample compared element by element with the
    GPU's (`gpu` = ids, dists, stats of the batch at the same (l, e))."""
    import oracle
    cores = oracle.ncores()
    m = 64
    t0 = time.perf_counter()
    index.oracle_search(X, Q[:m], k, l, e, cores)
    dt = time.perf_counter() - t0
    m2 = int(min(len(Q), max(m, m * seconds / max(dt, 1e-3))))
    t0 = time.perf_counter()
    oi, od, ost = index.oracle_search(X, Q[:m2], k, l, e, cores)
    dt = time.perf_counter() - t0
    m1 = int(max(8, min(m2, m2 * 3.0 / max(dt * cores, 1e-3))))
    t0 = time.perf_counter()
    index.oracle_search(X, Q[:m1], k, l, e, 1)
    dt1 = time.perf_counter() - t0
    gi, gd, gs = gpu
    par = parity_report((gi[:m2], gd[:m2], gs[:m2]), (oi, od, ost), exact, gt=gt[:m2])
    return ({"value": round(m2 / dt, 1), "unit": "queries/s", "cores": cores, "kind": "oracle",
             "cpu_model": cpu_model(),
             "one_thread": {"value": round(m1 / dt1, 1), "queries": m1, "seconds": round(dt1, 2)},
             "sample": f"first {m2} of the {len(Q)} queries, same graph, l={l}, e={e}, {dt:.1f} s "
                       f"on {cores} threads; {m1} queries on 1 thread"}, par)


def cpu_build_baseline(torch, g, cfg, X, l_build, l_local=0, m=10000):
    """Algorithm 2 on the first m points: the oracle (plain C, one thread -- the paper's
    CPU baselines are single-threaded) and the GPU build of the same sample with
    the same partition (group size 256 = the auto rule at this size), compared
    bit-exact.  The oracle's Algorithm 2 on the full config (all cores) is
    tools/oracle_alg2_full.py (minutes; profiles/r02/oracle_alg2_full_C2.json)."""
    import oracle
    Xs = np.ascontiguousarray(X[:m])
    S = 256
    t0 = time.perf_counter()
    ref, _, _ = oracle.alg2(Xs, cfg.degree // 2, cfg.degree, S, l_build=l_build,
                            metric=cfg.metric, l_local=l_local)
    t_cpu = time.perf_counter() - t0
    Xd = torch.from_numpy(Xs).cuda()
    g.build(Xd, metric=cfg.metric, degree=cfg.degree, l_build=l_build, group_size=S,
            l_local=l_local)  # warm
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    gr = g.build(Xd, metric=cfg.metric, degree=cfg.degree, l_build=l_build, group_size=S,
                 l_local=l_local)
    torch.cuda.synchronize()
    t_gpu = time.perf_counter() - t0
    return {"oracle_s": round(t_cpu, 3), "gpu_s": round(t_gpu, 4), "cores": 1, "kind": "oracle",
            "adjacency_equal": bool((gr.adjacency() == ref).all()),
            "sample": f"Algorithm 2 on the first {m} points (degree {cfg.degree}, "
                      f"l_build {l_build}, l_local {l_local or l_build}, group size {S})"}


def run_reference(args):
    """The oracle timed as it stands (CPU, all host cores) -- the reference arm."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import torch
    import oracle
    import paper_conf_icde_yuwzqzl22_b200 as g
    cfg = syn.CONFIGS[args.config]
    k = cfg.k
    X, Qs = make_workload(cfg, 0, max(1, args.batches))
    Qs = Qs if isinstance(Qs, list) else [Qs]
    Q = Qs[0]
    # index set-up (not timed): the graph the GPU arm searches (deterministic) and
    # the same (l, e) operating point, selected the same way
    Xd = torch.from_numpy(X).cuda()
    index = BenchIndex(g, cfg, Xd, args.l_build, args.l_local)
    Qd = torch.from_numpy(np.concatenate(Qs)).cuda()
    gt = ground_truth(torch, Xd, Qd, k, cfg.metric)
    Qds = [Qd[b * len(Q):(b + 1) * len(Q)] for b in range(len(Qs))]
    pipe = Pipeline(torch, index, Qds, k, args.streams)
    l_star, e_star, _, _ = select_operating_point(
        torch, index, Qd, gt, k, args.target,
        lambda l, e: min(pipe.run(3 * len(Qs), l, e) for _ in range(3)))
    index.oracle_search(X, Q[:2], k, l_star, e_star, 1)   # materialise the host copy
    del Qd, Qds, pipe
    cores = oracle.ncores()
    per_step = 48
    for _ in range(args.warmup):
        index.oracle_search(X, Q[:16], k, l_star, e_star, cores)
    t0 = time.perf_counter()
    index.oracle_search(X, Q[:per_step], k, l_star, e_star, cores)
    dt = time.perf_counter() - t0
    per_step = int(max(cores, min(len(Q), per_step * 6.0 / max(dt, 1e-3))))
    times = []
    for s in range(args.steps):
        a = (s * per_step) % max(1, len(Q) - per_step)
        t0 = time.perf_counter()
        index.oracle_search(X, Q[a:a + per_step], k, l_star, e_star, cores)
        times.append(time.perf_counter() - t0)
    tot = sum(times)
    v = per_step * args.steps / tot
    sample = (f"{per_step} queries/step of the {len(Q)}-query batch, same graph, "
              f"l={l_star}, e={e_star}")
    print(json.dumps({
        "impl": "reference", "metric": "queries/sec at recall@10=0.95", "value": round(v, 1),
        "unit": "queries/s", "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(tot / args.steps * 1e3, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": workload_name(cfg, index.kind) + f", k={k}", "l": l_star,
                   "e": e_star},
        "cpu_baseline": {"value": round(v, 1), "unit": "queries/s", "cores": cores,
                         "kind": "oracle", "sample": sample},
        "e2e": {"value": round(v, 1), "unit": "queries/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    elif syn.CONFIGS[args.config].shards > 1:
        run_sharded(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
