// build_inst.cu (compiled once per NV4 with -DGANNS_NV4=...) -- GGraphCon NSW construction, Algorithm 2 (§IV-B, P:253-297,
// Alg. 2), on sm_100a.
//
// Data (device):
//   gid  [n][d_max] int32 / gdist [n][d_max] fp32 : G in build form, rows
//        ascending by (dist, id); gid becomes the final graph (no conversion).
//   gpid [n][d_min] int32 / gpd [n][d_min] fp32   : G'
//   Eu / Ed [s][d_min]                            : backward edges E of one round,
//        fixed slot j*d_min + r for the j-th vertex of P_i (no atomics)
//   indeg / fill / segoff [n], touched [s*d_min], seg [s*d_min] : GatherScatter
//
// Kernels (one warp per unit of work; the search is the same fused warp program
// as ganns_search, ganns_dev.cuh):
//   K2 phase1_kernel    one warp per group P_i: sequential insertion into the
//                       local graph G_i (Alg. 2 lines 2-8)
//   K3 round_search     one warp per v in P_i: Search(G_0, v) merged with v.N'
//                       -> new v.N, backward edges -> E (lines 10-17)
//   K4 gather/scatter   group E by source vertex u (line 19) -- see below
//   K5 round_merge      one warp per distinct u: u.N <- first d_max of
//                       merge(u.N, E segment of u) (lines 20-22)
//
// GatherScatter, B200 form: instead of a device-wide bitonic sort of E plus a
// flag prefix sum, each E entry bumps indeg[u]; the first bump appends u
// to `touched`; segments are carved out of `seg` with one atomicAdd per distinct
// u; entries are scattered into their segment.  Only the segment *order* is
// non-deterministic, and K5 keeps the d_max smallest (dist, id) keys of
// row ∪ segment, which does not depend on it -- the graph is bit-identical to
// sorting E by (u, dist, v) (R-C17).
#include "ganns_dev.cuh"
#include "ganns_internal.h"

#ifndef GANNS_NV4
#error "compile with -DGANNS_NV4=<1|2|4|8>"
#endif

#include <algorithm>
#include <cmath>
#include <vector>

namespace ganns {

constexpr int kBuildWarps = 1;   // one warp per CTA spreads the latency-bound build searches over all SMs

// Insert key kx into a warp-distributed ascending row of d_max keys (TPL per
// lane, slot j = t*32 + lane); the last key falls off when the row is full
// (P:281).  Keys at j >= d_max are kept at +inf.  Returns the insert position.
template <int TPL>
__device__ __forceinline__ int row_insert(uint64_t (&key)[TPL], uint64_t kx, int d_max, int lane) {
  int pos = 0;
#pragma unroll
  for (int t = 0; t < TPL; ++t) pos += __popc(__ballot_sync(kFull, key[t] < kx));
  if (pos >= d_max) return pos;
  uint64_t up[TPL], last[TPL];
#pragma unroll
  for (int t = 0; t < TPL; ++t) {
    uint32_t lo = __shfl_up_sync(kFull, uint32_t(key[t]), 1);
    uint32_t hi = __shfl_up_sync(kFull, uint32_t(key[t] >> 32), 1);
    up[t] = (uint64_t(hi) << 32) | lo;
    last[t] = shfl64(key[t], 31);
  }
#pragma unroll
  for (int t = 0; t < TPL; ++t) {
    const int j = t * 32 + lane;
    uint64_t prev = lane == 0 ? (t > 0 ? last[t > 0 ? t - 1 : 0] : kKeyInf) : up[t];
    uint64_t nv = j < pos ? key[t] : (j == pos ? kx : prev);
    key[t] = j < d_max ? nv : kKeyInf;
  }
  return pos;
}

template <int TPL>
__device__ __forceinline__ void row_load(uint64_t (&key)[TPL], const int32_t* gid, const float* gdist,
                                         int64_t u, int d_max, int lane) {
#pragma unroll
  for (int t = 0; t < TPL; ++t) {
    const int j = t * 32 + lane;
    int32_t id = j < d_max ? *reinterpret_cast<const volatile int32_t*>(gid + size_t(u) * d_max + j) : -1;
    float dd = j < d_max ? *reinterpret_cast<const volatile float*>(gdist + size_t(u) * d_max + j) : 0.f;
    key[t] = id >= 0 ? mkkey(dd, id) : kKeyInf;
  }
}

template <int TPL>
__device__ __forceinline__ void row_store(const uint64_t (&key)[TPL], int32_t* gid, float* gdist,
                                          int64_t u, int d_max, int from, int lane) {
#pragma unroll
  for (int t = 0; t < TPL; ++t) {
    const int j = t * 32 + lane;
    if (j < d_max && j >= from) {
      bool empty = key_empty(key[t]);
      gid[size_t(u) * d_max + j] = empty ? -1 : key_id(key[t]);
      gdist[size_t(u) * d_max + j] = empty ? __int_as_float(0x7f800000) : key_dist(key[t]);
    }
  }
}

struct BuildDev {
  GraphView g;          // g.nbr == gid
  int32_t* gid;
  float* gdist;
  int32_t* gpid;
  float* gpd;
  int d_min, l_build, e_build;
  int l_local, e_local;   // Phase-1 searches on the local graphs (<= l_build)
  unsigned long long* stats;   // [3] iterations, comps, searches
};

__device__ __forceinline__ void add_stats(unsigned long long* st, const SearchStats& s, int lane) {
  if (lane == 0) {
    atomicAdd(st + 0, (unsigned long long)s.iters);
    atomicAdd(st + 1, (unsigned long long)s.comps);
    atomicAdd(st + 2, 1ull);
  }
}

// ------------------------------------------------------------------ K2
// Phase 1: local graph construction (Alg. 2 lines 2-8).
template <int NV4, int TPL, bool L2>
__global__ void __launch_bounds__(kBuildWarps * 32)
phase1_kernel(BuildDev B, int64_t group_size, int64_t ngroups,
              const __grid_constant__ CUtensorMap tmap) {
  B.g.tmap = &tmap;
  extern __shared__ __align__(128) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t gi = int64_t(blockIdx.x) * kBuildWarps + w;
  if (gi >= ngroups) return;
  WarpSmem ws = carve_warp_smem(
      smem + size_t(w) * warp_smem_bytes(B.l_build, TPL, NV4, B.g.d4, kBuildStageRounds),
      B.l_build, TPL, NV4, B.g.d4, kBuildStageRounds);
  if (lane == 0) mbar_init(ws.mbar, 1);
  __syncwarp();
  uint64_t* sN = ws.sN;
  const int64_t lo = gi * group_size;
  const int64_t hi = lo + group_size < B.g.n ? lo + group_size : B.g.n;
  const int d = B.g.d4 * 4;
  for (int64_t v = lo + 1; v < hi; ++v) {
    // Step 1 (line 5): v.N, v.N' := Search(G_i, v, d_min), entry = group's first vertex
    SearchStats st;
    const int cnt = warp_search<NV4, TPL, L2, true>(B.g, B.g.X + size_t(v) * d, int32_t(lo),
                                                    B.l_local, B.e_local, ws, st);
    add_stats(B.stats, st, lane);
    const int m = cnt < B.d_min ? cnt : B.d_min;
    for (int j = lane; j < m; j += 32) {
      uint64_t k = unflag(sN[j]);
      B.gid[size_t(v) * B.g.d_max + j] = key_id(k);
      B.gdist[size_t(v) * B.g.d_max + j] = key_dist(k);
      B.gpid[size_t(v) * B.d_min + j] = key_id(k);
      B.gpd[size_t(v) * B.d_min + j] = key_dist(k);
    }
    __syncwarp();
    // Step 2 (lines 6-8): insert v into u.N for every u in v.N (sorted, truncated).
    // The u are distinct, so their rows are independent: CH rows are loaded at once
    // (one memory round trip per chunk instead of per row).
    constexpr int CH = TPL >= 4 ? 2 : 8 / TPL;
    for (int r0 = 0; r0 < m; r0 += CH) {
      uint64_t key[CH][TPL];
      uint64_t kf[CH];
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        kf[c] = r0 + c < m ? unflag(sN[r0 + c]) : kKeyInf;
        if (r0 + c < m) row_load<TPL>(key[c], B.gid, B.gdist, key_id(kf[c]), B.g.d_max, lane);
      }
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        if (r0 + c >= m) break;   // warp-uniform
        const int32_t u = key_id(kf[c]);
        const int pos = row_insert<TPL>(key[c], mkkey(key_dist(kf[c]), int32_t(v)), B.g.d_max, lane);
        row_store<TPL>(key[c], B.gid, B.gdist, u, B.g.d_max, pos, lane);
      }
      __syncwarp();
    }
  }
}

// ------------------------------------------------------------------ K3
// Phase 2 Step 1 (Alg. 2 lines 10-17) + the counting half of K4.
template <int NV4, int TPL, bool L2>
__global__ void __launch_bounds__(kBuildWarps * 32)
round_search_kernel(BuildDev B, int64_t lo, int64_t hi, int32_t* __restrict__ Eu,
                    float* __restrict__ Ed, int32_t* __restrict__ indeg,
                    int32_t* __restrict__ touched, int32_t* __restrict__ counters,
                    const __grid_constant__ CUtensorMap tmap, const UpperLayers U, int layer) {
  B.g.tmap = &tmap;
  extern __shared__ __align__(128) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t v = lo + int64_t(blockIdx.x) * kBuildWarps + w;
  if (v >= hi) return;
  WarpSmem ws = carve_warp_smem(
      smem + size_t(w) * warp_smem_bytes(B.l_build, TPL, NV4, B.g.d4, kBuildStageRounds),
      B.l_build, TPL, NV4, B.g.d4, kBuildStageRounds);
  if (lane == 0) mbar_init(ws.mbar, 1);
  __syncwarp();
  uint64_t* sN = ws.sN;
  uint64_t* sT = ws.sT;
  const int d = B.g.d4 * 4;
  // line 12: v.N := Search(G_0, v, d_min); G_0 = P_0..P_{i-1}, entry = vertex 0;
  // HNSW: enter through a greedy descent of the finished upper layers,
  // kept only if the vertex reached is already in G_0 (R-H2)
  int32_t entry = 0;
  if (U.top > layer) {
    const int32_t c = descend<NV4, TPL, L2>(B.g, U, layer + 1, B.g.X + size_t(v) * d, ws);
    entry = c < lo ? c : 0;
  }
  SearchStats st;
  const int cnt = warp_search<NV4, TPL, L2, false>(B.g, B.g.X + size_t(v) * d, entry, B.l_build,
                                                   B.e_build, ws, st);
  add_stats(B.stats, st, lane);
  const int dm = B.d_min;
  const int cs = cnt < dm ? cnt : dm;
  // v.N' -> sT[0..cg)
  int cg = 0;
  for (int j = lane; j < dm; j += 32) {
    int32_t id = B.gpid[size_t(v) * dm + j];
    sT[j] = id >= 0 ? mkkey(B.gpd[size_t(v) * dm + j], id) : kKeyInf;
  }
  __syncwarp();
  for (int j = 0; j < dm; ++j) cg += key_empty(sT[j]) ? 0 : 1;
  // line 14: v.N := first d_min of merge(search result, v.N') (R-C16); rank merge
  const int64_t slot0 = (v - lo) * dm;
  const int nf = cs + cg < dm ? cs + cg : dm;
  int32_t* row = B.gid + size_t(v) * B.g.d_max;
  float* rowd = B.gdist + size_t(v) * B.g.d_max;
  for (int j = lane; j < B.g.d_max; j += 32) {   // v's Phase-1 backward edges are dropped (R-C15)
    if (j >= nf) { row[j] = -1; rowd[j] = __int_as_float(0x7f800000); }
  }
  for (int j = lane; j < dm; j += 32)
    if (j >= nf) Eu[slot0 + j] = -1;
  for (int i = lane; i < cs + cg; i += 32) {
    uint64_t key;
    int rank = 0;
    if (i < cs) {
      key = unflag(sN[i]);
      for (int j = 0; j < cg; ++j) rank += sT[j] < key ? 1 : 0;
      rank += i;
    } else {
      key = sT[i - cs];
      for (int j = 0; j < cs; ++j) rank += unflag(sN[j]) < key ? 1 : 0;
      rank += i - cs;
    }
    if (rank < dm) {
      const int32_t u = key_id(key);
      const float dd = key_dist(key);
      row[rank] = u;
      rowd[rank] = dd;
      // line 17: E := E u (u -> v, delta(u, v)) in a fixed slot
      Eu[slot0 + rank] = u;
      Ed[slot0 + rank] = dd;
      if (atomicAdd(&indeg[u], 1) == 0) touched[atomicAdd(&counters[0], 1)] = u;
    }
  }
}

// ------------------------------------------------------------------ K4
// Carve one segment per distinct source vertex u (grid-stride over `touched`).
static __global__ void alloc_segments_kernel(const int32_t* __restrict__ touched,
                                      const int32_t* __restrict__ indeg,
                                      int32_t* __restrict__ segoff, int32_t* counters) {
  const int32_t nt = counters[0];
  for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < nt; i += gridDim.x * blockDim.x) {
    const int32_t u = touched[i];
    segoff[u] = atomicAdd(&counters[1], indeg[u]);
  }
}

// Scatter each E entry (u -> v, delta) into u's segment as the key (delta, v).
static __global__ void scatter_edges_kernel(const int32_t* __restrict__ Eu, const float* __restrict__ Ed,
                                     int64_t nslots, int d_min, int64_t lo,
                                     const int32_t* __restrict__ segoff, int32_t* __restrict__ fill,
                                     uint64_t* __restrict__ seg) {
  for (int64_t j = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; j < nslots;
       j += int64_t(gridDim.x) * blockDim.x) {
    const int32_t u = Eu[j];
    if (u < 0) continue;
    const int32_t p = atomicAdd(&fill[u], 1);
    seg[segoff[u] + p] = mkkey(Ed[j], int32_t(lo + j / d_min));
  }
}

// ------------------------------------------------------------------ K5
// Phase 2 Step 3 (Alg. 2 lines 20-22): per distinct u, keep the first
// d_max of merge(u.N, E segment of u).  Resets the per-u counters for the next round.
template <int TPL>
__global__ void __launch_bounds__(kBuildWarps * 32)
round_merge_kernel(int32_t* __restrict__ gid, float* __restrict__ gdist, int d_max,
                   const int32_t* __restrict__ touched, int32_t* __restrict__ indeg,
                   int32_t* __restrict__ fill, const int32_t* __restrict__ segoff,
                   const uint64_t* __restrict__ seg, const int32_t* __restrict__ counters) {
  const int lane = threadIdx.x & 31;
  const int32_t nt = counters[0];
  const int32_t nwarps = gridDim.x * kBuildWarps;
  for (int32_t i = blockIdx.x * kBuildWarps + (threadIdx.x >> 5); i < nt; i += nwarps) {
    const int32_t u = touched[i];
    const int32_t m = indeg[u], off = segoff[u];
    uint64_t key[TPL];
    row_load<TPL>(key, gid, gdist, u, d_max, lane);
    int from = d_max;
    for (int32_t c = 0; c < m; c += 32) {
      const uint64_t x = c + lane < m ? seg[off + c + lane] : kKeyInf;
      const int tw = (d_max - 1) >> 5, tl = (d_max - 1) & 31;
      uint64_t worst = 0;
#pragma unroll
      for (int t = 0; t < TPL; ++t) {
        uint64_t wv = shfl64(key[t], tl);
        if (t == tw) worst = wv;
      }
      unsigned b = __ballot_sync(kFull, x < worst);
      while (b) {
        const int src = __ffs(b) - 1;
        b &= b - 1;
        const int pos = row_insert<TPL>(key, shfl64(x, src), d_max, lane);
        from = pos < from ? pos : from;
      }
    }
    row_store<TPL>(key, gid, gdist, u, d_max, from, lane);
    if (lane == 0) {
      indeg[u] = 0;
      fill[u] = 0;
    }
  }
}

// ------------------------------------------------------------------ host
template <int NV4, int TPL, bool L2>
static cudaError_t set_smem_attrs() {
  static std::atomic<uint64_t> done{0};   // per instantiation, per device
  return once_per_device(done, [] {
    const int mx = 227 * 1024;
    cudaError_t e = cudaFuncSetAttribute(phase1_kernel<NV4, TPL, L2>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(round_search_kernel<NV4, TPL, L2>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    return e;
  });
}

template <typename T>
struct DevBuf {
  T* p = nullptr;
  cudaError_t alloc(size_t count) { return cudaMalloc(&p, std::max<size_t>(count, 1) * sizeof(T)); }
  ~DevBuf() { if (p) cudaFree(p); }
};

#define GANNS_TRY(...)                                           \
  do {                                                           \
    cudaError_t _e = (__VA_ARGS__);                              \
    if (_e != cudaSuccess) return cuda_fail(_e, #__VA_ARGS__);   \
  } while (0)

static __global__ void fill_rows_kernel(int32_t* ids, float* dists, int64_t count) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < count;
       i += int64_t(gridDim.x) * blockDim.x) {
    ids[i] = -1;
    dists[i] = __int_as_float(0x7f800000);
  }
}

template <int NV4, int TPL, bool L2>
static int build_t(BuildArgs& a, cudaStream_t s) {
  GANNS_TRY(set_smem_attrs<NV4, TPL, L2>());
  const int64_t n = a.n, S = a.group_size;
  const int64_t ngroups = (n + S - 1) / S;
  const int dm = a.d_min, dmax = a.d_max;
  DevBuf<float> gdist, gpd, Ed;
  DevBuf<int32_t> gpid, Eu, indeg, fill, segoff, touched, counters;
  DevBuf<uint64_t> seg;
  DevBuf<unsigned long long> stats;
  GANNS_TRY(gdist.alloc(size_t(n) * dmax));
  GANNS_TRY(gpid.alloc(size_t(n) * dm));
  GANNS_TRY(gpd.alloc(size_t(n) * dm));
  GANNS_TRY(Eu.alloc(size_t(S) * dm));
  GANNS_TRY(Ed.alloc(size_t(S) * dm));
  GANNS_TRY(indeg.alloc(size_t(n)));
  GANNS_TRY(fill.alloc(size_t(n)));
  GANNS_TRY(segoff.alloc(size_t(n)));
  GANNS_TRY(touched.alloc(size_t(S) * dm));
  GANNS_TRY(seg.alloc(size_t(S) * dm));
  GANNS_TRY(counters.alloc(2));
  GANNS_TRY(stats.alloc(3));
  GANNS_TRY(cudaMemsetAsync(indeg.p, 0, sizeof(int32_t) * n, s));
  GANNS_TRY(cudaMemsetAsync(fill.p, 0, sizeof(int32_t) * n, s));
  GANNS_TRY(cudaMemsetAsync(stats.p, 0, sizeof(unsigned long long) * 3, s));
  fill_rows_kernel<<<148 * 8, 256, 0, s>>>(a.out_nbr, gdist.p, n * dmax);
  fill_rows_kernel<<<148 * 8, 256, 0, s>>>(gpid.p, gpd.p, n * dm);
  count_launch(2);
  GANNS_TRY(cudaGetLastError());

  BuildDev B;
  B.g = GraphView{a.out_nbr, a.X, nullptr, n, dmax, a.d / 4, a.metric};
  CUtensorMap tmap;
  GANNS_TRY(uses_tma(NV4) ? encode_row_tmap(a.X, n, a.d, &tmap) : zero_tmap(&tmap));
  B.gid = a.out_nbr;
  B.gdist = gdist.p;
  B.gpid = gpid.p;
  B.gpd = gpd.p;
  B.d_min = dm;
  B.l_build = a.l_build;
  B.e_build = a.e_build;
  B.l_local = a.l_local > 0 ? a.l_local : a.l_build;
  B.e_local = a.e_local > 0 ? a.e_local : a.e_build;
  B.stats = stats.p;
  const size_t smem =
      size_t(kBuildWarps) * warp_smem_bytes(a.l_build, TPL, NV4, a.d / 4, kBuildStageRounds);
  if (smem > 227 * 1024) return fail(-4, "build: shared memory per CTA exceeds 227 KB");

  // Phase 1 (lines 2-8): all local graphs in parallel, one warp per group
  phase1_kernel<NV4, TPL, L2><<<unsigned((ngroups + kBuildWarps - 1) / kBuildWarps),
                                kBuildWarps * 32, smem, s>>>(B, S, ngroups, tmap);
  count_launch();
  GANNS_TRY(cudaGetLastError());

  // Phase 2 (lines 9-22): merge P_1..P_t into G_0, one round per group
  UpperLayers U;
  U.top = a.upper.top;
  for (int j = 0; j < kMaxLayers; ++j) {
    U.nbr[j] = a.upper.nbr[j];
    U.n[j] = a.upper.n[j];
  }
  int64_t rounds = 0;
  const int64_t last = a.max_rounds < 0 ? ngroups - 1 : std::min<int64_t>(ngroups - 1, a.max_rounds);
  for (int64_t i = 1; i <= last; ++i) {
    const int64_t lo = i * S, hi = std::min(lo + S, n);
    const int64_t nv = hi - lo, nslots = nv * dm;
    GANNS_TRY(cudaMemsetAsync(counters.p, 0, sizeof(int32_t) * 2, s));
    round_search_kernel<NV4, TPL, L2><<<unsigned((nv + kBuildWarps - 1) / kBuildWarps),
                                        kBuildWarps * 32, smem, s>>>(
        B, lo, hi, Eu.p, Ed.p, indeg.p, touched.p, counters.p, tmap, U, a.layer);
    const unsigned gs = unsigned(std::min<int64_t>((nslots + 255) / 256, 148 * 4));
    alloc_segments_kernel<<<gs, 256, 0, s>>>(touched.p, indeg.p, segoff.p, counters.p);
    scatter_edges_kernel<<<gs, 256, 0, s>>>(Eu.p, Ed.p, nslots, dm, lo, segoff.p, fill.p, seg.p);
    const unsigned gm = unsigned(std::min<int64_t>((nslots + kBuildWarps - 1) / kBuildWarps, 148 * 8));
    round_merge_kernel<TPL><<<gm, kBuildWarps * 32, 0, s>>>(a.out_nbr, gdist.p, dmax, touched.p,
                                                           indeg.p, fill.p, segoff.p, seg.p,
                                                           counters.p);
    count_launch(4);
    GANNS_TRY(cudaGetLastError());
    ++rounds;
  }
  unsigned long long hs[3];
  GANNS_TRY(cudaMemcpyAsync(hs, stats.p, sizeof(hs), cudaMemcpyDeviceToHost, s));
  GANNS_TRY(cudaStreamSynchronize(s));
  a.stats[0] = hs[0];
  a.stats[1] = hs[1];
  a.stats[2] = hs[2];
  a.stats[3] = uint64_t(rounds);
  return 0;
}

template <int NV4, int TPL>
static int build_m(BuildArgs& a, cudaStream_t s) {
#ifdef GANNS_DEV_ONE
  return build_t<NV4, TPL, true>(a, s);
#endif
  return a.metric == 0 ? build_t<NV4, TPL, true>(a, s) : build_t<NV4, TPL, false>(a, s);
}
template <int NV4>
int run_build_nv(BuildArgs& a, cudaStream_t s) {
#ifdef GANNS_DEV_ONE
  return build_m<NV4, 1>(a, s);
#endif
  switch (tpl_for(a.d_max)) {
    case 1: return build_m<NV4, 1>(a, s);
    case 2: return build_m<NV4, 2>(a, s);
    case 4: return build_m<NV4, 4>(a, s);
  }
  return fail(-4, "unsupported degree");
}

template int run_build_nv<GANNS_NV4>(BuildArgs&, cudaStream_t);

}  // namespace ganns
