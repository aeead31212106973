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
#include "search_group.cuh"   // includes ganns_dev.cuh
#include "../../include/ganns.h"
#include "ganns_internal.h"

#ifndef GANNS_NV4
#error "compile with -DGANNS_NV4=<1|2|4|8>"
#endif

#include <algorithm>
#include <cstdlib>
#include <cmath>
#include <new>
#include <type_traits>
#include <vector>

namespace ganns {

// Programmatic dependent launch (PDL): the kernels of a Phase-2 round (K3, K4a,
// K4b, K5, and the staged form's apply) are launched with programmatic stream
// serialization, so each grid is scheduled while its predecessor drains (a round's
// search kernel ends with its slowest search, most CTAs having exited) and waits
// for the predecessor's completion and memory with griddepcontrol.wait before it
// reads anything the predecessor wrote.  Without the launch attribute the wait
// returns at once (the predecessor has completed).
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
// (an explicit griddepcontrol.launch_dependents at the start of K4a/K4b/K5 was
// measured slower: Phase 2 0.311 -> 0.317 s; the implicit trigger at CTA exit is kept)

template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*k)(KArgs...), unsigned grid, unsigned block, size_t smem,
                              cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

constexpr int kBuildWarps = 1;   // one warp per CTA spreads the latency-bound build searches over all SMs
// d > 256 (GANNS_BUILD_GROUP): a build search is run by a warp group, as the wide
// batched search (search_group.cuh): warp 0 runs the loop, all kGroupWarps warps
// reduce their column slices of each staged row -- one CTA of kGroupWarps warps
// per search (per group in Phase 1)
#ifndef GANNS_BUILD_GROUP
#define GANNS_BUILD_GROUP 1
#endif
template <int NV4>
constexpr bool kBuildGroup = GANNS_BUILD_GROUP != 0 && !uses_tma(NV4);
template <int NV4>
constexpr int kBuildThreads = kBuildGroup<NV4> ? kGroupWarps * 32 : kBuildWarps * 32;
// one-warp searches: a Phase-2 round of s = 1536 searches needs 1536 / 148 = 10.4
// resident CTAs per SM (one wave; shared memory holds 12-13): the register budget
// must not cap residency below that (<= 168 registers at 12 CTAs of one warp)
template <int NV4>
constexpr int kBuildMinBlocks = kBuildGroup<NV4> ? kGroupMinBlocks : 12;
template <int NV4, bool L2>
using BuildGroupDist = GroupDist<(NV4 >= 4 ? NV4 / 4 : 1), L2>;
#ifndef GANNS_BUILD_PREDICT
#define GANNS_BUILD_PREDICT 0
#endif
// GANNS_BUILD_PREDICT=1: the build searches predict the next exploration and load its
// adjacency row early (ganns_dev.cuh: warp_search_with, PREDICT).  Off: measured on
// the GPU clock (C2, 8 builds each) Phase 1 0.1244 vs 0.1199 s, Phase 2 0.4256 vs
// 0.4078 s with / without (profiles/r02/build_phases_predict_ab.log) -- the extra
// warp-min and load sit on the chain and the hidden adjacency latency is small (the
// adjacency rows mostly hit L2)
constexpr bool kBuildPredict = GANNS_BUILD_PREDICT != 0;
// The build searches' stage is filled by cp.async (ganns_dev.cuh: cpasync_fill_quad) for
// d <= 256, and (d_max <= 32) the next exploration's rows are gathered
// speculatively while the lazy check, sort and merge run (warp_search_with, SPEC).
// A build search is a latency chain: a Phase-2 round lasts as long as its slowest
// search (1.05x, tools/round_tail.py), which runs 1.7x the mean iteration count.
#ifndef GANNS_BUILD_CPASYNC
#define GANNS_BUILD_CPASYNC 1
#endif
#ifndef GANNS_BUILD_SPEC
#define GANNS_BUILD_SPEC 1
#endif
template <int NV4>
constexpr bool kBuildCpAsync = GANNS_BUILD_CPASYNC != 0 && uses_tma(NV4);
template <int NV4, int TPL>
constexpr bool kBuildSpec = GANNS_BUILD_SPEC != 0 && kBuildCpAsync<NV4> && TPL == 1 && !kBuildPredict;
// GANNS_BUILD_P1: Phase 1 (l_local searches on the local graphs) uses the same
// cp.async + speculation form as Phase 2; else the TMA tile::gather4 form
#ifndef GANNS_BUILD_P1
#define GANNS_BUILD_P1 1
#endif
template <int NV4>
constexpr bool kP1CpAsync = kBuildCpAsync<NV4> && GANNS_BUILD_P1 != 0;
template <int NV4, int TPL>
constexpr bool kP1Spec = kBuildSpec<NV4, TPL> && GANNS_BUILD_P1 != 0;
#ifndef GANNS_BUILD_T_OUT
#define GANNS_BUILD_T_OUT 1
#endif

// Per-warp shared memory of a build search: the search's area, then (cp.async
// form) T outside the stage
template <int NV4, int TPL>
__host__ __device__ constexpr size_t build_warp_bytes(int l, int d4, int wrows) {
  return warp_smem_bytes(l, TPL, NV4, d4, kBuildStageRounds, wrows) +
         (kBuildCpAsync<NV4> && GANNS_BUILD_T_OUT ? t_bytes(TPL) : 0);
}
// wrows: d > 256, rows per TMA round of the build search (BuildDev::wrows_p1/_p2)
template <int NV4, int TPL>
__device__ __forceinline__ WarpSmem carve_build_smem(uint8_t* smem, int w, int l, int d4, int wrows) {
  uint8_t* base = smem + size_t(w) * build_warp_bytes<NV4, TPL>(l, d4, wrows);
  WarpSmem ws = carve_warp_smem(base, l, TPL, NV4, d4, kBuildStageRounds, wrows);
  if constexpr (kBuildCpAsync<NV4> && GANNS_BUILD_T_OUT) {
    ws.sT = reinterpret_cast<uint64_t*>(base + warp_smem_bytes(l, TPL, NV4, d4, kBuildStageRounds, wrows));
  }
  return ws;
}

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
  int wrows_p1, wrows_p2;   // d > 256: rows per TMA round in Phase 1 / Phase 2
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
__global__ void __launch_bounds__(kBuildThreads<NV4>, kBuildMinBlocks<NV4>)
phase1_kernel(BuildDev B, int64_t group_size, int64_t g0, int64_t g1,
              const __grid_constant__ CUtensorMap tmap) {
  B.g.tmap = &tmap;
  extern __shared__ __align__(128) uint8_t smem[];
  constexpr bool GROUP = kBuildGroup<NV4>;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t gi = g0 + int64_t(blockIdx.x) * kBuildWarps + (GROUP ? 0 : w);   // groups [g0, g1)
  if (gi >= g1) return;
  WarpSmem ws = carve_build_smem<NV4, TPL>(smem, GROUP ? 0 : w, B.l_build, B.g.d4, B.wrows_p1);
  BuildGroupDist<NV4, L2> gdist;
  if constexpr (GROUP) {
    gdist.gs = carve_group(smem + build_warp_bytes<NV4, TPL>(B.l_build, B.g.d4, B.wrows_p1));
    gdist.kc = 0;
    if (threadIdx.x == 0) mbar_init(ws.mbar, 1);
    __syncthreads();
    if (w != 0) {
      group_helper_loop<(NV4 >= 4 ? NV4 / 4 : 1), L2>(B.g, B.g.X, gdist.gs, ws, w, lane);
      return;
    }
  } else {
    if (lane == 0) mbar_init(ws.mbar, 1);
    __syncwarp();
  }
  uint64_t* sN = ws.sN;
  const int64_t lo = gi * group_size;
  const int64_t hi = lo + group_size < B.g.n ? lo + group_size : B.g.n;
  const int d = B.g.d4 * 4;
  for (int64_t v = lo + 1; v < hi; ++v) {
    // Step 1 (line 5): v.N, v.N' := Search(G_i, v, d_min), entry = group's first vertex
    SearchStats st;
    int cnt;
    if constexpr (GROUP) {
      group_new_query(gdist, B.g, B.g.X, v, lane);
      cnt = warp_search_with<BuildGroupDist<NV4, L2>, TPL, true>(B.g, gdist, int32_t(lo), B.l_local,
                                                                 B.e_local, ws, st);
    } else {
      cnt = warp_search<NV4, TPL, L2, true, kBuildPredict, kP1Spec<NV4, TPL>, kP1CpAsync<NV4>>(
          B.g, B.g.X + size_t(v) * d, int32_t(lo), B.l_local, B.e_local, ws, st);
    }
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
    constexpr int CH = TPL >= 4 ? 2 : 8 / TPL;   // (16 rows at once: Phase 1 0.094 -> 0.096 s)
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
  if constexpr (GROUP) gdist.post(kCmdExit, lane);
}

// The end of a Phase-2 search of v (Alg. 2 lines 14-17): v.N := first d_min of
// merge(search result, v.N') (R-C16); fused form: v's row, its E slots and the
// in-degree counts; staged form: the forward row F only.
template <int TPL>
__device__ __forceinline__ void round_finish(const BuildDev& B, int64_t v, int64_t lo, int64_t v0,
                                             int cnt, const SearchStats& st, WarpSmem& ws, int lane,
                                             int32_t* __restrict__ Eu, float* __restrict__ Ed,
                                             int32_t* __restrict__ indeg,
                                             int32_t* __restrict__ touched,
                                             int32_t* __restrict__ counters,
                                             int32_t* __restrict__ F_ids,
                                             float* __restrict__ F_dists) {
  uint64_t* sN = ws.sN;
  uint64_t* sT = ws.sT;
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
  const bool staged = F_ids != nullptr;
  if (staged) {
    for (int j = lane; j < dm; j += 32)
      if (j >= nf) {
        F_ids[size_t(v - v0) * dm + j] = -1;
        F_dists[size_t(v - v0) * dm + j] = __int_as_float(0x7f800000);
      }
  } else {
    for (int j = lane; j < B.g.d_max; j += 32) {   // v's Phase-1 backward edges are dropped (R-C15)
      if (j >= nf) { row[j] = -1; rowd[j] = __int_as_float(0x7f800000); }
    }
    for (int j = lane; j < dm; j += 32)
      if (j >= nf) Eu[slot0 + j] = -1;
  }
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
      if (staged) {
        F_ids[size_t(v - v0) * dm + rank] = u;
        F_dists[size_t(v - v0) * dm + rank] = dd;
        continue;
      }
      row[rank] = u;
      rowd[rank] = dd;
      // line 17: E := E u (u -> v, delta(u, v)) in a fixed slot
      Eu[slot0 + rank] = u;
      Ed[slot0 + rank] = dd;
      if (atomicAdd(&indeg[u], 1) == 0) touched[atomicAdd(&counters[0], 1)] = u;
    }
  }
}

// ------------------------------------------------------------------ K3
// Phase 2 Step 1 (Alg. 2 lines 10-17) + the counting half of K4, for
// the vertices [v0, v1) of P_i = [lo, hi).  Fused form (F_ids == nullptr, one GPU):
// v's row, its E slots and the in-degree counts are written here.  Staged form
// (multi-GPU build): only the new forward row F (first d_min) is written, to
// F_ids / F_dists [(v - v0)][d_min]; apply_forward_kernel consumes the F of all of
// P_i after the exchange.
// HNSW: the instance that enters through the descent of the upper layers (the
// plain NSW build's instance carries no descent code)
template <int NV4, int TPL, bool L2, bool HNSW>
__global__ void __launch_bounds__(kBuildThreads<NV4>, kBuildMinBlocks<NV4>)
round_search_kernel(BuildDev B, int64_t lo, int64_t v0, int64_t v1, int32_t* __restrict__ Eu,
                    float* __restrict__ Ed, int32_t* __restrict__ indeg,
                    int32_t* __restrict__ touched, int32_t* __restrict__ counters,
                    int32_t* __restrict__ F_ids, float* __restrict__ F_dists,
                    const __grid_constant__ CUtensorMap tmap, const UpperLayers U, int layer) {
  pdl_wait();   // G_0 as the previous round's K5 left it
  B.g.tmap = &tmap;
  extern __shared__ __align__(128) uint8_t smem[];
  // the HNSW instance keeps the one-warp form (its descent is the leader's alone)
  constexpr bool GROUP = kBuildGroup<NV4> && !HNSW;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t v = v0 + int64_t(blockIdx.x) * kBuildWarps + (kBuildGroup<NV4> ? 0 : w);
  if (v >= v1) return;
  if constexpr (kBuildGroup<NV4> && HNSW)
    if (w != 0) return;
  WarpSmem ws = carve_build_smem<NV4, TPL>(smem, kBuildGroup<NV4> ? 0 : w, B.l_build, B.g.d4,
                                           B.wrows_p2);
  BuildGroupDist<NV4, L2> gdist;
  if constexpr (GROUP) {
    gdist.gs = carve_group(smem + build_warp_bytes<NV4, TPL>(B.l_build, B.g.d4, B.wrows_p2));
    gdist.kc = 0;
    if (threadIdx.x == 0) mbar_init(ws.mbar, 1);
    __syncthreads();
    if (w != 0) {
      group_helper_loop<(NV4 >= 4 ? NV4 / 4 : 1), L2>(B.g, B.g.X, gdist.gs, ws, w, lane);
      return;
    }
  } else {
    if (lane == 0) mbar_init(ws.mbar, 1);
    __syncwarp();
  }
  const int d = B.g.d4 * 4;
  // line 12: v.N := Search(G_0, v, d_min); G_0 = P_0..P_{i-1}, entry = vertex 0;
  // HNSW: enter through a greedy descent of the finished upper layers,
  // kept only if the vertex reached is already in G_0 (R-H2)
  int32_t entry = 0;
  if constexpr (HNSW) {
    if (U.top > layer) {
      const int32_t c = descend<NV4, TPL, L2, kBuildCpAsync<NV4>>(B.g, U, layer + 1,
                                                                 B.g.X + size_t(v) * d, ws);
      entry = c < lo ? c : 0;
    }
  }
  SearchStats st;
  int cnt;
  if constexpr (GROUP) {
    group_new_query(gdist, B.g, B.g.X, v, lane);
    cnt = warp_search_with<BuildGroupDist<NV4, L2>, TPL, false>(B.g, gdist, entry, B.l_build,
                                                                B.e_build, ws, st);
    gdist.post(kCmdExit, lane);
  } else {
    cnt = warp_search<NV4, TPL, L2, false, kBuildPredict, kBuildSpec<NV4, TPL>, kBuildCpAsync<NV4>>(
        B.g, B.g.X + size_t(v) * d, entry, B.l_build, B.e_build, ws, st);
  }
  round_finish<TPL>(B, v, lo, v0, cnt, st, ws, lane, Eu, Ed, indeg, touched, counters, F_ids,
                    F_dists);
}

// Staged form, after the exchange: the F of every v in P_i = [lo, hi) becomes v's
// row (R-C15) and its E slots (line 17), and the in-degrees are counted -- exactly
// what the fused round_search_kernel writes.  One warp per v.
static __global__ void apply_forward_kernel(const int32_t* __restrict__ F_ids,
                                            const float* __restrict__ F_dists, int64_t lo,
                                            int64_t hi, int d_min, int d_max,
                                            int32_t* __restrict__ gid, float* __restrict__ gdist,
                                            int32_t* __restrict__ Eu, float* __restrict__ Ed,
                                            int32_t* __restrict__ indeg,
                                            int32_t* __restrict__ touched,
                                            int32_t* __restrict__ counters) {
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t v = lo + int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); v < hi;
       v += nwarps) {
    const size_t f0 = size_t(v - lo) * d_min;
    for (int j = lane; j < d_max; j += 32) {
      const int32_t u = j < d_min ? F_ids[f0 + j] : -1;
      const float dd = j < d_min ? F_dists[f0 + j] : __int_as_float(0x7f800000);
      gid[size_t(v) * d_max + j] = u;
      gdist[size_t(v) * d_max + j] = u >= 0 ? dd : __int_as_float(0x7f800000);
      if (j < d_min) {
        Eu[f0 + j] = u;
        Ed[f0 + j] = dd;
        if (u >= 0 && atomicAdd(&indeg[u], 1) == 0) touched[atomicAdd(&counters[0], 1)] = u;
      }
    }
  }
}

// ------------------------------------------------------------------ K4
// Carve one segment per distinct source vertex u (grid-stride over `touched`).
static __global__ void alloc_segments_kernel(const int32_t* __restrict__ touched,
                                      const int32_t* __restrict__ indeg,
                                      int32_t* __restrict__ segoff, int32_t* counters) {
  pdl_wait();
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
  pdl_wait();
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
// d_max of merge(u.N, E segment of u).  Resets the per-u counters and the next
// round's GatherScatter counters (double-buffered: round i uses counters[2(i&1)..];
// the other pair was last read by round i-1's kernels, which have completed).
// One warp per u, kMergeWarps per CTA, enough warps for one u each: a warp's work is
// a dependent chain (row load -> inserts -> store), so fewer warps looping over
// several u's made K5 latency-bound (28 us per round at 1184 warps).
constexpr int kMergeWarps = 8;
template <int TPL>
__global__ void __launch_bounds__(kMergeWarps * 32)
round_merge_kernel(int32_t* __restrict__ gid, float* __restrict__ gdist, int d_max,
                   const int32_t* __restrict__ touched, int32_t* __restrict__ indeg,
                   int32_t* __restrict__ fill, const int32_t* __restrict__ segoff,
                   const uint64_t* __restrict__ seg, const int32_t* __restrict__ counters,
                   int32_t* __restrict__ next_counters) {
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int32_t nt = counters[0];
  if (blockIdx.x == 0 && threadIdx.x < 2) next_counters[threadIdx.x] = 0;
  const int32_t nwarps = gridDim.x * kMergeWarps;
  for (int32_t i = blockIdx.x * kMergeWarps + (threadIdx.x >> 5); i < nt; i += nwarps) {
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
      e = cudaFuncSetAttribute(round_search_kernel<NV4, TPL, L2, false>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(round_search_kernel<NV4, TPL, L2, true>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, mx);
    return e;
  });
}

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

// The state of one Algorithm-2 construction (BuildState, ganns_internal.h) for
// this (NV4, TPL, L2) instance: the kernels' argument block and launch shapes.
struct BuildDevState {
  BuildDev B;
  UpperLayers U;
  size_t smem_p1, smem_p2;
};

template <int NV4, int TPL, bool L2>
static int phase1_t(BuildState& st, int64_t g0, int64_t g1, cudaStream_t s) {
  auto* ds = static_cast<BuildDevState*>(st.dev);
  if (g1 <= g0) return 0;
  // all local graphs of [g0, g1) in parallel, one warp per group (lines 2-8)
  phase1_kernel<NV4, TPL, L2><<<unsigned((g1 - g0 + kBuildWarps - 1) / kBuildWarps),
                                kBuildThreads<NV4>, ds->smem_p1, s>>>(ds->B, st.S, g0, g1, st.tmap);
  count_launch();
  GANNS_TRY(cudaGetLastError());
  return 0;
}

// the GatherScatter counters of round i (double-buffered, see round_merge_kernel)
static int32_t* round_counters(BuildState& st, int64_t i) { return st.counters + 2 * (i & 1); }

template <int NV4, int TPL, bool L2>
static int round_search_t(BuildState& st, int64_t i, int64_t v0, int64_t v1, int32_t* f_ids,
                          float* f_dists, cudaStream_t s) {
  auto* ds = static_cast<BuildDevState*>(st.dev);
  const int64_t lo = i * st.S;
  if (v1 <= v0) return 0;
  // fused form: this round's GatherScatter counters (zeroed by the previous round's
  // K5, or at begin for rounds 1 and 2)
  const unsigned grid = unsigned((v1 - v0 + kBuildWarps - 1) / kBuildWarps);
  if (ds->U.top > st.a.layer)
    GANNS_TRY(launch_pdl(round_search_kernel<NV4, TPL, L2, true>, grid, kBuildThreads<NV4>, ds->smem_p2,
                         s, ds->B, lo, v0, v1, st.Eu, st.Ed, st.indeg, st.touched,
                         round_counters(st, i), f_ids, f_dists, st.tmap, ds->U, st.a.layer));
  else
    GANNS_TRY(launch_pdl(round_search_kernel<NV4, TPL, L2, false>, grid, kBuildThreads<NV4>, ds->smem_p2,
                         s, ds->B, lo, v0, v1, st.Eu, st.Ed, st.indeg, st.touched,
                         round_counters(st, i), f_ids, f_dists, st.tmap, ds->U, st.a.layer));
  count_launch();
  return 0;
}

// Steps 2-3 of round i (lines 19-22) after the E slots and in-degrees are in place.
template <int TPL>
static int round_merge_t(BuildState& st, int64_t i, cudaStream_t s) {
  const int64_t lo = i * st.S, hi = std::min(lo + st.S, st.a.n);
  const int64_t nslots = (hi - lo) * st.a.d_min;
  const unsigned gs = unsigned(std::min<int64_t>((nslots + 255) / 256, 148 * 4));
  int32_t* ctr = round_counters(st, i);
  GANNS_TRY(launch_pdl(alloc_segments_kernel, gs, 256, 0, s, st.touched, st.indeg, st.segoff, ctr));
  GANNS_TRY(launch_pdl(scatter_edges_kernel, gs, 256, 0, s, st.Eu, st.Ed, nslots, st.a.d_min, lo,
                       st.segoff, st.fill, st.seg));
  const unsigned gm = unsigned(std::min<int64_t>((nslots + kMergeWarps - 1) / kMergeWarps, 148 * 16));
  GANNS_TRY(launch_pdl(round_merge_kernel<TPL>, gm, kMergeWarps * 32, 0, s, st.a.out_nbr, st.gdist,
                       st.a.d_max, st.touched, st.indeg, st.fill, st.segoff, st.seg, ctr,
                       round_counters(st, i + 1)));
  count_launch(3);
  return 0;
}

template <int TPL>
static int round_apply_t(BuildState& st, int64_t i, const int32_t* f_ids, const float* f_dists,
                         cudaStream_t s) {
  const int64_t lo = i * st.S, hi = std::min(lo + st.S, st.a.n);
  GANNS_TRY(launch_pdl(apply_forward_kernel, unsigned(std::min<int64_t>((hi - lo + 7) / 8, 148 * 8)),
                       256, 0, s, f_ids, f_dists, lo, hi, st.a.d_min, st.a.d_max, st.a.out_nbr,
                       st.gdist, st.Eu, st.Ed, st.indeg, st.touched, round_counters(st, i)));
  count_launch();
  return round_merge_t<TPL>(st, i, s);
}

template <int NV4, int TPL, bool L2>
static int begin_t(BuildState& st, cudaStream_t s) {
  GANNS_TRY(set_smem_attrs<NV4, TPL, L2>());
  BuildArgs& a = st.a;
  const int64_t n = a.n, S = a.group_size;
  const int dm = a.d_min, dmax = a.d_max;
  st.S = S;
  st.ngroups = (n + S - 1) / S;
  auto* ds = new (std::nothrow) BuildDevState();
  if (!ds) return fail(GANNS_ENOMEM, "host allocation failed");
  st.dev = ds;
  st.dev_free = [](void* p) { delete static_cast<BuildDevState*>(p); };
  auto alloc = [s](auto*& p, size_t count) {
    void* q = nullptr;
    cudaError_t e = pool_alloc(&q, std::max<size_t>(count, 1) * sizeof(*p), s);
    p = static_cast<std::remove_reference_t<decltype(p)>>(q);
    return e;
  };
  GANNS_TRY(alloc(st.gdist, size_t(n) * dmax));
  GANNS_TRY(alloc(st.gpid, size_t(n) * dm));
  GANNS_TRY(alloc(st.gpd, size_t(n) * dm));
  GANNS_TRY(alloc(st.Eu, size_t(S) * dm));
  GANNS_TRY(alloc(st.Ed, size_t(S) * dm));
  GANNS_TRY(alloc(st.indeg, size_t(n)));
  GANNS_TRY(alloc(st.fill, size_t(n)));
  GANNS_TRY(alloc(st.segoff, size_t(n)));
  GANNS_TRY(alloc(st.touched, size_t(S) * dm));
  GANNS_TRY(alloc(st.seg, size_t(S) * dm));
  GANNS_TRY(alloc(st.counters, 4));
  GANNS_TRY(cudaMemsetAsync(st.counters, 0, sizeof(int32_t) * 4, s));
  GANNS_TRY(alloc(st.stats, 3));
  GANNS_TRY(cudaMemsetAsync(st.indeg, 0, sizeof(int32_t) * n, s));
  GANNS_TRY(cudaMemsetAsync(st.fill, 0, sizeof(int32_t) * n, s));
  GANNS_TRY(cudaMemsetAsync(st.stats, 0, sizeof(unsigned long long) * 3, s));
  fill_rows_kernel<<<148 * 8, 256, 0, s>>>(a.out_nbr, st.gdist, n * dmax);
  fill_rows_kernel<<<148 * 8, 256, 0, s>>>(st.gpid, st.gpd, n * dm);
  count_launch(2);
  GANNS_TRY(cudaGetLastError());

  BuildDev& B = ds->B;
  B.g = GraphView{a.out_nbr, a.X, nullptr, n, dmax, a.d / 4, a.metric};
  B.g.prof = prof_buffer();
  GANNS_TRY(uses_tma(NV4) ? encode_row_tmap(a.X, n, a.d, &st.tmap) : zero_tmap(&st.tmap));
  B.gid = a.out_nbr;
  B.gdist = st.gdist;
  B.gpid = st.gpid;
  B.gpd = st.gpd;
  B.d_min = dm;
  B.l_build = a.l_build;
  B.e_build = a.e_build;
  B.l_local = a.l_local > 0 ? a.l_local : a.l_build;
  B.e_local = a.e_local > 0 ? a.e_local : a.e_build;
  B.stats = st.stats;
  // d > 256: rows per TMA round (1-D bulk copies); GANNS_BUILD_WROWS overrides the
  // default 8.  Fitting a round's searches into one wave of resident warps with
  // fewer rows per round was measured slower on C3 (3.12 s at R = 8 in 1.5 waves,
  // 3.17 s at R = 5, 3.31 s at R = 4): the second wave runs in the first one's
  // tail (a round lasts as long as its slowest search)
  static const int forced_wrows = [] {
    const char* e = std::getenv("GANNS_BUILD_WROWS");
    const int r = e ? std::atoi(e) : 0;
    return r >= 1 && r <= kWideStageRows ? r : kWideStageRows;
  }();
  B.wrows_p1 = B.wrows_p2 = forced_wrows;
  const size_t garea = kBuildGroup<NV4> ? group_area_bytes() : 0;
  ds->smem_p1 = size_t(kBuildWarps) * build_warp_bytes<NV4, TPL>(a.l_build, a.d / 4, B.wrows_p1) + garea;
  ds->smem_p2 = size_t(kBuildWarps) * build_warp_bytes<NV4, TPL>(a.l_build, a.d / 4, B.wrows_p2) + garea;
  if (std::max(ds->smem_p1, ds->smem_p2) > 227 * 1024)
    return fail(GANNS_ENOTSUP, "build: shared memory per CTA exceeds 227 KB");
  ds->U.top = a.upper.top;
  for (int j = 0; j < kMaxLayers; ++j) {
    ds->U.nbr[j] = a.upper.nbr[j];
    ds->U.n[j] = a.upper.n[j];
  }
  st.phase1 = phase1_t<NV4, TPL, L2>;
  st.round_search = round_search_t<NV4, TPL, L2>;
  st.round_merge = round_merge_t<TPL>;
  st.round_apply = round_apply_t<TPL>;
  return 0;
}

template <int NV4, int TPL>
static int begin_m(BuildState& st, cudaStream_t s) {
#ifdef GANNS_DEV_ONE
  return begin_t<NV4, TPL, true>(st, s);
#endif
  return st.a.metric == 0 ? begin_t<NV4, TPL, true>(st, s) : begin_t<NV4, TPL, false>(st, s);
}
template <int NV4>
int build_begin_nv(BuildState& st, cudaStream_t s) {
#ifdef GANNS_DEV_ONE
  return begin_m<NV4, 1>(st, s);
#endif
  switch (tpl_for(st.a.d_max)) {
    case 1: return begin_m<NV4, 1>(st, s);
    case 2: return begin_m<NV4, 2>(st, s);
    case 4: return begin_m<NV4, 4>(st, s);
  }
  return fail(GANNS_ENOTSUP, "unsupported degree");
}

template int build_begin_nv<GANNS_NV4>(BuildState&, cudaStream_t);

}  // namespace ganns
