// search_inst.cu -- K1 instantiations for one NV4 (= float4 per lane per row);
// compiled once per NV4 in {1, 2, 4, 8} with -DGANNS_NV4=... so the template
// instances build in parallel.  See ganns_dev.cuh for the algorithm.
#include "ganns_dev.cuh"
#include "ganns_internal.h"
#include "search_group.cuh"

#include <cstdlib>

#ifndef GANNS_NV4
#error "compile with -DGANNS_NV4=<1|2|4|8>"
#endif

namespace ganns {

#ifndef GANNS_PAIR_STAGES
#define GANNS_PAIR_STAGES 1
#endif
// 2 warps per CTA, 2-round form: a warp whose sibling has left takes over both
// stages (1 round per exploration) -- shortens the drain of a batch
constexpr bool kPairStages = GANNS_PAIR_STAGES != 0 && GANNS_SEARCH_WARPS % 2 == 0 &&
                             GANNS_SEARCH_ROUNDS == 2 && GANNS_SEARCH_POOL == 0;

// Persistent: every warp pulls queries from a per-launch ticket counter until
// the batch is exhausted, so the last wave is balanced at query granularity.
// HNSW (Section IV-D): each query first descends the upper layers
// greedily (the GANNS search with l = e = 1 per layer, over the permuted rows Xp)
// in the same warp, then searches layer 0 from perm[vertex reached] -- no separate
// entry kernel, and the descent's latency hides behind the other warps' searches.
struct HnswUpper {
  UpperLayers U;
  const float* Xp;
  int64_t np;
  const int32_t* perm;
  uint32_t* dstats;     // nullable [nq][2]: the descent's iterations, distance computations
};
template <int NV4, int TPL, bool L2, bool HNSW>
__global__ void __launch_bounds__(kSearchWarps * 32, NV4 == 1 ? kMinBlocksPerSM : kMinBlocksWide)
search_kernel(GraphView g, const float* __restrict__ Q, int64_t nq, int k, int l, int e,
              int32_t entry, int32_t* __restrict__ out_ids, float* __restrict__ out_dists,
              uint32_t* __restrict__ stats, int32_t* __restrict__ ticket,
              const int32_t* __restrict__ entries, int wrows, int solo,
              const __grid_constant__ CUtensorMap tmap, const __grid_constant__ HnswUpper H,
              const __grid_constant__ CUtensorMap tmap_up) {
  g.tmap = &tmap;
  extern __shared__ __align__(128) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpSmem ws;
  if constexpr (kSearchPool > 0) {
    ws = carve_pooled_smem(smem, w, kSearchWarps, kSearchPool, l, TPL, NV4, g.d4,
                           kSearchStageRounds);
    if (w == 0 && lane < kSearchPool) {
      mbar_init(ws.pool_mbar + lane, 1);
      ws.pool_owner[lane] = -1;
      ws.pool_phase[lane] = 0;
    }
    __syncthreads();
  } else if (kPairStages && uses_tma(NV4)) {
    // [stage 0 .. W-1][warp 0: N/mbar/bitmap .. warp W-1][one flag per warp pair];
    // each stage region also holds its warp's T (ganns_dev.cuh: t_bytes); warps
    // 2p and 2p+1 are partners with contiguous stages
    const size_t sb = stage_region_bytes(NV4, g.d4, kSearchStageRounds, TPL);
    const size_t rb = warp_tail_bytes(l);
    ws = carve_warp_smem(smem + size_t(w) * sb, l, TPL, NV4, g.d4, kSearchStageRounds);
    carve_warp_tail(ws, smem + kSearchWarps * sb + size_t(w) * rb, l);
    ws.pair_stage = reinterpret_cast<float4*>(smem + size_t(w & ~1) * sb);
    ws.pair_flag = reinterpret_cast<volatile int*>(smem + kSearchWarps * (sb + rb)) + (w >> 1);
    ws.pair_bar = 1 + (w >> 1);
    if (lane == 0 && (w & 1) == 0) *ws.pair_flag = 0;
    if (lane == 0) mbar_init(ws.mbar, 1);
    __syncthreads();
    if (solo && (w & 1)) {
      // latency mode (a batch that fits one wave at one query per CTA): the odd
      // warp hands its stage to its partner before taking any query, so every
      // query runs with one TMA round of 32 rows per exploration -- the same
      // hand-over as when the ticket runs out (below)
      fence_proxy_async_smem();
      __threadfence_block();
      if (lane == 0) atomicExch(const_cast<int*>(ws.pair_flag), 1);
      __syncwarp();
      pair_bar_arrive(ws.pair_bar);
      return;
    }
  } else {
    ws = carve_warp_smem(
        smem + size_t(w) * warp_smem_bytes(l, TPL, NV4, g.d4, kSearchStageRounds, wrows), l, TPL,
        NV4, g.d4, kSearchStageRounds, wrows);
    if (lane == 0) mbar_init(ws.mbar, 1);
    __syncwarp();
  }
  uint64_t* sN = ws.sN;
  for (;;) {
  int32_t qt = 0;
  if (lane == 0) qt = atomicAdd(ticket, 1);
  const int64_t q = __shfl_sync(kFull, qt, 0);
  if (q >= nq) {
    // this warp's stage is idle from now on: the sibling may take it over
    if (ws.pair_flag != nullptr && ws.rounds == 2) {
      // hand the stage to the sibling: this warp's last stage writes (its T) are
      // ordered before the sibling's TMA by the pair barrier (arrive here, sync
      // there when it takes the stage, or arrive when it leaves as well)
      fence_proxy_async_smem();
      __threadfence_block();
      if (lane == 0) atomicExch(const_cast<int*>(ws.pair_flag), 1);
      __syncwarp();
      pair_bar_arrive(ws.pair_bar);
    }
    break;
  }
  SearchStats st;
  const float* qrow = Q + size_t(q) * (g.d4 * 4);
  int32_t ent = entries != nullptr ? entries[q] : entry;   // HNSW: per-query entry
  if constexpr (HNSW) {
    GraphView gu = g;
    gu.X = H.Xp;
    gu.n = H.np;
    gu.tmap = &tmap_up;
    SearchStats ds{0u, 0u, 0u};
    ent = H.perm[descend<NV4, TPL, L2>(gu, H.U, 1, qrow, ws, H.dstats != nullptr ? &ds : nullptr)];
    if (H.dstats != nullptr && lane == 0) {
      H.dstats[size_t(q) * 2 + 0] = ds.iters;
      H.dstats[size_t(q) * 2 + 1] = ds.comps;
    }
  }
  const int cnt = warp_search<NV4, TPL, L2, false>(g, qrow, ent, l, e, ws, st);
  // output: the first k of N, (-1, +inf) padded (R-C8)
  for (int i = lane; i < k; i += 32) {
    uint64_t key = i < cnt ? unflag(sN[i]) : kKeyInf;
    bool empty = key_empty(key);
    out_ids[size_t(q) * k + i] = empty ? -1 : key_id(key);
    out_dists[size_t(q) * k + i] = empty ? __int_as_float(0x7f800000) : key_dist(key);
  }
  if (stats != nullptr && lane == 0) {
    stats[size_t(q) * 3 + 0] = st.iters;
    stats[size_t(q) * 3 + 1] = st.comps;
    stats[size_t(q) * 3 + 2] = st.merged;
  }
  __syncwarp();
  }
}

// Rows per TMA round of the wide form (d > 256): the largest R <= 8 whose
// resident warps hold the whole batch in one wave (a second, nearly empty wave
// would cost a full query latency); R = 8 when no R >= 4 fits.  GANNS_WIDE_ROWS
// overrides (developer knob).
template <int NV4, int TPL, bool L2>
static int pick_wide_rows(const SearchLaunch& a, int sms) {
  if (uses_tma(NV4)) return kWideStageRows;
  static const int forced = [] {
    const char* e = std::getenv("GANNS_WIDE_ROWS");
    return e ? std::atoi(e) : 0;
  }();
  if (forced >= 1 && forced <= kWideStageRows) return forced;
  for (int r = kWideStageRows; r >= 4; --r) {
    int per_sm = 0;
    const size_t smem = size_t(kSearchWarps) * warp_smem_bytes(a.l, TPL, NV4, a.d / 4,
                                                               kSearchStageRounds, r);
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, search_kernel<NV4, TPL, L2, false>,
                                                      kSearchWarps * 32, smem) != cudaSuccess)
      return kWideStageRows;
    if (int64_t(per_sm) * sms * kSearchWarps >= a.nq) return r;
  }
  return kWideStageRows;
}

// GANNS_SOLO=1 enables the latency mode (off by default: back-to-back small batches
// on several streams lose their overlap -- each solo batch holds most of the SMs'
// shared memory; measured 0.61 vs 0.89 per-GPU efficiency on the 8-way strong-scaling
// proxy, profiles/r02/ab_solo_latency_mode.log)
static bool solo_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("GANNS_SOLO");
    return e && e[0] == '1';
  }();
  return on;
}

template <int NV4, int TPL, bool L2, bool HNSW = false>
static cudaError_t launch_t(const SearchLaunch& a, cudaStream_t s) {
  auto kern = search_kernel<NV4, TPL, L2, HNSW>;
  static std::atomic<uint64_t> attr_done{0};   // per instantiation, per device
  {
    cudaError_t e = once_per_device(attr_done, [&] {
      cudaError_t r = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           227 * 1024);
      if (r == cudaSuccess)
        r = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
      return r;
    });
    if (e != cudaSuccess) return e;
  }
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int wrows = kSearchPool > 0 ? kWideStageRows : pick_wide_rows<NV4, TPL, L2>(a, sms);
  size_t smem = kSearchPool > 0
                    ? pooled_cta_bytes(a.l, TPL, NV4, a.d / 4, kSearchStageRounds, kSearchWarps,
                                       kSearchPool)
                : kPairStages && uses_tma(NV4)
                    ? kSearchWarps * (stage_region_bytes(NV4, a.d / 4, kSearchStageRounds, TPL) +
                                      warp_tail_bytes(a.l)) +
                          ((kSearchWarps / 2 * 4 + 15) & ~15)
                    : size_t(kSearchWarps) *
                          warp_smem_bytes(a.l, TPL, NV4, a.d / 4, kSearchStageRounds, wrows);
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  {
    // developer knob (occupancy experiments): extra shared memory per CTA
    static const long pad = [] {
      const char* e = std::getenv("GANNS_DEBUG_SEARCH_SMEM_PAD");
      return e ? std::atol(e) : 0L;
    }();
    smem += size_t(pad);
  }
  GraphView g{a.nbr, a.X, nullptr, a.n, a.d_max, a.d / 4, a.metric};
  g.prof = prof_buffer();
  CUtensorMap tmap;
  cudaError_t err = uses_tma(NV4) ? encode_row_tmap(a.X, a.n, a.d, &tmap) : zero_tmap(&tmap);
  if (err != cudaSuccess) return err;
  HnswUpper H{};
  CUtensorMap tmap_up;
  err = zero_tmap(&tmap_up);
  if (err != cudaSuccess) return err;
  if constexpr (HNSW) {
    H.U.top = a.upper->top;
    for (int j = 0; j < kMaxLayers; ++j) {
      H.U.nbr[j] = a.upper->nbr[j];
      H.U.n[j] = a.upper->n[j];
    }
    H.Xp = a.Xp;
    H.np = a.np;
    H.perm = a.perm;
    H.dstats = a.dstats;
    err = encode_row_tmap(a.Xp, a.np, a.d, &tmap_up);
    if (err != cudaSuccess) return err;
  }
  err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kSearchWarps * 32, smem);
  if (err != cudaSuccess) return err;
  int64_t blocks = (a.nq + kSearchWarps - 1) / kSearchWarps;
  const int64_t resident = int64_t(sms) * (per_sm > 0 ? per_sm : 1);
  // latency mode: when one query per CTA fits in one wave, give each query both
  // stages of its CTA (one TMA round per exploration, shorter per-query latency)
  const int solo = kPairStages && uses_tma(NV4) && solo_enabled() && a.nq <= resident ? 1 : 0;
  if (solo) blocks = a.nq;
  if (blocks > resident) blocks = resident;
  err = cudaMemsetAsync(a.ticket, 0, sizeof(int32_t), s);
  if (err != cudaSuccess) return err;
  kern<<<dim3(unsigned(blocks)), kSearchWarps * 32, smem, s>>>(
      g, a.Q, a.nq, a.k, a.l, a.e, a.entry, a.out_ids, a.out_dists, a.stats, a.ticket, a.entries,
      wrows, solo, tmap, H, tmap_up);
  count_launch();
  return cudaGetLastError();
}

// Wide rows (d > 256): a warp group per query (search_group.cuh).  The rows per
// TMA round R are picked as for the one-warp form (largest R <= 8 that holds the
// batch in one wave).  GANNS_WIDE_GROUP=0 selects the one-warp form (A/B knob).
static bool wide_group_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("GANNS_WIDE_GROUP");
    return !(e && e[0] == '0');
  }();
  return on;
}

template <int CG, int TPL, bool L2>
static cudaError_t launch_group_t(const SearchLaunch& a, cudaStream_t s) {
  auto kern = search_group_kernel<CG, TPL, L2>;
  static std::atomic<uint64_t> attr_done{0};   // per instantiation, per device
  {
    cudaError_t e = once_per_device(attr_done, [&] {
      cudaError_t r = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           227 * 1024);
      if (r == cudaSuccess)
        r = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
      return r;
    });
    if (e != cudaSuccess) return e;
  }
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int d4 = a.d / 4;
  auto smem_for = [&](int r) {
    return warp_smem_bytes(a.l, TPL, 8, d4, 1, r) + group_area_bytes();
  };
  static const int forced = [] {
    const char* e = std::getenv("GANNS_WIDE_ROWS");
    return e ? std::atoi(e) : 0;
  }();
  int wrows = kWideStageRows;
  if (forced >= 1 && forced <= kWideStageRows) {
    wrows = forced;
  } else {
    for (int r = kWideStageRows; r >= 4; --r) {
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kGroupWarps * 32,
                                                        smem_for(r)) != cudaSuccess)
        break;
      if (int64_t(per_sm) * sms >= a.nq) {
        wrows = r;
        break;
      }
    }
  }
  const size_t smem = smem_for(wrows);
  if (smem > 227 * 1024) return cudaErrorInvalidValue;
  GraphView g{a.nbr, a.X, nullptr, a.n, a.d_max, d4, a.metric};
  g.prof = prof_buffer();
  cudaError_t err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kGroupWarps * 32, smem);
  if (err != cudaSuccess) return err;
  int64_t blocks = a.nq;
  const int64_t resident = int64_t(sms) * (per_sm > 0 ? per_sm : 1);
  if (blocks > resident) blocks = resident;
  err = cudaMemsetAsync(a.ticket, 0, sizeof(int32_t), s);
  if (err != cudaSuccess) return err;
  kern<<<dim3(unsigned(blocks)), kGroupWarps * 32, smem, s>>>(
      g, a.Q, a.nq, a.k, a.l, a.e, a.entry, a.out_ids, a.out_dists, a.stats, a.ticket, a.entries,
      wrows);
  count_launch();
  return cudaGetLastError();
}

template <int NV4, int TPL>
static cudaError_t launch_m(const SearchLaunch& a, cudaStream_t s) {
#if GANNS_NV4 >= 4
  if (wide_group_enabled())
    return a.metric == 0 ? launch_group_t<NV4 / 4, TPL, true>(a, s)
                         : launch_group_t<NV4 / 4, TPL, false>(a, s);
#endif
#ifdef GANNS_DEV_ONE
  return launch_t<NV4, TPL, true>(a, s);
#endif
  if constexpr (uses_tma(NV4))
    if (a.upper != nullptr && a.upper->top > 0)
      return a.metric == 0 ? launch_t<NV4, TPL, true, true>(a, s)
                           : launch_t<NV4, TPL, false, true>(a, s);
  return a.metric == 0 ? launch_t<NV4, TPL, true>(a, s) : launch_t<NV4, TPL, false>(a, s);
}
template <int NV4>
cudaError_t launch_search_nv(const SearchLaunch& a, cudaStream_t s) {
#ifdef GANNS_DEV_ONE
  return launch_m<NV4, 1>(a, s);
#endif
  switch (tpl_for(a.d_max)) {
    case 1: return launch_m<NV4, 1>(a, s);
    case 2: return launch_m<NV4, 2>(a, s);
    case 4: return launch_m<NV4, 4>(a, s);
  }
  return cudaErrorInvalidValue;
}

template cudaError_t launch_search_nv<GANNS_NV4>(const SearchLaunch&, cudaStream_t);

// HNSW query entries: one warp per query descends the upper layers
// greedily (GANNS with l = e = 1 per layer) over the permuted points and writes
// the layer-0 entry perm[reached vertex].
template <int NV4, int TPL, bool L2>
__global__ void __launch_bounds__(kSearchWarps * 32)
hnsw_entry_kernel(GraphView g, const UpperLayers U, const float* __restrict__ Q, int64_t nq,
                  const int32_t* __restrict__ perm, int32_t* __restrict__ entries,
                  uint32_t* __restrict__ dstats, const __grid_constant__ CUtensorMap tmap) {
  extern __shared__ __align__(128) uint8_t smem[];
  g.tmap = &tmap;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpSmem ws = carve_warp_smem(
      smem + size_t(w) * warp_smem_bytes(1, TPL, NV4, g.d4, kSearchStageRounds), 1, TPL, NV4, g.d4,
      kSearchStageRounds);
  if (lane == 0) mbar_init(ws.mbar, 1);
  __syncwarp();
  const int64_t q = int64_t(blockIdx.x) * kSearchWarps + w;
  if (q >= nq) return;
  SearchStats ds{0u, 0u, 0u};
  const int32_t c = descend<NV4, TPL, L2>(g, U, 1, Q + size_t(q) * (g.d4 * 4), ws,
                                          dstats != nullptr ? &ds : nullptr);
  if (lane == 0) {
    entries[q] = perm[c];
    if (dstats != nullptr) {
      dstats[size_t(q) * 2 + 0] = ds.iters;
      dstats[size_t(q) * 2 + 1] = ds.comps;
    }
  }
}

template <int NV4, int TPL, bool L2>
static cudaError_t entries_t(const EntryLaunch& a, cudaStream_t s) {
  auto kern = hnsw_entry_kernel<NV4, TPL, L2>;
  const size_t smem = size_t(kSearchWarps) * warp_smem_bytes(1, TPL, NV4, a.d / 4, kSearchStageRounds);
  cudaError_t err = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (err != cudaSuccess) return err;
  GraphView g{nullptr, a.Xp, nullptr, a.np, a.d_max, a.d / 4, a.metric};
  CUtensorMap tmap;
  err = uses_tma(NV4) ? encode_row_tmap(a.Xp, a.np, a.d, &tmap) : zero_tmap(&tmap);
  if (err != cudaSuccess) return err;
  UpperLayers U;
  U.top = a.upper.top;
  for (int j = 0; j < kMaxLayers; ++j) {
    U.nbr[j] = a.upper.nbr[j];
    U.n[j] = a.upper.n[j];
  }
  const int64_t blocks = (a.nq + kSearchWarps - 1) / kSearchWarps;
  kern<<<unsigned(blocks), kSearchWarps * 32, smem, s>>>(g, U, a.Q, a.nq, a.perm, a.entries,
                                                        a.dstats, tmap);
  count_launch();
  return cudaGetLastError();
}

template <int NV4>
cudaError_t launch_entries_nv(const EntryLaunch& a, cudaStream_t s) {
  const bool l2 = a.metric == 0;
  switch (tpl_for(a.d_max)) {
    case 1: return l2 ? entries_t<NV4, 1, true>(a, s) : entries_t<NV4, 1, false>(a, s);
#ifndef GANNS_DEV_ONE
    case 2: return l2 ? entries_t<NV4, 2, true>(a, s) : entries_t<NV4, 2, false>(a, s);
    case 4: return l2 ? entries_t<NV4, 4, true>(a, s) : entries_t<NV4, 4, false>(a, s);
#endif
  }
  return cudaErrorInvalidValue;
}

template cudaError_t launch_entries_nv<GANNS_NV4>(const EntryLaunch&, cudaStream_t);


}  // namespace ganns
