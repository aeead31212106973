// ganns_dev.cuh -- device side of the GANNS search (§III-B),
// shared by the batched search kernel (search.cu) and the GGraphCon build kernels
// (build.cu).  sm_100a only.
//
// One warp owns one query (the paper's "thread block per query" with n_t = 32
// threads, R-C20).  Per query the warp keeps, in shared memory:
//   sN  : candidate array N, up to l packed keys (lazy update), ascending
//   sT  : the surviving visiting entries T, compacted in sorted order;
//         it lives inside the TMA stage (idle during the merge)
//   sBM : a bitmap of the positions of N that T entries land on in the merge
// A key is (orderable fp32 distance << 32) | id; bit 31 of the id word is the
// "explored" flag, so the flag travels with its entry through the merge.
// The visiting array T lives in registers: lane j holds the j-th neighbour of
// the exploring vertex (TPL = ceil(d_max/32) slots per lane).
//
// Per iteration (the paper's six phases, Fig. 3):
//   (1) candidate locating  -- __ballot_sync / __ffs over 32-entry chunks of N
//       from a "first possibly unexplored" hint
//   (2) neighbourhood exploration -- one coalesced load of the adjacency row
//   (3) bulk distance -- the neighbour rows gathered by TMA (tile::gather4, or
//       1-D bulk copies) into the warp's shared-memory stage, all rows of a round
//       in flight on one mbarrier; partial sums reduced by a transposing butterfly
//       so lane j ends with delta(q, T[j])
//   (4) lazy check -- entries that cannot enter N (>= its l-th key when full)
//       are skipped; the rest binary-search N; equal key => duplicate, dropped
//       (R-C1).  The probe gives rank_N(t) for free.
//   (5) sort -- rank of each surviving entry among the survivors (R-C2 order);
//       this yields the sorted order of T without moving data
//   (6) merge -- position(t) = rank_N(t) + rank_T(t); N is rebuilt in place from
//       the position bitmap, from the last chunk down to the first changed one
//       (P:210-212).  Duplicates never reach the merge.
#pragma once
#include <cuda.h>   // CUtensorMap (type only; the map is encoded on the host)
#include <cstdint>
#include <cuda_runtime.h>

namespace ganns {

constexpr uint32_t kExplored = 0x80000000u;
constexpr uint64_t kKeyInf = ~0ull;
constexpr unsigned kFull = 0xffffffffu;

// fp32 -> uint32 preserving order (negative values flipped); +0 canonical.
__device__ __forceinline__ uint32_t f2o(float f) {
  uint32_t b = __float_as_uint(f);
  return b ^ (uint32_t(int32_t(b) >> 31) | 0x80000000u);
}
__device__ __forceinline__ float o2f(uint32_t o) {
  uint32_t b = (o & 0x80000000u) ? (o ^ 0x80000000u) : ~o;
  return __uint_as_float(b);
}
__device__ __forceinline__ uint64_t mkkey(float d, int32_t id) {
  return (uint64_t(f2o(d)) << 32) | uint32_t(id);
}
__device__ __forceinline__ uint64_t unflag(uint64_t k) { return k & ~uint64_t(kExplored); }
__device__ __forceinline__ int32_t key_id(uint64_t k) { return int32_t(uint32_t(k) & 0x7fffffffu); }
__device__ __forceinline__ float key_dist(uint64_t k) { return o2f(uint32_t(k >> 32)); }
__device__ __forceinline__ bool key_empty(uint64_t k) { return uint32_t(k >> 32) == 0xffffffffu; }

__device__ __forceinline__ uint64_t shfl64(uint64_t v, int src) {
  uint32_t lo = __shfl_sync(kFull, uint32_t(v), src);
  uint32_t hi = __shfl_sync(kFull, uint32_t(v >> 32), src);
  return (uint64_t(hi) << 32) | lo;
}
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
// Bulk L2 prefetch of one vector row (TMA unit, no registers held): issued for
// every neighbour as soon as the adjacency row arrives, so the register-staged
// loads of the bulk-distance passes find their lines in L2.
__device__ __forceinline__ void prefetch_row_l2(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(p), "r"(bytes) : "memory");
}
// ---- TMA (cp.async.bulk) + mbarrier helpers (sm_90+; SASS UBLKCP / SYNCS)
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return uint32_t(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* m, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t phase) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done) : "r"(smem_u32(m)), "r"(phase) : "memory");
  } while (!done);
}
// 1-D bulk copy global -> shared, completion counted on mbarrier m (bytes % 16 == 0)
__device__ __forceinline__ void tma_row(void* dst, const void* src, uint32_t bytes, uint64_t* m) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(m))
      : "memory");
}
// Shared-memory 128-bit load kept in program order (bounds register pressure:
// ptxas may not hoist all passes' loads of a round ahead of their math).
__device__ __forceinline__ float4 lds128_ordered(const float4* p) {
  float4 r;
  asm volatile("ld.volatile.shared.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "r"(smem_u32(p)));
  return r;
}
// stage hand-over of a warp pair (named barrier `id`, the pair's 64 threads)
// (non-.aligned forms: the two warps reach the barrier through different instructions)
__device__ __forceinline__ void pair_bar_arrive(int id) {
  __syncwarp();
  asm volatile("barrier.arrive %0, 64;" ::"r"(id) : "memory");
}
__device__ __forceinline__ void pair_bar_sync(int id) {
  __syncwarp();
  asm volatile("barrier.sync %0, 64;" ::"r"(id) : "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

template <bool COHERENT>
__device__ __forceinline__ int32_t load_nbr(const int32_t* p) {
  if constexpr (COHERENT) return *reinterpret_cast<const volatile int32_t*>(p);
  else return __ldg(p);
}

// Everything a warp needs to search one graph.
struct GraphView {
  const int32_t* nbr;   // [n][d_max] ids, -1 padded
  const float* X;       // [n][d]
  const CUtensorMap* tmap;   // 2-D map of X (box = 1 row) for TMA tile::gather4; the
                             // address of the launching kernel's __grid_constant__ param
  int64_t n;
  int d_max;
  int d4;               // d / 4
  int metric;           // 0 L2, 1 IP, 2 COSINE
  // GANNS_PROFILE builds: per-phase cycle counters (ganns_profile_read), else null
  unsigned long long* prof = nullptr;
};

// Per-phase timers of the search loop (the analogue of the paper's time
// breakdowns, Fig. 7, Fig. 10).  Compiled in only with -DGANNS_PROFILE=1
// (a separate library build): lane 0 of each warp reads clock64() at the phase
// boundaries and adds the cycles to prof[0..5] = candidate locating, neighbourhood
// exploration (adjacency row), bulk distance (gather + math), lazy check, sort,
// merge; prof[6] = iterations, prof[7] = searches; inside the bulk distance
// prof[8] = cycles from the start of a gather to its last TMA issue, prof[9] =
// cycles waiting on the gather's mbarrier, prof[10] = TMA rounds; prof[11] =
// explorations whose adjacency row the speculation had already loaded; prof[12] /
// prof[13] = the largest cycles / iterations of one search (max, not sum).
#ifndef GANNS_PROFILE
#define GANNS_PROFILE 0
#endif
enum { kProfLocate = 0, kProfExplore, kProfDistance, kProfLazy, kProfSort, kProfMerge };


// Per-search counters (kept in registers, identical to the oracle's stats[0,1,3]).
struct SearchStats {
  uint32_t iters, comps, merged;
};

// Per-warp shared memory: [stage: 32 vector rows, TMA destination][N][T][mbar][bitmap]
__host__ __device__ constexpr int lpad32(int l) { return (l + 31) & ~31; }
// uses_tma: the tile::gather4 tensor map is used (d <= 256: the map's box is one
// row of <= 256 elements); wider rows are staged with 1-D bulk copies.
__host__ __device__ constexpr bool uses_tma(int nv4) { return nv4 <= 2; }
constexpr int kWideStageRows = 8;   // d > 256: rows per TMA round (4 rounds per exploration)
// The <= 32 rows of one exploration are staged in `rounds` TMA rounds (1 or 2):
// 2 rounds halve the stage (more resident warps, the throughput-bound batched
// search); 1 round saves a memory round trip (the latency-bound build).
#ifndef GANNS_SEARCH_ROUNDS
#define GANNS_SEARCH_ROUNDS 2
#endif
// GANNS_LATE_FENCE: the segment form's TMA rounds are issued without a proxy
// fence (the stage's earlier generic READS are complete: their values were
// consumed before the issue); the only generic WRITES to the stage (T, by the
// merge) are followed by fence.proxy.async right after the merge.  Keeps the
// fence's MEMBAR off the gather's issue path.
#ifndef GANNS_LATE_FENCE
#define GANNS_LATE_FENCE 1
#endif
// GANNS_SKIP_LB: an exploration none of whose neighbours is below N's l-th key
// skips the lazy check's binary searches (nothing can enter N)
#ifndef GANNS_SKIP_LB
#define GANNS_SKIP_LB 1
#endif
// GANNS_LB_PRELOAD: load N's l-th key and the lazy check's first probes before the
// bulk-distance gather (their latency hides under it)
#ifndef GANNS_LB_PRELOAD
#define GANNS_LB_PRELOAD 1
#endif
#ifndef GANNS_PREFETCH_R2
#define GANNS_PREFETCH_R2 0
#endif
// GANNS_WIDE_HINT: d > 256 -- warm the later TMA rounds' rows in L2 at exploration
// start.  Off: on C3 (1M x 960) the prefetched rows are evicted before their TMA
// round reads them (~95 MB of prefetches in flight vs the 126 MB L2) -- with the hint
// 37.4 GB of DRAM reads per 1K-query step (1.09 x algorithmic) and 189.6K QPS,
// without it 31.4 GB (0.92 x) and 222.4K QPS (profiles/r02/ab_c3_wide_hint.log)
#ifndef GANNS_WIDE_HINT
#define GANNS_WIDE_HINT 0
#endif
constexpr int kSearchStageRounds = GANNS_SEARCH_ROUNDS;
constexpr int kBuildStageRounds = 1;
// wrows: rows per TMA round of the wide (d > 256) form, 1..kWideStageRows (the
// search launcher lowers it so that a small batch fits one wave of warps)
__host__ __device__ constexpr size_t stage_bytes(int nv4, int d4, int rounds,
                                                 int wrows = kWideStageRows) {
  return uses_tma(nv4) ? size_t(32 / rounds) * d4 * 16 : size_t(wrows) * d4 * 16;
}
// T (the surviving visiting entries, written and read only by the merge) lives
// in the stage: the stage is idle from the end of an exploration's distance math
// to the next exploration's first TMA round (whose issue is preceded by a
// proxy fence).  The stage region is therefore at least T's size.
__host__ __device__ constexpr size_t t_bytes(int tpl) { return size_t(tpl) * 32 * 8; }
__host__ __device__ constexpr size_t stage_region_bytes(int nv4, int d4, int rounds, int tpl,
                                                        int wrows = kWideStageRows) {
  return stage_bytes(nv4, d4, rounds, wrows) > t_bytes(tpl) ? stage_bytes(nv4, d4, rounds, wrows)
                                                           : t_bytes(tpl);
}
// the rest of a warp's area: N (lpad32(l) keys), the mbarrier (16 B), the merge
// bitmap (lpad32(l) bits, 16-B rounded); a multiple of 16 B
__host__ __device__ constexpr size_t warp_tail_bytes(int l) {
  return size_t(lpad32(l)) * 8 + 16 + ((size_t(lpad32(l) / 32) * 4 + 15) & ~size_t(15));
}
__host__ __device__ constexpr size_t warp_smem_bytes(int l, int tpl, int nv4, int d4, int rounds,
                                                     int wrows = kWideStageRows) {
  // rounded to 128 B: the stage (first) must be 128-B aligned for tensor TMA
  return (stage_region_bytes(nv4, d4, rounds, tpl, wrows) + warp_tail_bytes(l) + 127) &
         ~size_t(127);
}
struct WarpSmem {
  float4* stage;
  uint64_t* sN;
  uint64_t* sT;
  uint64_t* mbar;
  uint32_t* sBM;
  uint32_t phase;   // parity of the next mbarrier phase to wait for
  int rounds;       // TMA rounds per exploration (1 or 2)
  int wrows;        // wide form: rows per TMA round (1..kWideStageRows)
  // CTA-shared stage pool (pool > 0): a warp holds a stage buffer only from its
  // gather to the end of its distance math, so fewer buffers than warps suffice
  int pool;
  float4* pool_stage;       // pool buffers, pool_stride bytes apart
  uint32_t pool_stride;
  uint64_t* pool_mbar;      // one mbarrier per buffer
  int* pool_owner;          // -1 = free
  uint32_t* pool_phase;     // parity of each buffer's next phase
  int held;                 // buffer held by this warp, -1 = none
  // stage pairing (search kernel, 2 warps per CTA, 2-round form): the CTA's two
  // stages are contiguous at pair_stage; once the sibling warp has left (*pair_flag
  // != 0) this warp switches to 1 round of 32 rows over both stages -- one memory
  // round trip per exploration for the last queries of a batch
  float4* pair_stage;
  volatile int* pair_flag;
  int pair_bar;   // named barrier of the pair (64 threads): leaver arrives, taker syncs
#if GANNS_PROFILE
  unsigned long long p_issue = 0, p_wait = 0, p_rounds = 0;   // lane 0's gather timers
#endif
};
// Per-CTA layout of the pooled search kernel: [pool stages][per-warp N/T/bitmap][pool meta]
__host__ __device__ constexpr size_t pooled_warp_bytes(int l, int tpl) {
  return (size_t(lpad32(l)) * 8 + size_t(tpl) * 32 * 8 + 16 + 128 + 15) & ~size_t(15);
}
__host__ __device__ constexpr size_t pooled_cta_bytes(int l, int tpl, int nv4, int d4, int rounds,
                                                      int warps, int pool) {
  return size_t(pool) * stage_bytes(nv4, d4, rounds) + size_t(warps) * pooled_warp_bytes(l, tpl) +
         size_t(pool) * 16;
}
// N, mbarrier and bitmap of a warp at `tail` (16-B aligned, warp_tail_bytes(l))
__device__ __forceinline__ void carve_warp_tail(WarpSmem& w, uint8_t* tail, int l) {
  w.sN = reinterpret_cast<uint64_t*>(tail);
  w.mbar = w.sN + lpad32(l);
  w.sBM = reinterpret_cast<uint32_t*>(w.mbar + 2);
}
__device__ __forceinline__ WarpSmem carve_warp_smem(uint8_t* base, int l, int tpl, int nv4, int d4,
                                                   int rounds, int wrows = kWideStageRows) {
  WarpSmem w;
  w.rounds = rounds;
  w.wrows = wrows;
  w.stage = reinterpret_cast<float4*>(base);
  w.sT = reinterpret_cast<uint64_t*>(base);   // shares the stage (see t_bytes)
  carve_warp_tail(w, base + stage_region_bytes(nv4, d4, rounds, tpl, wrows), l);
  w.phase = 0;
  w.pool = 0;
  w.held = -1;
  w.pair_stage = nullptr;
  w.pair_flag = nullptr;
  return w;
}
// pooled layout: warp w of `warps`; lane 0 of warp 0 initialises the pool
__device__ __forceinline__ WarpSmem carve_pooled_smem(uint8_t* cta, int w, int warps, int pool, int l,
                                                     int tpl, int nv4, int d4, int rounds) {
  WarpSmem s;
  s.rounds = rounds;
  s.wrows = kWideStageRows;
  const size_t sb = stage_bytes(nv4, d4, rounds);
  s.pool = pool;
  s.pool_stage = reinterpret_cast<float4*>(cta);
  s.pool_stride = uint32_t(sb);
  uint8_t* wb = cta + size_t(pool) * sb + size_t(w) * pooled_warp_bytes(l, tpl);
  s.sN = reinterpret_cast<uint64_t*>(wb);
  s.sT = s.sN + lpad32(l);
  s.mbar = nullptr;
  s.sBM = reinterpret_cast<uint32_t*>(s.sT + tpl * 32 + 2);
  uint8_t* meta = cta + size_t(pool) * sb + size_t(warps) * pooled_warp_bytes(l, tpl);
  s.pool_mbar = reinterpret_cast<uint64_t*>(meta);
  s.pool_owner = reinterpret_cast<int*>(s.pool_mbar + pool);
  s.pool_phase = reinterpret_cast<uint32_t*>(s.pool_owner + pool);
  s.stage = nullptr;
  s.phase = 0;
  s.held = -1;
  s.pair_stage = nullptr;
  s.pair_flag = nullptr;
  return s;
}
// acquire a free pool buffer (lane 0 spins on the owner words), make it current
__device__ __forceinline__ void stage_acquire(WarpSmem& ws, int lane) {
  if (ws.pool == 0) return;
  int b = -1;
  if (lane == 0) {
    const int me = int(threadIdx.x >> 5);
    for (;;) {
      for (int i = 0; i < ws.pool && b < 0; ++i)
        if (atomicCAS(&ws.pool_owner[i], -1, me) == -1) b = i;
      if (b >= 0) break;
      __nanosleep(64);
    }
    __threadfence_block();
  }
  b = __shfl_sync(kFull, b, 0);
  __syncwarp();
  ws.held = b;
  ws.stage = reinterpret_cast<float4*>(reinterpret_cast<char*>(ws.pool_stage) + size_t(b) * ws.pool_stride);
  ws.mbar = ws.pool_mbar + b;
  ws.phase = ws.pool_phase[b];
}
__device__ __forceinline__ void stage_release(WarpSmem& ws, int lane) {
  if (ws.pool == 0) return;
  __syncwarp();   // every lane's reads of the stage are done
  if (lane == 0) {
    ws.pool_phase[ws.held] = ws.phase;
    __threadfence_block();
    atomicExch(&ws.pool_owner[ws.held], -1);
  }
  __syncwarp();
  ws.held = -1;
}

// Vector layout per dimension bucket (NV4 = template selector, see nv4_for):
// S lanes share one row, each lane owning C float4 columns (i4 = lane%S + S*f).
// d <= 128: 8 lanes x 4 float4 per row, so one warp-wide 128-bit load covers 4
// rows (each 128 B-coalesced) and 8 rows are in flight per lane per group pass.
template <int NV4> struct VecLayout;
template <> struct VecLayout<1> { static constexpr int S = 8, C = 4; };    // d <= 128
template <> struct VecLayout<2> { static constexpr int S = 16, C = 4; };   // d <= 256
template <> struct VecLayout<4> { static constexpr int S = 32, C = 4; };   // d <= 512
template <> struct VecLayout<8> { static constexpr int S = 32, C = 8; };   // d <= 1024

// Packed fp32x2 arithmetic (sm_100a FADD2 / FFMA2): one instruction per two
// lanes of a float4, halving the FP instruction count of the bulk distance.
// The two halves are summed at the end (the order of an fp32 sum; exact on the
// integer-grid inputs, R-C18).
__device__ __forceinline__ uint64_t pk2(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ float hsum2(uint64_t v) {
  float lo, hi;
  asm("mov.b64 {%0,%1}, %2;" : "=f"(lo), "=f"(hi) : "l"(v));
  return lo + hi;
}
template <bool L2>
__device__ __forceinline__ uint64_t accum4(uint64_t acc, const float4& q, const float4& x) {
  const uint64_t qa = pk2(q.x, q.y), qb = pk2(q.z, q.w);
  const uint64_t xa = pk2(x.x, x.y), xb = pk2(x.z, x.w);
  if constexpr (L2) {
    uint64_t ta, tb;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(ta) : "l"(qa), "l"(xa));
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(tb) : "l"(qb), "l"(xb));
    asm("fma.rn.f32x2 %0, %1, %1, %0;" : "+l"(acc) : "l"(ta));
    asm("fma.rn.f32x2 %0, %1, %1, %0;" : "+l"(acc) : "l"(tb));
  } else {
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(qa), "l"(xa));
    asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(qb), "l"(xb));
  }
  return acc;
}

// Bulk distance for the <= 32 neighbours held one per lane (u_mine,
// -1 = none): returns, in lane j, the raw sum for u_j (L2: squared distance,
// IP/COSINE: dot product).
// Math layout: S-lane segments; in pass g segment s works on the row of lane
// g + S*s (its 8 lanes read 128 B contiguous from shared memory, conflict-free);
// after S passes a transposing butterfly inside the segment leaves lane j with
// row j's total.
// Gather: the rows of the passes of one round are fetched by TMA bulk copies
// (one cp.async.bulk per lane that owns a row of the round) into the warp's
// stage buffer and waited for with a single mbarrier phase -- ROUNDS memory
// round trips per iteration, no registers held in flight.
template <int S, int C, bool L2, bool FULL, int ROUNDS>
__device__ __forceinline__ float tma_dot(const GraphView& g, const float4 (&qv)[C],
                                         int32_t u_mine, int lane, WarpSmem& ws) {
  static_assert(S % ROUNDS == 0, "passes must split evenly into rounds");
  constexpr int PPR = S / ROUNDS;                   // passes per round
  const int sl = lane & (S - 1), seg = lane / S;
  const uint32_t rowbytes = uint32_t(g.d4) * 16u;
  // lane j = g + S*s holds the row of pass g of segment s; it is staged in round
  // g / PPR at slot (g % PPR) + PPR*s
  const int my_round = sl / PPR;
  const int my_slot = sl % PPR + PPR * seg;
  int coff[C];
#pragma unroll
  for (int f = 0; f < C; ++f) coff[f] = (FULL || sl + S * f < g.d4) ? sl + S * f : g.d4 - 1;
  float p[S];
#if GANNS_PREFETCH_R2
  // rows of the later rounds start towards L2 now (no extra traffic: they are read
  // by this exploration's next TMA round)
  if constexpr (ROUNDS > 1)
    if (u_mine >= 0 && my_round > 0)
      prefetch_row_l2(reinterpret_cast<const char*>(g.X) + uint64_t(uint32_t(u_mine)) * rowbytes,
                      rowbytes);
#endif
  stage_acquire(ws, lane);
#pragma unroll
  for (int r = 0; r < ROUNDS; ++r) {
#if GANNS_PROFILE
    const long long t_g0 = clock64();
#endif
    // tile::gather4 (d % 8 == 0, so every group of 4 rows starts 128-B aligned):
    // lane 4m of this round fetches the rows of lanes 4m..4m+3 into 4 consecutive
    // stage slots with ONE TMA instruction; absent neighbours get an out-of-range
    // row coordinate (zero-filled, no memory traffic).  Otherwise one 1-D bulk
    // copy per row.
    const bool g4 = (g.d4 & 1) == 0;
    const int32_t uo = u_mine >= 0 ? u_mine : 0x7fffffff;
    // rows of stage slots my_slot+1..+3 of this round: with >= 4 passes per round
    // they belong to the next 3 lanes; otherwise to lane r*PPR + k%PPR + S*(k/PPR)
    int32_t u1, u2, u3;
    if constexpr (PPR % 4 == 0) {
      u1 = __shfl_down_sync(kFull, uo, 1);
      u2 = __shfl_down_sync(kFull, uo, 2);
      u3 = __shfl_down_sync(kFull, uo, 3);
    } else {
      auto lane_of = [r](int k) { return r * PPR + k % PPR + S * (k / PPR); };
      u1 = __shfl_sync(kFull, uo, lane_of((my_slot + 1) & 31));
      u2 = __shfl_sync(kFull, uo, lane_of((my_slot + 2) & 31));
      u3 = __shfl_sync(kFull, uo, lane_of((my_slot + 3) & 31));
    }
    const bool issuer = g4 ? ((my_slot & 3) == 0 && my_round == r && (uo & u1 & u2 & u3) != 0x7fffffff)
                           : (u_mine >= 0 && my_round == r);
    const unsigned vm = __ballot_sync(kFull, issuer);
    if (vm) {
      __syncwarp();
#if !GANNS_LATE_FENCE
      fence_proxy_async_smem();   // earlier generic accesses of the stage precede the async writes
#endif
      if (lane == 0)
        mbar_arrive_expect_tx(ws.mbar, uint32_t(__popc(vm)) * (g4 ? 4u : 1u) * rowbytes);
      __syncwarp();
      char* dst = reinterpret_cast<char*>(ws.stage) + size_t(my_slot) * rowbytes;
      if (issuer) {
        if (g4)
          asm volatile(
              "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
              " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(smem_u32(dst)),
              "l"(g.tmap), "r"(0), "r"(uo), "r"(u1), "r"(u2), "r"(u3), "r"(smem_u32(ws.mbar))
              : "memory");
        else
          tma_row(dst, reinterpret_cast<const char*>(g.X) + uint64_t(uint32_t(u_mine)) * rowbytes,
                  rowbytes, ws.mbar);
      }
#if GANNS_PROFILE
      const long long t_g1 = clock64();
#endif
      mbar_wait(ws.mbar, ws.phase);
      ws.phase ^= 1u;
#if GANNS_PROFILE
      const long long t_g2 = clock64();
      ws.p_issue += t_g1 - t_g0;
      ws.p_wait += t_g2 - t_g1;
      ws.p_rounds += 1;
#endif
    }
#pragma unroll
    for (int gg = 0; gg < PPR; ++gg) {
      const float4* rp = ws.stage + size_t(gg + PPR * seg) * g.d4;
      float4 x[C];
#pragma unroll
      for (int f = 0; f < C; ++f) x[f] = lds128_ordered(rp + coff[f]);
      uint64_t acc = 0;
#pragma unroll
      for (int f = 0; f < C; ++f)
        if (FULL || sl + S * f < g.d4) acc = accum4<L2>(acc, qv[f], x[f]);
      p[r * PPR + gg] = hsum2(acc);
    }
  }
  stage_release(ws, lane);
#pragma unroll
  for (int half = S / 2; half >= 1; half >>= 1) {
    const bool up = lane & half;
#pragma unroll
    for (int i = 0; i < half; ++i) {
      float send = up ? p[i] : p[i + half];
      float keep = up ? p[i + half] : p[i];
      p[i] = keep + __shfl_xor_sync(kFull, send, half);
    }
  }
  return p[0];
}

// One-round segment form with the stage filled by per-lane async copies
// (cp.async.cg, SASS LDGSTS: 16 B per lane, 512 B per warp instruction, L2 only)
// instead of TMA -- the form of the build searches (CPA).  The row of lane L goes
// to slot L as in tma_dot's one-round layout, so the math is the same.  Rows are
// copied in pass order in two commit groups: the first half of the passes starts
// its math while the second half's rows still arrive.  No mbarrier and no
// uniform-register issue loop (a tile::gather4 per 4 rows costs one ELECT / R2UR
// waterfall iteration per issuing lane), and no proxy fence: cp.async writes are
// generic-proxy writes.
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
// 4 x 16 B at byte offsets 0, 128, 256, 384 of src -> dst, where u >= 0 (one
// predicate, no branch)
__device__ __forceinline__ void cp_async_4x128(uint32_t dst, const void* src, int32_t u) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ge.s32 p, %2, 0;\n\t"
      "@p cp.async.cg.shared.global [%0], [%1], 16;\n\t"
      "@p cp.async.cg.shared.global [%0+128], [%1+128], 16;\n\t"
      "@p cp.async.cg.shared.global [%0+256], [%1+256], 16;\n\t"
      "@p cp.async.cg.shared.global [%0+384], [%1+384], 16;\n\t}" ::"r"(dst),
      "l"(src), "r"(u)
      : "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
// 4 x 16 B at byte offsets 0, 128, 256, 384 of src -> dst, copy i where u >= 0 and
// bit i of mask (the row's tail chunks of a d that is not a multiple of 32 floats)
__device__ __forceinline__ void cp_async_4x128_m(uint32_t dst, const void* src, int32_t u,
                                                 uint32_t mask) {
  asm volatile(
      "{\n\t.reg .pred p, q0, q1, q2, q3;\n\t.reg .b32 t;\n\tsetp.ge.s32 p, %2, 0;\n\t"
      "and.b32 t, %3, 1;\n\tsetp.ne.and.b32 q0, t, 0, p;\n\t"
      "and.b32 t, %3, 2;\n\tsetp.ne.and.b32 q1, t, 0, p;\n\t"
      "and.b32 t, %3, 4;\n\tsetp.ne.and.b32 q2, t, 0, p;\n\t"
      "and.b32 t, %3, 8;\n\tsetp.ne.and.b32 q3, t, 0, p;\n\t"
      "@q0 cp.async.cg.shared.global [%0], [%1], 16;\n\t"
      "@q1 cp.async.cg.shared.global [%0+128], [%1+128], 16;\n\t"
      "@q2 cp.async.cg.shared.global [%0+256], [%1+256], 16;\n\t"
      "@q3 cp.async.cg.shared.global [%0+384], [%1+384], 16;\n\t}" ::"r"(dst),
      "l"(src), "r"(u), "r"(mask)
      : "memory");
}

// cpasync_fill_quad: each copy instruction moves 4 rows x 128 B -- lanes 8r..8r+7
// copy 16-B chunks c = lane % 8 + 8 j of row 4k + r -- so a lane needs the ids of 8
// rows (8 shuffles, 8 addresses, one predicate per 4 copies) for its 32 (d = 128)
// or 64 (d = 256) copies: ~90 instructions per exploration at d = 128, against 160
// with one row per instruction (a shuffle, predicate and address per row; Phase 1
// 0.0955 -> 0.0929 s) and ~580 for a first version with a per-row copy loop
// (instruction-cache misses; 3x slower builds).
// Other d (d % 4 == 0, a row of d4 16-B chunks): the same layout with the row size
// at run time and the chunks >= d4 masked off (FULL = false).
template <int S, bool FULL = true>
__device__ __forceinline__ void cpasync_fill_quad(const GraphView& g, int32_t u_mine, int lane,
                                                  const WarpSmem& ws) {
  const uint32_t rowbytes = FULL ? uint32_t(S) * 64u : uint32_t(g.d4) * 16u;   // FULL: d4 = S * C
  constexpr int NJ = S / 2;                          // 16-B chunks per lane per row (max)
  const int r = lane >> 3, c0 = lane & 7;
  uint32_t cmask[NJ / 4];   // chunks c0 + 8 j < d4, 4 per copy block
#pragma unroll
  for (int b = 0; b < NJ / 4; ++b) {
    cmask[b] = 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) cmask[b] |= (FULL || c0 + 8 * (4 * b + i) < g.d4) ? (1u << i) : 0u;
  }
  const uint32_t sbase = smem_u32(ws.stage) + uint32_t(r) * rowbytes + uint32_t(c0) * 16u;
  const char* xb = reinterpret_cast<const char*>(g.X) + c0 * 16;
#pragma unroll
  for (int h = 0; h < 2; ++h) {
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      // row quad k (rows 4k..4k+3) belongs to the first half of the passes iff its
      // rows' pass index (row % S) is < S / 2
      if (((4 * k) % S < S / 2) != (h == 0)) continue;
      const int32_t u = __shfl_sync(kFull, u_mine, 4 * k + r);
      const uint32_t dst = sbase + uint32_t(4 * k) * rowbytes;
      const char* src = xb + uint64_t(uint32_t(u >= 0 ? u : 0)) * rowbytes;
#pragma unroll
      for (int j = 0; j < NJ; j += 4) {
        if constexpr (FULL) cp_async_4x128(dst + 128u * j, src + 128 * j, u);
        else cp_async_4x128_m(dst + 128u * j, src + 128 * j, u, cmask[j / 4]);
      }
    }
    cp_async_commit();
  }
}

// the math over a stage filled by cpasync_fill_quad (its two groups must be this
// thread's last two commits; any older group is waited for as well).  The stage
// loads are plain (not lds128_ordered): ptxas may hoist a half's 4 x C loads ahead
// of its math -- the build searches are latency-bound and have registers to spare
// (the waits' "memory" clobbers keep every load after its group's wait)
#ifndef GANNS_CPA_ORDERED
#define GANNS_CPA_ORDERED 0
#endif
template <int S, int C, bool L2, bool FULL>
__device__ __forceinline__ float cpasync_math(const GraphView& g, const float4 (&qv)[C], int lane,
                                              WarpSmem& ws) {
  const int sl = lane & (S - 1), seg = lane / S;
  int coff[C];
#pragma unroll
  for (int f = 0; f < C; ++f) coff[f] = (FULL || sl + S * f < g.d4) ? sl + S * f : g.d4 - 1;
  float p[S];
#pragma unroll
  for (int gg = 0; gg < S; ++gg) {
    if (gg == 0) {
      cp_async_wait<1>();
      __syncwarp();
    } else if (gg == S / 2) {
      cp_async_wait<0>();
      __syncwarp();
    }
    const float4* rp = ws.stage + size_t(gg + S * seg) * g.d4;
    float4 x[C];
#pragma unroll
    for (int f = 0; f < C; ++f) x[f] = GANNS_CPA_ORDERED ? lds128_ordered(rp + coff[f]) : rp[coff[f]];
    uint64_t acc = 0;
#pragma unroll
    for (int f = 0; f < C; ++f)
      if (FULL || sl + S * f < g.d4) acc = accum4<L2>(acc, qv[f], x[f]);
    p[gg] = hsum2(acc);
  }
#pragma unroll
  for (int half = S / 2; half >= 1; half >>= 1) {
    const bool up = lane & half;
#pragma unroll
    for (int i = 0; i < half; ++i) {
      float send = up ? p[i] : p[i + half];
      float keep = up ? p[i + half] : p[i];
      p[i] = keep + __shfl_xor_sync(kFull, send, half);
    }
  }
  return p[0];
}

// Whole-warp form (S = 32, d > 256): rows are staged R = ws.wrows (<= 8) at a
// time by 1-D TMA bulk copies (one per row, issued by the lane owning the
// neighbour), ceil(32 / R) rounds; each lane reads float4 columns lane + 32f of
// every staged row from shared memory; per round a transposing butterfly over
// the top 3 lane bits (8 slots; slots >= R add 0) and a plain reduction over the
// rest leave lane j with row j's total.
template <int C, bool L2, bool FULL>
__device__ __forceinline__ float wide_dot(const GraphView& g, const float4 (&qv)[C],
                                          int32_t u_mine, int lane, WarpSmem& ws) {
  constexpr int RM = kWideStageRows;   // butterfly width
  const int R = ws.wrows;
  const int my_round = lane / R, my_slot = lane - my_round * R;
  const uint32_t rowbytes = uint32_t(g.d4) * 16u;
  float dres = 0.f;
  stage_acquire(ws, lane);
#pragma unroll 1
  for (int r = 0; r * R < 32; ++r) {
    const bool mine = u_mine >= 0 && my_round == r;
    const unsigned vm = __ballot_sync(kFull, mine);
    if (vm) {
      __syncwarp();
      fence_proxy_async_smem();
      if (lane == 0) mbar_arrive_expect_tx(ws.mbar, uint32_t(__popc(vm)) * rowbytes);
      __syncwarp();
      if (mine)
        tma_row(reinterpret_cast<char*>(ws.stage) + size_t(my_slot) * rowbytes,
                reinterpret_cast<const char*>(g.X) + uint64_t(uint32_t(u_mine)) * rowbytes,
                rowbytes, ws.mbar);
      mbar_wait(ws.mbar, ws.phase);
      ws.phase ^= 1u;
    }
    float p[RM];
#pragma unroll
    for (int i = 0; i < RM; ++i) {
      uint64_t acc = 0;
      if (i < R) {
        const float4* rp = ws.stage + size_t(i) * g.d4;
#pragma unroll
        for (int f = 0; f < C; ++f)
          if (FULL || lane + 32 * f < g.d4) acc = accum4<L2>(acc, qv[f], rp[lane + 32 * f]);
      }
      p[i] = hsum2(acc);
    }
    // transposing butterfly over lane bits 4,3,2 (8 slots), then bits 1,0
#pragma unroll
    for (int st = 0; st < 3; ++st) {
      const int half = RM >> (st + 1), off = 16 >> st;
      const bool up = lane & off;
#pragma unroll
      for (int i = 0; i < half; ++i) {
        float send = up ? p[i] : p[i + half];
        float keep = up ? p[i + half] : p[i];
        p[i] = keep + __shfl_xor_sync(kFull, send, off);
      }
    }
    p[0] += __shfl_xor_sync(kFull, p[0], 2);
    p[0] += __shfl_xor_sync(kFull, p[0], 1);
    // lane L holds the total of slot (L >> 2) of this round
    const float got = __shfl_sync(kFull, p[0], (my_slot & (RM - 1)) << 2);
    if (my_round == r) dres = got;
  }
  stage_release(ws, lane);
  return dres;
}

// CPA (build searches, d <= 256): the stage is filled by cp.async (cpasync_fill_quad),
// one round of <= 32 rows
template <int NV4, bool L2, bool CPA = false>
__device__ __forceinline__ float group_distances(const GraphView& g,
                                                 const float4 (&qv)[VecLayout<NV4>::C],
                                                 int32_t u_mine, float cbase, float qinv,
                                                 int lane, WarpSmem& ws) {
  constexpr int S = VecLayout<NV4>::S, C = VecLayout<NV4>::C;
  static_assert(uses_tma(NV4) == (S < 32), "tile::gather4 is used exactly for the segment form");
  const bool full = g.d4 == S * C;
  float dot;
  if constexpr (S < 32) {
    if constexpr (CPA) {
      if (full) {
        cpasync_fill_quad<S>(g, u_mine, lane, ws);
        dot = cpasync_math<S, C, L2, true>(g, qv, lane, ws);
      } else {
        cpasync_fill_quad<S, false>(g, u_mine, lane, ws);
        dot = cpasync_math<S, C, L2, false>(g, qv, lane, ws);
      }
    } else if (ws.rounds == 1)
      dot = full ? tma_dot<S, C, L2, true, 1>(g, qv, u_mine, lane, ws)
                 : tma_dot<S, C, L2, false, 1>(g, qv, u_mine, lane, ws);
#if GANNS_SEARCH_ROUNDS == 4
    else if (ws.rounds == 4)
      dot = full ? tma_dot<S, C, L2, true, 4>(g, qv, u_mine, lane, ws)
                 : tma_dot<S, C, L2, false, 4>(g, qv, u_mine, lane, ws);
#endif
    else
      dot = full ? tma_dot<S, C, L2, true, 2>(g, qv, u_mine, lane, ws)
                 : tma_dot<S, C, L2, false, 2>(g, qv, u_mine, lane, ws);
  } else {
    dot = full ? wide_dot<C, L2, true>(g, qv, u_mine, lane, ws)
               : wide_dot<C, L2, false>(g, qv, u_mine, lane, ws);
  }
  if constexpr (L2) return dot;
  else return cbase - dot * qinv;   // IP: 0 - dot (exact); COSINE: 1 - dot/||q||
}


// Bulk-distance policy of one warp (the default): the query slice lives in this
// warp's registers and the warp computes all distances of an exploration itself.
template <int NV4, bool L2, bool CPA = false>
struct WarpDist {
  static_assert(!CPA || uses_tma(NV4), "the cp.async form is the segment form (d <= 256)");
  static constexpr int S = VecLayout<NV4>::S, C = VecLayout<NV4>::C;
  float4 qv[C];
  float cbase, qinv;
  // query slice in registers: lane owns float4 columns
  // lane%S + S*f (every S-lane segment holds a full copy of q)
  __device__ __forceinline__ void load(const GraphView& g, const float* __restrict__ qrow, int lane) {
    const float4* q4 = reinterpret_cast<const float4*>(qrow);
#pragma unroll
    for (int f = 0; f < C; ++f) {
      int i4 = (lane & (S - 1)) + S * f;
      qv[f] = i4 < g.d4 ? q4[i4] : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    cbase = 0.f;
    qinv = 1.f;
    if (!L2 && g.metric == 2) {
      float s = 0.f;
#pragma unroll
      for (int f = 0; f < C; ++f)
        s += qv[f].x * qv[f].x + qv[f].y * qv[f].y + qv[f].z * qv[f].z + qv[f].w * qv[f].w;
#pragma unroll
      for (int off = S / 2; off >= 1; off >>= 1) s += __shfl_xor_sync(kFull, s, off);
      cbase = 1.f;
      qinv = 1.f / sqrtf(s);
    }
  }
  // wide rows are staged in several rounds: warm the later rounds' rows in L2 as
  // soon as the adjacency row is known
  __device__ __forceinline__ void explore_hint(const GraphView& g, int32_t u_mine, int lane,
                                               const WarpSmem& ws) {
#if GANNS_WIDE_HINT
    if constexpr (!uses_tma(NV4))
      if (u_mine >= 0 && lane >= ws.wrows)
        prefetch_row_l2(g.X + size_t(u_mine) * (g.d4 * 4), uint32_t(g.d4) * 16u);
#endif
  }
  // SPEC (build searches, CPA): the gather of an exploration's rows is
  // issued by fill() -- possibly one iteration early -- and reduced by math()
  __device__ __forceinline__ void fill(const GraphView& g, int32_t u_mine, int lane, WarpSmem& ws) {
    if constexpr (uses_tma(NV4)) {
      if (g.d4 == S * C) cpasync_fill_quad<S>(g, u_mine, lane, ws);
      else cpasync_fill_quad<S, false>(g, u_mine, lane, ws);
    }
  }
  // a fill whose rows are not needed (a missed speculation) completes
  __device__ __forceinline__ void drain(WarpSmem&) {
    cp_async_wait<0>();
    __syncwarp();
  }
  __device__ __forceinline__ float math(const GraphView& g, int lane, WarpSmem& ws) {
    float dot = 0.f;
    if constexpr (uses_tma(NV4))
      dot = g.d4 == S * C ? cpasync_math<S, C, L2, true>(g, qv, lane, ws)
                          : cpasync_math<S, C, L2, false>(g, qv, lane, ws);
    if constexpr (L2) return dot;
    else return cbase - dot * qinv;
  }
  __device__ __forceinline__ float operator()(const GraphView& g, int32_t u_mine, int lane,
                                              WarpSmem& ws) {
    if constexpr (uses_tma(NV4))
      if (ws.pair_flag != nullptr && ws.rounds == 2) {
        int f = 0;
        if (lane == 0) f = atomicAdd(const_cast<int*>(ws.pair_flag), 0);   // atomic: orders the handover
        if (__shfl_sync(kFull, f, 0) != 0) {
          // the sibling has left: its bar.arrive (after its last writes to its
          // stage, which held its T) pairs with this bar.sync -- a CTA-level
          // happens-before edge for the stage hand-over
          pair_bar_sync(ws.pair_bar);
          ws.rounds = 1;
          ws.stage = ws.pair_stage;
        }
      }
    return group_distances<NV4, L2, CPA>(g, qv, u_mine, cbase, qinv, lane, ws);
  }
};

// The GANNS search of one query by one warp.  On return sN[0..cnt) holds N
// (ascending, explored flags set); returns cnt.  COHERENT: read the graph with
// coherent loads (the build modifies it inside the same kernel).  DIST computes
// the bulk distances of one exploration (WarpDist: this warp alone; GroupDist:
// this warp and its helper warps, search_group.cu).  PREDICT (the latency-bound
// build searches): right after the lazy check, the vertex explored next is
// predicted -- the smallest surviving neighbour always enters N, so it is next
// whenever it precedes the second unexplored entry w -- and its adjacency row is
// loaded while the sort and merge run.  Results never depend on the prediction.
// SPEC (build searches with the cp.async gather, CPA; d_max <= 32): right after an exploration's
// distance math, the rows of w (the second unexplored entry, whose adjacency row
// the speculation loads with v's) are gathered into the stage -- the stage is
// idle during the lazy check, sort and merge (T lives outside it).  When w is
// the next vertex explored (2/3 to 4/5 of the iterations in the C2 build), its
// rows have arrived meanwhile; otherwise the copies are drained and the right
// rows gathered.  Results never depend on the speculation.
template <class DIST, int TPL, bool COHERENT, bool PREDICT = false, bool SPEC = false>
__device__ int warp_search_with(const GraphView& g, DIST& dist, int32_t entry, int l, int e,
                                WarpSmem& ws, SearchStats& st) {
  static_assert(!(SPEC && PREDICT), "one speculation at a time");
  static_assert(!SPEC || TPL == 1, "SPEC gathers one 32-row round");
  const int lane = threadIdx.x & 31;
  uint64_t* sN = ws.sN;
  uint64_t* sT = ws.sT;
  uint32_t* sBM = ws.sBM;
  const int lp = lpad32(l);
  const int nwords = lp >> 5;
  // init: N = [(delta(q, entry), entry, unexplored)]
  for (int i = lane; i < lp; i += 32) sN[i] = kKeyInf;
  if (lane < nwords) sBM[lane] = 0u;
  {
    int32_t u = lane == 0 ? entry : -1;
    float dd = dist(g, u, lane, ws);
    if (lane == 0) sN[0] = mkkey(dd, entry);
  }
  __syncwarp();
  st.iters = 0;
  st.comps = 1;
  st.merged = 0;
  int cnt = 1;
  int hint = 0;   // every position < hint is explored
  const int lim_e = e < l ? e : l;

  // speculation: the adjacency row of the second unexplored entry is loaded
  // together with the first one's; if that vertex is the next one explored, its
  // row is already in registers (saves one dependent global load per hit)
  int32_t spec_v = -1;
  int32_t spec_u[TPL];
  int32_t pred_v = -1;      // PREDICT: the vertex predicted after the last lazy check
  int32_t pred_u[TPL];
  int32_t gath_v = -1;      // SPEC: the vertex whose neighbours' rows are in the stage
#if GANNS_PROFILE
  unsigned long long pc[6] = {0, 0, 0, 0, 0, 0};
  unsigned long long p_spec = 0;
  ws.p_issue = ws.p_wait = ws.p_rounds = 0;
  long long tp = clock64();
#define GANNS_PROF_MARK(i)          \
  {                                 \
    const long long t_ = clock64(); \
    pc[i] += t_ - tp;               \
    tp = t_;                        \
  }
#else
#define GANNS_PROF_MARK(i)
#endif
  for (;;) {
    // (1) candidate locating: first unexplored entry of N[0..min(e,|N|))
    const int lim = lim_e < cnt ? lim_e : cnt;
    int found = -1;
    int32_t v = 0, w = -1;
    uint64_t wkey = kKeyInf;   // PREDICT: w's key
    for (int c = hint >> 5; (c << 5) < lim; ++c) {
      int p = (c << 5) + lane;
      uint64_t k = p < lim ? sN[p] : kKeyInf;
      unsigned b = __ballot_sync(kFull, p < lim && !(uint32_t(k) & kExplored));
      if (b) {
        int src = __ffs(b) - 1;
        found = (c << 5) + src;
        if (lane == src) sN[p] = k | kExplored;   // mark explored
        v = __shfl_sync(kFull, key_id(k), src);
        const unsigned b2 = b & (b - 1);
        const int32_t wk = __shfl_sync(kFull, key_id(k), b2 ? __ffs(b2) - 1 : 0);
        w = b2 ? wk : -1;
        if constexpr (PREDICT) wkey = b2 ? unflag(shfl64(k, __ffs(b2) - 1)) : kKeyInf;
        break;
      }
    }
    if (found < 0) break;
    __syncwarp();   // the explored mark (one lane's store) is visible to the whole warp
    st.iters++;
    GANNS_PROF_MARK(kProfLocate);
    // (2) neighbourhood exploration: T <- out-neighbours of v
    int32_t u[TPL];
    const bool hitp = PREDICT && v == pred_v;
    const bool hit = !hitp && v == spec_v;
    const int32_t* row = g.nbr + size_t(v) * g.d_max;
    const int32_t* wrow = g.nbr + size_t(w < 0 ? 0 : w) * g.d_max;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      const int j = t * 32 + lane;
      const int32_t ur = (!hit && !hitp && j < g.d_max) ? load_nbr<COHERENT>(row + j) : -1;
      const int32_t uw = (w >= 0 && j < g.d_max) ? load_nbr<COHERENT>(wrow + j) : -1;
      u[t] = hitp ? pred_u[t] : hit ? spec_u[t] : ur;
      spec_u[t] = uw;
    }
    spec_v = w;
    pred_v = -1;
#if GANNS_PROFILE
    p_spec += hit ? 1 : 0;
    if (__ballot_sync(kFull, u[0] >= 0) == 0xdeadbeefu) st.merged += 0;   // waits for the row
    GANNS_PROF_MARK(kProfExplore);
#endif
    // the lazy check's key-independent loads, issued before the gather so their
    // latency hides under it (the latency-bound build searches, SPEC; the batched
    // search measured 1.5-2.5 % slower with it): N's l-th key and the first 4-ary
    // step's three probes (N's distances do not change until the merge; the
    // explored flag set by the locate step is masked off)
    constexpr bool kPre = GANNS_LB_PRELOAD != 0 && SPEC;
    uint64_t worst_pre = kKeyInf;
    uint32_t probe[3] = {0u, 0u, 0u};
    if constexpr (kPre) {
      worst_pre = cnt == l ? unflag(sN[l - 1]) : kKeyInf;
      if (cnt > 3) {
        const uint32_t* sNd0 = reinterpret_cast<const uint32_t*>(sN) + 1;
        const int q0 = cnt >> 2;
#pragma unroll
        for (int i = 0; i < 3; ++i) probe[i] = sNd0[2 * ((i + 1) * q0)];
      }
    }
    // (3) bulk distance computation
#pragma unroll
    for (int t = 0; t < TPL; ++t) dist.explore_hint(g, u[t], lane, ws);
    uint64_t key[TPL];
    if constexpr (SPEC) {
#if GANNS_PROFILE
      // SPEC timers: p_issue = cycles issuing copies (both fills), p_wait = the
      // math incl. its waits, p_rounds = explorations whose rows were gathered ahead
      const long long t_s0 = clock64();
      ws.p_rounds += v == gath_v ? 1 : 0;
#endif
      if (v != gath_v) {   // not gathered ahead: drain the speculative copies, gather
        if (gath_v >= 0) dist.drain(ws);
        dist.fill(g, u[0], lane, ws);
      }
#if GANNS_PROFILE
      const long long t_s1 = clock64();
#endif
      const float dd = dist.math(g, lane, ws);
      key[0] = u[0] >= 0 ? mkkey(dd, u[0]) : kKeyInf;
      st.comps += __popc(__ballot_sync(kFull, u[0] >= 0));
      __syncwarp();   // every lane's stage reads precede the next copies into it
#if GANNS_PROFILE
      const long long t_s2 = clock64();
#endif
      gath_v = -1;
      if (w >= 0) {   // spec_u = w's adjacency row (loaded with v's)
        dist.fill(g, spec_u[0], lane, ws);
        gath_v = w;
      }
#if GANNS_PROFILE
      const long long t_s3 = clock64();
      ws.p_issue += (t_s1 - t_s0) + (t_s3 - t_s2);
      ws.p_wait += t_s2 - t_s1;
#endif
    } else {
#pragma unroll
      for (int t = 0; t < TPL; ++t) {
        float dd = dist(g, u[t], lane, ws);
        key[t] = u[t] >= 0 ? mkkey(dd, u[t]) : kKeyInf;
        st.comps += __popc(__ballot_sync(kFull, u[t] >= 0));
      }
    }
    __syncwarp();   // every lane's stage reads precede the merge's writes of T (it shares the stage)
    GANNS_PROF_MARK(kProfDistance);
    // (4) lazy check (R-C1): drop entries already in N; entries that
    // cannot enter N (>= its l-th key while N is full) are dropped as well.
    const uint64_t worst = kPre ? worst_pre : cnt == l ? unflag(sN[l - 1]) : kKeyInf;
#if GANNS_SKIP_LB
    if (cnt == l) {
      unsigned below = 0;
#pragma unroll
      for (int t = 0; t < TPL; ++t) below |= __ballot_sync(kFull, u[t] >= 0 && key[t] < worst);
      if (below == 0) {
        hint = found + 1;
        __syncwarp();
        GANNS_PROF_MARK(kProfLazy);
        continue;
      }
    }
#endif
    bool cand[TPL];
    int rN[TPL];
    unsigned cb[TPL];
    int ncand = 0;
    // the distance halves of N's keys (word 2i + 1 of key i): the lower_bound
    // compares 32-bit distances only -- one load and one compare per probe, no
    // flag masking; equal distances (rare) are resolved on the full key after
    const uint32_t* sNd = reinterpret_cast<const uint32_t*>(sN) + 1;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      cand[t] = u[t] >= 0 && key[t] < worst;
      // 4-ary lower_bound of key[t]'s distance in N[0..cnt): three independent
      // probes per step; the trip count depends only on cnt (warp-uniform)
      const uint64_t kt = key[t];
      const uint32_t kd = uint32_t(kt >> 32);
      int base = 0, len = cnt;   // invariant: lower_bound in [base, base + len]
      if (kPre && len > 3) {   // the first step on the preloaded probes
        const int q = len >> 2;
        const int c = (probe[0] < kd ? 1 : 0) + (probe[1] < kd ? 1 : 0) + (probe[2] < kd ? 1 : 0);
        base += c * q;
        len = c < 3 ? q : len - 3 * q;
      }
      while (len > 3) {
        const int q = len >> 2;
        const int c = (sNd[2 * (base + q)] < kd ? 1 : 0) + (sNd[2 * (base + 2 * q)] < kd ? 1 : 0) +
                      (sNd[2 * (base + 3 * q)] < kd ? 1 : 0);
        base += c * q;
        len = c < 3 ? q : len - 3 * q;
      }
      int r = base;
#pragma unroll
      for (int i = 0; i < 3; ++i) r += (i < len && sNd[2 * (base + i)] < kd) ? 1 : 0;
      // r = first entry with distance >= kd; entries of equal distance follow in id
      // order: skip the smaller ids -- then N[r] is the full-key lower_bound
      uint64_t nk = r < cnt ? unflag(sN[r]) : kKeyInf;
      while (nk < kt) {
        ++r;
        nk = r < cnt ? unflag(sN[r]) : kKeyInf;
      }
      rN[t] = r;
      if (nk == kt) cand[t] = false;   // lazy check: in N (R-C1)
      cb[t] = __ballot_sync(kFull, cand[t]);
      ncand += __popc(cb[t]);
    }
    if (ncand == 0) {
      hint = found + 1;
      __syncwarp();
      GANNS_PROF_MARK(kProfLazy);
      continue;
    }
    GANNS_PROF_MARK(kProfLazy);
    if constexpr (PREDICT) {
      uint64_t mk = kKeyInf;
#pragma unroll
      for (int t = 0; t < TPL; ++t) mk = cand[t] && key[t] < mk ? key[t] : mk;
#pragma unroll
      for (int off = 16; off >= 1; off >>= 1) {
        const uint64_t o = shfl64(mk, lane ^ off);
        mk = o < mk ? o : mk;
      }
      if (mk < wkey) {   // the smallest survivor precedes w: it is explored next
        pred_v = key_id(mk);
        const int32_t* prow = g.nbr + size_t(pred_v) * g.d_max;
#pragma unroll
        for (int t = 0; t < TPL; ++t) {
          const int j = t * 32 + lane;
          pred_u[t] = j < g.d_max ? load_nbr<COHERENT>(prow + j) : -1;
        }
      }
    }
    // (5) sort: rank of each survivor among the survivors, (dist, id) order
    int rT[TPL];
#pragma unroll
    for (int t = 0; t < TPL; ++t) rT[t] = 0;
#pragma unroll
    for (int s = 0; s < TPL; ++s) {
      unsigned m = cb[s];
      while (m) {   // four survivors per round: independent shuffles in flight
        int src[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          src[i] = m ? __ffs(m) - 1 : -1;
          m &= m ? m - 1 : 0u;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const uint64_t ks = shfl64(key[s], src[i] < 0 ? 0 : src[i]);
#pragma unroll
          for (int t = 0; t < TPL; ++t) rT[t] += (src[i] >= 0 && ks < key[t]) ? 1 : 0;
        }
      }
    }
    GANNS_PROF_MARK(kProfSort);
    // (6) candidate update: merge T into N keeping l entries
    int pmin = lp, nins = 0;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      const int pos = rN[t] + rT[t];
      const bool ins = cand[t] && pos < l;
      if (ins) {
        // a new candidate is likely to be explored soon: warm its adjacency row in L2
        asm volatile("prefetch.global.L2 [%0];" ::"l"(g.nbr + size_t(u[t]) * g.d_max));
        sT[rT[t]] = key[t];
        atomicOr(&sBM[pos >> 5], 1u << (pos & 31));
      }
      nins += __popc(__ballot_sync(kFull, ins));
      // the smallest survivor (rank 0 among the survivors) always enters N and
      // has the smallest position of all insertions: pmin = its rank in N
      const unsigned m0 = __ballot_sync(kFull, cand[t] && rT[t] == 0);
      if (m0) pmin = __shfl_sync(kFull, rN[t], __ffs(m0) - 1);
    }
    const int ncnt = cnt + ncand < l ? cnt + ncand : l;
    if (nins > 0) {
      __syncwarp();
      st.merged += nins;
      // rebuild N in place from the last chunk down: output p takes the compacted
      // T entry #(T positions < p) or N[p - #(T positions < p)].  Four chunks per
      // step: every source of a chunk lies at or below it, so reading the four
      // chunks' sources before writing any of them is safe
      int suffix = 0;   // T positions at or above the current chunk
      const int c_lo = pmin >> 5;
      for (int c0 = (ncnt - 1) >> 5; c0 >= c_lo; c0 -= 4) {
        uint64_t val[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int c = c0 - j;
          val[j] = 0;
          if (c >= c_lo) {
            const uint32_t word = sBM[c];
            suffix += __popc(word);
            const int p = (c << 5) + lane;
            const bool isT = (word >> lane) & 1u;
            const int tb = nins - suffix + __popc(word & lanemask_lt());
            if (p < ncnt) val[j] = isT ? sT[tb] : sN[p - tb];
          }
        }
        __syncwarp();
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int c = c0 - j;
          if (c >= c_lo) {
            const int p = (c << 5) + lane;
            if (p < ncnt) sN[p] = val[j];
            if (lane == 0) sBM[c] = 0u;
          }
        }
        __syncwarp();
      }
#if GANNS_LATE_FENCE
      if constexpr (!SPEC)
        fence_proxy_async_smem();   // T's generic writes (in the stage) precede the next TMA writes
#endif
      hint = pmin < found + 1 ? pmin : found + 1;
    } else {
      hint = found + 1;
    }
    cnt = ncnt;
    __syncwarp();
    GANNS_PROF_MARK(kProfMerge);
  }
  if constexpr (SPEC)
    if (gath_v >= 0) dist.drain(ws);   // the last speculation's copies land before the stage is reused
#if GANNS_PROFILE
  if (g.prof != nullptr && lane == 0) {
#pragma unroll
    for (int i = 0; i < 6; ++i) atomicAdd(g.prof + i, pc[i]);
    atomicAdd(g.prof + 6, (unsigned long long)st.iters);
    atomicAdd(g.prof + 7, 1ull);
    atomicAdd(g.prof + 8, ws.p_issue);
    atomicAdd(g.prof + 9, ws.p_wait);
    atomicAdd(g.prof + 10, ws.p_rounds);
    atomicAdd(g.prof + 11, p_spec);
    unsigned long long tot = 0;
#pragma unroll
    for (int i = 0; i < 6; ++i) tot += pc[i];
    atomicMax(g.prof + 12, tot);
    atomicMax(g.prof + 13, (unsigned long long)st.iters);
  }
#endif
#undef GANNS_PROF_MARK
  return cnt;
}

// CPA: the build searches' cp.async gathers (group_distances); SPEC requires it
template <int NV4, int TPL, bool L2, bool COHERENT, bool PREDICT = false, bool SPEC = false,
          bool CPA = SPEC>
__device__ __forceinline__ int warp_search(const GraphView& g, const float* __restrict__ qrow,
                                           int32_t entry, int l, int e, WarpSmem& ws,
                                           SearchStats& st) {
  static_assert(!SPEC || CPA, "the speculative gather is a cp.async gather");
  WarpDist<NV4, L2, CPA> dist;
  dist.load(g, qrow, threadIdx.x & 31);
  return warp_search_with<WarpDist<NV4, L2, CPA>, TPL, COHERENT, PREDICT, SPEC>(g, dist, entry, l,
                                                                               e, ws, st);
}

// ---------------------------------------------------------------- HNSW
// Upper layers of an HNSW index (Section IV-D): layer j (1..top) is a
// graph over the shuffled-id prefix [0, n[j]) of the permuted points.
constexpr int kMaxLayers = 16;
struct UpperLayers {
  int top;                              // highest layer; 0 = no upper layers
  const int32_t* nbr[kMaxLayers];       // nbr[j], j = 1..top: [n[j]][d_max], shuffled ids
  int64_t n[kMaxLayers];
};

// Greedy descent: the GANNS search with l = e = 1 (the best candidate only) from
// shuffled id 0 through layers top..stop; returns the vertex reached.  `base`
// carries the permuted points (and their tensor map) and the degree.
// With l = e = 1 the loop of warp_search reduces to: N = [(delta(q, c), c)];
// explore c, compute its neighbours' distances; the lazy check keeps the entries
// below N's only key (an equal key is c itself); the merge keeps the smallest --
// so c moves to its nearest neighbour by (dist, id) while that one is nearer,
// and the search ends when none is.  This form keeps no N, T or bitmap (fewer
// live registers in the kernels that inline it); results and counters (per
// layer: 1 + the neighbours of every explored vertex; one iteration per
// exploration) equal warp_search's at l = e = 1.
#ifndef GANNS_DESCEND_NOINLINE
#define GANNS_DESCEND_NOINLINE 0
#endif
#if GANNS_DESCEND_NOINLINE
#define GANNS_DESCEND_ATTR __noinline__
#else
#define GANNS_DESCEND_ATTR
#endif
template <int NV4, int TPL, bool L2, bool CPA = false>
__device__ GANNS_DESCEND_ATTR int32_t descend(const GraphView& base, const UpperLayers& U, int stop,
                           const float* __restrict__ q, WarpSmem& ws,
                           SearchStats* acc = nullptr) {
  const int lane = threadIdx.x & 31;
  WarpDist<NV4, L2, CPA> dist;
  dist.load(base, q, lane);
  int32_t cur = 0;
  for (int j = U.top; j >= stop; --j) {
    GraphView gv = base;
    gv.nbr = U.nbr[j];
    gv.n = U.n[j];
    // N = [(delta(q, cur), cur)]: one distance computation per layer
    const float dc = __shfl_sync(kFull, dist(gv, lane == 0 ? cur : -1, lane, ws), 0);
    uint64_t best = mkkey(dc, cur);
    uint32_t iters = 0, comps = 1;
    for (;;) {
      ++iters;
      const int32_t* row = gv.nbr + size_t(cur) * gv.d_max;
      int32_t u[TPL];
#pragma unroll
      for (int t = 0; t < TPL; ++t) {
        const int jj = t * 32 + lane;
        u[t] = jj < gv.d_max ? __ldg(row + jj) : -1;
      }
      uint64_t mk = kKeyInf;
#pragma unroll
      for (int t = 0; t < TPL; ++t) {
        const float dd = dist(gv, u[t], lane, ws);
        const uint64_t kt = u[t] >= 0 ? mkkey(dd, u[t]) : kKeyInf;
        mk = kt < mk ? kt : mk;
        comps += __popc(__ballot_sync(kFull, u[t] >= 0));
      }
#pragma unroll
      for (int off = 16; off >= 1; off >>= 1) {
        const uint64_t o = shfl64(mk, lane ^ off);
        mk = o < mk ? o : mk;
      }
      __syncwarp();   // the stage's reads precede the next gather
      if (!(mk < best)) break;
      best = mk;
      cur = key_id(mk);
    }
    if (acc != nullptr) {   // the descent's own counters (bench: its algorithmic bytes)
      acc->iters += iters;
      acc->comps += comps;
    }
  }
  return cur;
}

}  // namespace ganns
