// search_group.cuh -- K1 for wide rows (d > 256): a warp group per query.
//
// The paper gives each query one thread block and lets its threads
// share the bulk distance computation.  On B200 a 960-float row costs one
// warp ~8 dependent shared-memory loads and 16 dependent packed FMAs per lane,
// and a small high-dimension batch (GIST1M-shaped: 1K queries, ~7 per SM) leaves
// too few warps per SM to hide that latency: one warp per query spends as long
// computing as waiting for memory.  Here a CTA of kGroupWarps warps owns one
// query:
//   * warp 0 (the leader) runs the whole GANNS loop of ganns_dev.cuh -- candidate
//     locating, exploration, lazy check, sort, merge -- unchanged;
//   * its bulk-distance step is shared: the leader publishes the
//     neighbour ids, issues the TMA bulk copies of each round's rows into the
//     CTA's stage, and every warp of the group reduces its own slice of the
//     columns (warp w owns float4 columns w*32 + lane + 32*G*f) for every staged
//     row; per-warp row partials meet in shared memory and the leader adds them.
// Commands pass through shared memory behind named barriers (barrier 1: a
// command is published; barrier 2: a round's partials are written and the stage
// may be refilled).  Results are those of the one-warp search: the same N after
// every iteration (distances are exact on integer-grid inputs whatever the
// summation order, R-C18; cosine to rounding).
#pragma once
#include "ganns_dev.cuh"

namespace ganns {

constexpr int kGroupWarps = 4;
constexpr int kGroupMinBlocks = 7;   // <= 73 registers: 7 queries (28 warps) per SM
enum : int { kCmdDist = 0, kCmdNewQuery = 1, kCmdExit = 2 };

// Per-CTA group area, after the leader's WarpSmem block.
struct GroupShared {
  int32_t* sU;      // [32] neighbour ids of the current exploration (-1 = none)
  float* sPart;     // [kGroupWarps][32] per-warp partial sums, one per row
  float* sNorm;     // [kGroupWarps] partial |q|^2 (cosine)
  int32_t* sCmd;    // [2] command words, alternating
  int64_t* sQ;      // query index of kCmdNewQuery
};
__host__ __device__ constexpr size_t group_area_bytes() {
  return 32 * 4 + size_t(kGroupWarps) * 32 * 4 + 16 * 4 + 16;
}
__device__ __forceinline__ GroupShared carve_group(uint8_t* p) {
  GroupShared s;
  s.sU = reinterpret_cast<int32_t*>(p);
  s.sPart = reinterpret_cast<float*>(p + 128);
  s.sNorm = s.sPart + kGroupWarps * 32;
  s.sCmd = reinterpret_cast<int32_t*>(s.sNorm + 8);
  s.sQ = reinterpret_cast<int64_t*>(s.sCmd + 8);
  return s;
}
// Non-.aligned form: the leader and the helpers reach a barrier through different
// barrier instructions (bar.sync is barrier.sync.aligned, which requires the same
// instruction in every thread).
__device__ __forceinline__ void group_bar(int id) {
  __syncwarp();
  asm volatile("barrier.sync %0, %1;" ::"r"(id), "r"(kGroupWarps * 32) : "memory");
}

// Query slice of warp w: float4 columns w*32 + lane + 32*G*f, f < CG.
template <int CG>
__device__ __forceinline__ float group_load_query(const GraphView& g, const float* __restrict__ qrow,
                                                  int w, int lane, float4 (&qv)[CG]) {
  const float4* q4 = reinterpret_cast<const float4*>(qrow);
  float s = 0.f;
#pragma unroll
  for (int f = 0; f < CG; ++f) {
    const int c = w * 32 + lane + 32 * kGroupWarps * f;
    qv[f] = c < g.d4 ? q4[c] : make_float4(0.f, 0.f, 0.f, 0.f);
    s += qv[f].x * qv[f].x + qv[f].y * qv[f].y + qv[f].z * qv[f].z + qv[f].w * qv[f].w;
  }
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) s += __shfl_xor_sync(kFull, s, off);
  return s;
}

// One exploration's bulk distances, executed by every warp of the group: R =
// ws.wrows rows per TMA round (lane j's row is staged in round j / R, slot j % R);
// the leader issues the copies, every warp waits on the same mbarrier phase,
// reduces its columns of each staged row (transposing butterfly over 8 slots,
// then two plain steps: lane 4s holds slot s) and writes its partial of row j to
// sPart[w][j].  u_mine is identical in every warp (read from sU), so the
// per-round ballots -- and the skipped empty rounds -- agree across the group.
template <int CG, bool L2, bool LEADER>
__device__ __forceinline__ void group_rounds(const GraphView& g, const float4 (&qv)[CG],
                                             int32_t u_mine, int lane, int w, WarpSmem& ws,
                                             float* __restrict__ sPart) {
  constexpr int RM = kWideStageRows;
  const int R = ws.wrows;
  const int my_round = lane / R, my_slot = lane - my_round * R;
  const uint32_t rowbytes = uint32_t(g.d4) * 16u;
#pragma unroll 1
  for (int r = 0; r * R < 32; ++r) {
    const bool mine = u_mine >= 0 && my_round == r;
    const unsigned vm = __ballot_sync(kFull, mine);
    if (!vm) continue;
    if constexpr (LEADER) {
      fence_proxy_async_smem();   // the group's reads of the stage (ordered by bar 2) precede the copies
      if (lane == 0) mbar_arrive_expect_tx(ws.mbar, uint32_t(__popc(vm)) * rowbytes);
      __syncwarp();
      if (mine)
        tma_row(reinterpret_cast<char*>(ws.stage) + size_t(my_slot) * rowbytes,
                reinterpret_cast<const char*>(g.X) + uint64_t(uint32_t(u_mine)) * rowbytes,
                rowbytes, ws.mbar);
    }
    mbar_wait(ws.mbar, ws.phase);
    ws.phase ^= 1u;
    float p[RM];
#pragma unroll
    for (int i = 0; i < RM; ++i) {
      uint64_t acc = 0;
      if (i < R) {
        const float4* rp = ws.stage + size_t(i) * g.d4;
        float4 x[CG];
#pragma unroll
        for (int f = 0; f < CG; ++f) {
          const int c = w * 32 + lane + 32 * kGroupWarps * f;
          x[f] = c < g.d4 ? rp[c] : make_float4(0.f, 0.f, 0.f, 0.f);
        }
#pragma unroll
        for (int f = 0; f < CG; ++f) acc = accum4<L2>(acc, qv[f], x[f]);
      }
      p[i] = hsum2(acc);
    }
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
    const int slot = lane >> 2;
    if ((lane & 3) == 0 && slot < R && r * R + slot < 32) sPart[w * 32 + r * R + slot] = p[0];
    group_bar(2);   // partials written; the stage may be refilled
  }
}

// The leader's distance policy for warp_search_with (ganns_dev.cuh).
template <int CG, bool L2>
struct GroupDist {
  float4 qv[CG];
  float cbase, qinv;
  GroupShared gs;
  int kc;   // commands posted so far (selects the command word)

  __device__ __forceinline__ void post(int cmd, int lane) {
    if (lane == 0) gs.sCmd[kc & 1] = cmd;
    ++kc;
    group_bar(1);
  }
  __device__ __forceinline__ void explore_hint(const GraphView& g, int32_t u_mine, int lane,
                                               const WarpSmem& ws) {
#if GANNS_WIDE_HINT
    if (u_mine >= 0 && lane >= ws.wrows)
      prefetch_row_l2(g.X + size_t(u_mine) * (g.d4 * 4), uint32_t(g.d4) * 16u);
#endif
  }
  __device__ __forceinline__ float operator()(const GraphView& g, int32_t u_mine, int lane,
                                              WarpSmem& ws) {
    // an exploration with no neighbour (ragged or isolated rows) involves no helper
    if (__ballot_sync(kFull, u_mine >= 0) == 0) return 0.f;
    gs.sU[lane] = u_mine;
    post(kCmdDist, lane);
    group_rounds<CG, L2, true>(g, qv, u_mine, lane, 0, ws, gs.sPart);
    float dot = 0.f;
#pragma unroll
    for (int w = 0; w < kGroupWarps; ++w) dot += gs.sPart[w * 32 + lane];
    if constexpr (L2) return dot;
    else return cbase - dot * qinv;   // IP: 0 - dot (exact); COSINE: 1 - dot/||q||
  }
};

// Helper warps (w != 0): execute the leader's commands until it posts kCmdExit.
// A new query's row is Q[*gs.sQ] (the search's queries, or the build's points).
template <int CG, bool L2>
__device__ __forceinline__ void group_helper_loop(const GraphView& g, const float* __restrict__ Q,
                                                  const GroupShared& gs, WarpSmem& ws, int w,
                                                  int lane) {
  float4 qv[CG];
  int kc = 0;
  for (;;) {
    group_bar(1);
    const int cmd = gs.sCmd[kc & 1];
    ++kc;
    if (cmd == kCmdExit) return;
    if (cmd == kCmdNewQuery) {
      const float s = group_load_query<CG>(g, Q + size_t(*gs.sQ) * (g.d4 * 4), w, lane, qv);
      if (lane == 0) gs.sNorm[w] = s;
      group_bar(2);
      continue;
    }
    group_rounds<CG, L2, false>(g, qv, gs.sU[lane], lane, w, ws, gs.sPart);
  }
}

// Leader: start the group's search of row q of Q (every warp loads its query slice;
// cosine needs the full |q|).
template <int CG, bool L2>
__device__ __forceinline__ void group_new_query(GroupDist<CG, L2>& dist, const GraphView& g,
                                                const float* __restrict__ Q, int64_t q, int lane) {
  if (lane == 0) *dist.gs.sQ = q;
  dist.post(kCmdNewQuery, lane);
  const float s0 = group_load_query<CG>(g, Q + size_t(q) * (g.d4 * 4), 0, lane, dist.qv);
  if (lane == 0) dist.gs.sNorm[0] = s0;
  group_bar(2);
  dist.cbase = 0.f;
  dist.qinv = 1.f;
  if (!L2 && g.metric == 2) {
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kGroupWarps; ++i) s += dist.gs.sNorm[i];
    dist.cbase = 1.f;
    dist.qinv = 1.f / sqrtf(s);
  }
}

template <int CG, int TPL, bool L2>
__global__ void __launch_bounds__(kGroupWarps * 32, kGroupMinBlocks)
search_group_kernel(GraphView g, const float* __restrict__ Q, int64_t nq, int k, int l, int e,
                    int32_t entry, int32_t* __restrict__ out_ids, float* __restrict__ out_dists,
                    uint32_t* __restrict__ stats, int32_t* __restrict__ ticket,
                    const int32_t* __restrict__ entries, int wrows) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const size_t wsb = warp_smem_bytes(l, TPL, 8, g.d4, 1, wrows);
  WarpSmem ws = carve_warp_smem(smem, l, TPL, 8, g.d4, 1, wrows);
  GroupShared gs = carve_group(smem + wsb);
  if (threadIdx.x == 0) mbar_init(ws.mbar, 1);
  __syncthreads();
  if (w != 0) {
    group_helper_loop<CG, L2>(g, Q, gs, ws, w, lane);
    return;
  }
  GroupDist<CG, L2> dist;
  dist.gs = gs;
  dist.kc = 0;
  uint64_t* sN = ws.sN;
  for (;;) {
    int32_t qt = 0;
    if (lane == 0) qt = atomicAdd(ticket, 1);
    const int64_t q = __shfl_sync(kFull, qt, 0);
    if (q >= nq) {
      dist.post(kCmdExit, lane);
      break;
    }
    group_new_query<CG, L2>(dist, g, Q, q, lane);
    SearchStats st;
    const int32_t ent = entries != nullptr ? entries[q] : entry;   // HNSW: per-query entry
    const int cnt = warp_search_with<GroupDist<CG, L2>, TPL, false>(g, dist, ent, l, e, ws, st);
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

}  // namespace ganns
