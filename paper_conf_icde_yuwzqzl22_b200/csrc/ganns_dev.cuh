// ganns_dev.cuh -- device side of the GANNS search (§III-B),
// shared by the batched search kernel (search.cu) and the GGraphCon build kernels
// (build.cu).  sm_100a only.
//
// One warp owns one query (the paper's "thread block per query" with n_t = 32
// threads, R-C20).  Per query the warp keeps, in shared memory:
//   sN  : candidate array N, up to l packed keys (lazy update), ascending
//   sT  : the surviving visiting entries T, compacted in sorted order
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
//   (3) bulk distance -- all d_max rows gathered with 128-bit read-only loads,
//       B rows in flight per lane; partial dot products reduced by a transposing
//       butterfly so lane j ends with delta(q, T[j])
//   (4) lazy check -- entries that cannot enter N (>= its l-th key when full)
//       are skipped; the rest binary-search N; equal key => duplicate, dropped
//       (R-C1).  The probe gives rank_N(t) for free.
//   (5) sort -- rank of each surviving entry among the survivors (R-C2 order);
//       this yields the sorted order of T without moving data
//   (6) merge -- position(t) = rank_N(t) + rank_T(t); N is rebuilt in place from
//       the position bitmap, from the last chunk down to the first changed one
//       (P:210-212).  Duplicates never reach the merge.
#pragma once
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
__device__ __forceinline__ float4 ldg_stream(const float4* p) {
  float4 r;
  asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
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
  int64_t n;
  int d_max;
  int d4;               // d / 4
  int metric;           // 0 L2, 1 IP, 2 COSINE
};

// Per-search counters (kept in registers, identical to the oracle's stats[0,1,3]).
struct SearchStats {
  uint32_t iters, comps, merged;
};

// Distances of the <= 32 rows in one T slot group, lane j -> delta(q, row of u_j).
// NV4 = float4 per lane per row (ceil(d/128)); B rows per batch.
template <int NV4, bool L2>
__device__ __forceinline__ float group_distances(const GraphView& g, const float4 (&qv)[NV4],
                                                 int32_t u_mine, float cbase, float qinv,
                                                 int lane) {
  constexpr int B = NV4 >= 8 ? 1 : 8 / NV4;
  constexpr int LOGB = B == 8 ? 3 : B == 4 ? 2 : B == 2 ? 1 : 0;
  const float4* X4 = reinterpret_cast<const float4*>(g.X);
  float dres = 0.f;
#pragma unroll
  for (int b = 0; b < 32 / B; ++b) {
    float4 buf[B][NV4];
    int32_t ub[B];
#pragma unroll
    for (int i = 0; i < B; ++i) {
      ub[i] = __shfl_sync(kFull, u_mine, b * B + i);
      const float4* row = X4 + size_t(ub[i] < 0 ? 0 : ub[i]) * g.d4;
#pragma unroll
      for (int f = 0; f < NV4; ++f) {
        int i4 = lane + 32 * f;
        buf[i][f] = (ub[i] >= 0 && i4 < g.d4) ? ldg_stream(row + i4) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
    float p[B];
#pragma unroll
    for (int i = 0; i < B; ++i) {
      float acc = 0.f;
#pragma unroll
      for (int f = 0; f < NV4; ++f) {
        const float4 x = buf[i][f], q = qv[f];
        if constexpr (L2) {
          float t0 = q.x - x.x, t1 = q.y - x.y, t2 = q.z - x.z, t3 = q.w - x.w;
          acc = fmaf(t0, t0, acc); acc = fmaf(t1, t1, acc);
          acc = fmaf(t2, t2, acc); acc = fmaf(t3, t3, acc);
        } else {
          acc = fmaf(q.x, x.x, acc); acc = fmaf(q.y, x.y, acc);
          acc = fmaf(q.z, x.z, acc); acc = fmaf(q.w, x.w, acc);
        }
      }
      p[i] = acc;
    }
    // transposing butterfly: after LOGB stages lane L holds batch entry
    // (L >> (5-LOGB)) summed over the lanes that differ in the top LOGB bits
#pragma unroll
    for (int s = 0; s < LOGB; ++s) {
      const int half = B >> (s + 1), off = 16 >> s;
      const bool up = lane & off;
#pragma unroll
      for (int i = 0; i < half; ++i) {
        float send = up ? p[i] : p[i + half];
        float keep = up ? p[i + half] : p[i];
        p[i] = keep + __shfl_xor_sync(kFull, send, off);
      }
    }
#pragma unroll
    for (int off = 16 >> LOGB; off >= 1; off >>= 1) p[0] += __shfl_xor_sync(kFull, p[0], off);
    float got = __shfl_sync(kFull, p[0], (lane & (B - 1)) << (5 - LOGB));
    if ((lane >> LOGB) == b) dres = got;
  }
  if constexpr (L2) return dres;
  else return cbase - dres * qinv;   // IP: 0 - dot (exact); COSINE: 1 - dot/||q||
}

// Shared-memory footprint of one warp's search state for list length l.
__host__ __device__ constexpr int lpad32(int l) { return (l + 31) & ~31; }
__host__ __device__ constexpr size_t warp_smem_bytes(int l, int tpl) {
  return size_t(lpad32(l)) * 8 + size_t(tpl) * 32 * 8 + 32 * 4;
}

// The GANNS search of one query by one warp.  On return sN[0..cnt) holds N
// (ascending, explored flags set); returns cnt.  COHERENT: read the graph with
// coherent loads (the build modifies it inside the same kernel).
template <int NV4, int TPL, bool L2, bool COHERENT>
__device__ int warp_search(const GraphView& g, const float* __restrict__ qrow, int32_t entry,
                           int l, int e, uint64_t* sN, uint64_t* sT, uint32_t* sBM,
                           SearchStats& st) {
  const int lane = threadIdx.x & 31;
  const int lp = lpad32(l);
  const int nwords = lp >> 5;
  // query slice in registers
  float4 qv[NV4];
  const float4* q4 = reinterpret_cast<const float4*>(qrow);
#pragma unroll
  for (int f = 0; f < NV4; ++f) {
    int i4 = lane + 32 * f;
    qv[f] = i4 < g.d4 ? q4[i4] : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  float cbase = 0.f, qinv = 1.f;
  if (!L2 && g.metric == 2) {
    float s = 0.f;
#pragma unroll
    for (int f = 0; f < NV4; ++f)
      s += qv[f].x * qv[f].x + qv[f].y * qv[f].y + qv[f].z * qv[f].z + qv[f].w * qv[f].w;
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) s += __shfl_xor_sync(kFull, s, off);
    cbase = 1.f;
    qinv = 1.f / sqrtf(s);
  }
  // init: N = [(delta(q, entry), entry, unexplored)]
  for (int i = lane; i < lp; i += 32) sN[i] = kKeyInf;
  if (lane < nwords) sBM[lane] = 0u;
  {
    int32_t u = lane == 0 ? entry : -1;
    float dd = group_distances<NV4, L2>(g, qv, u, cbase, qinv, lane);
    if (lane == 0) sN[0] = mkkey(dd, entry);
  }
  __syncwarp();
  st.iters = 0;
  st.comps = 1;
  st.merged = 0;
  int cnt = 1;
  int hint = 0;   // every position < hint is explored
  const int lim_e = e < l ? e : l;

  for (;;) {
    // (1) candidate locating
    const int lim = lim_e < cnt ? lim_e : cnt;
    int found = -1;
    int32_t v = 0;
    for (int c = hint >> 5; (c << 5) < lim; ++c) {
      int p = (c << 5) + lane;
      uint64_t k = p < lim ? sN[p] : kKeyInf;
      unsigned b = __ballot_sync(kFull, p < lim && !(uint32_t(k) & kExplored));
      if (b) {
        int src = __ffs(b) - 1;
        found = (c << 5) + src;
        if (lane == src) sN[p] = k | kExplored;   // mark explored
        v = __shfl_sync(kFull, key_id(k), src);
        break;
      }
    }
    if (found < 0) break;
    st.iters++;
    // (2) neighbourhood exploration: T <- out-neighbours of v
    int32_t u[TPL];
    const int32_t* row = g.nbr + size_t(v) * g.d_max;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      int j = t * 32 + lane;
      u[t] = j < g.d_max ? load_nbr<COHERENT>(row + j) : -1;
    }
    // (3) bulk distance computation
    uint64_t key[TPL];
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      float dd = group_distances<NV4, L2>(g, qv, u[t], cbase, qinv, lane);
      key[t] = u[t] >= 0 ? mkkey(dd, u[t]) : kKeyInf;
      st.comps += __popc(__ballot_sync(kFull, u[t] >= 0));
    }
    // (4) lazy check (R-C1): drop entries already in N; entries that
    // cannot enter N (>= its l-th key while N is full) are dropped as well.
    const uint64_t worst = cnt == l ? unflag(sN[l - 1]) : kKeyInf;
    bool cand[TPL];
    int rN[TPL];
    unsigned cb[TPL];
    int ncand = 0;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      cand[t] = u[t] >= 0 && key[t] < worst;
      rN[t] = 0;
      if (cand[t]) {
        int lo = 0, hi = cnt;   // lower_bound of key[t] in N[0..cnt)
        while (lo < hi) {
          int mid = (lo + hi) >> 1;
          if (unflag(sN[mid]) < key[t]) lo = mid + 1;
          else hi = mid;
        }
        rN[t] = lo;
        if (lo < cnt && unflag(sN[lo]) == key[t]) cand[t] = false;
      }
      cb[t] = __ballot_sync(kFull, cand[t]);
      ncand += __popc(cb[t]);
    }
    if (ncand == 0) {
      hint = found + 1;
      __syncwarp();
      continue;
    }
    // (5) sort: rank of each survivor among the survivors, (dist, id) order
    int rT[TPL];
#pragma unroll
    for (int t = 0; t < TPL; ++t) rT[t] = 0;
#pragma unroll
    for (int s = 0; s < TPL; ++s) {
      unsigned m = cb[s];
      while (m) {
        int src = __ffs(m) - 1;
        m &= m - 1;
        uint64_t ks = shfl64(key[s], src);
#pragma unroll
        for (int t = 0; t < TPL; ++t) rT[t] += (ks < key[t]) ? 1 : 0;
      }
    }
    // (6) candidate update: merge T into N keeping l entries
    int pmin = lp;
#pragma unroll
    for (int t = 0; t < TPL; ++t) {
      int pos = rN[t] + rT[t];
      if (cand[t] && pos < l) {
        sT[rT[t]] = key[t];
        atomicOr(&sBM[pos >> 5], 1u << (pos & 31));
        pmin = pos < pmin ? pos : pmin;
      }
    }
#pragma unroll
    for (int off = 16; off >= 1; off >>= 1) {
      int o = __shfl_xor_sync(kFull, pmin, off);
      pmin = o < pmin ? o : pmin;
    }
    const int ncnt = cnt + ncand < l ? cnt + ncand : l;
    if (pmin < l) {
      __syncwarp();
      uint32_t bmw = lane < nwords ? sBM[lane] : 0u;
      uint32_t pc = __popc(bmw), ex = pc;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        uint32_t o = __shfl_up_sync(kFull, ex, off);
        if (lane >= off) ex += o;
      }
      ex -= pc;   // exclusive prefix of popcounts
      st.merged += __shfl_sync(kFull, ex + pc, 31);
      for (int c = (ncnt - 1) >> 5; c >= (pmin >> 5); --c) {
        uint32_t word = __shfl_sync(kFull, bmw, c);
        uint32_t base = __shfl_sync(kFull, ex, c);
        int p = (c << 5) + lane;
        bool isT = (word >> lane) & 1u;
        int tb = int(base + __popc(word & lanemask_lt()));
        uint64_t val = 0;
        if (p < ncnt) val = isT ? sT[tb] : sN[p - tb];
        __syncwarp();
        if (p < ncnt) sN[p] = val;
        __syncwarp();
      }
      if (lane < nwords) sBM[lane] = 0u;
      hint = pmin < found + 1 ? pmin : found + 1;
    } else {
      hint = found + 1;
    }
    cnt = ncnt;
    __syncwarp();
  }
  return cnt;
}

}  // namespace ganns
