// knn.cu -- KNN graph by neighbours-of-neighbours iterations (NEXT-4; Section
// IV-D, after NN-Descent [9]) on sm_100a.
//
// Lists ids/dists [n][K] (SoA, rows ascending by (dist, id)) start from a random
// adjacency (an input) and are improved in iterations.  In iteration t, from the
// lists as they were at its start (R-K1):
//   reverse lists  R(v) = the K smallest (dist, w) with v in list(w) (R-K2):
//                  count / carve / scatter by target, per-vertex top-K select
//   proposals      one warp per v: S(v) = list(v) u R(v) (distinct); the rows of
//                  S(v) are staged in shared memory; lane j owns row a = S_j and
//                  sweeps b over S(v): the pair distance delta(a, b) is the paper's
//                  BulkDistanceComputation; a -> b is proposed only if it
//                  beats a's current K-th key (otherwise it cannot enter)
//   update         proposals bucketed by a (count / carve / scatter) and merged:
//                  list(a) <- the K smallest distinct (dist, id) of list(a) and
//                  its proposals -- Step 3 of the local-graphs merge
// Stops when no list changes.  Bit-exact with oracle ora_knn_descent on
// integer-grid data (the order of proposals inside a bucket does not matter).
#include "../../include/ganns.h"
#include "ganns_dev.cuh"
#include "ganns_internal.h"

#include <algorithm>
#include <vector>

namespace ganns {
namespace {

constexpr int kKnnWarps = 2;

template <bool L2>
__device__ __forceinline__ float row_dist_warp(const float4* __restrict__ a,
                                               const float4* __restrict__ b, int d4, int lane) {
  uint64_t acc = 0;
  for (int c = lane; c < d4; c += 32) acc = accum4<L2>(acc, a[c], b[c]);
  float s = hsum2(acc);
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) s += __shfl_xor_sync(kFull, s, off);
  return L2 ? s : 0.f - s;
}

// initial lists: distances of the random neighbours, sorted by (dist, id)
template <bool L2>
__global__ void knn_init_kernel(const float* __restrict__ X, int64_t n, int d4, int K,
                                const int32_t* __restrict__ init, int32_t* __restrict__ ids,
                                float* __restrict__ dists) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = int64_t(gridDim.x) * (blockDim.x >> 5);
  const float4* X4 = reinterpret_cast<const float4*>(X);
  for (int64_t v = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); v < n; v += nw) {
    uint64_t mine = kKeyInf;
    for (int j = 0; j < K; ++j) {
      const int32_t w = init[size_t(v) * K + j];
      const float dd = row_dist_warp<L2>(X4 + size_t(v) * d4, X4 + size_t(w) * d4, d4, lane);
      if (lane == j) mine = mkkey(dd, w);
    }
    int rank = 0;
    for (int j = 0; j < K; ++j) rank += shfl64(mine, j) < mine ? 1 : 0;
    if (lane < K) {
      ids[size_t(v) * K + rank] = key_id(mine);
      dists[size_t(v) * K + rank] = key_dist(mine);
    }
  }
}

// ---- bucketing helpers (counting + atomic segment carving; order-free)
__global__ void bucket_count_kernel(const int32_t* __restrict__ tgt, int64_t m,
                                    int32_t* __restrict__ cnt) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t t = tgt[i];
    if (t >= 0) atomicAdd(&cnt[t], 1);
  }
}
__global__ void bucket_carve_kernel(const int32_t* __restrict__ cnt, int64_t n,
                                    int64_t* __restrict__ off, unsigned long long* total) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n;
       i += int64_t(gridDim.x) * blockDim.x)
    if (cnt[i] > 0) off[i] = int64_t(atomicAdd(total, (unsigned long long)cnt[i]));
}

// reverse entries: list entry (v, j) = (dist, w) goes to w's bucket as (dist, v)
__global__ void rev_scatter_kernel(const int32_t* __restrict__ ids, const float* __restrict__ dists,
                                   int64_t n, int K, const int64_t* __restrict__ off,
                                   int32_t* __restrict__ fill, uint64_t* __restrict__ seg) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n * K;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t w = ids[i];
    if (w < 0) continue;
    const int32_t p = atomicAdd(&fill[w], 1);
    seg[off[w] + p] = mkkey(dists[i], int32_t(i / K));
  }
}

// insert kx into a warp-distributed ascending row (one key per lane, K <= 32);
// returns true when the row changed.  Equal keys (same id, same dist) are skipped.
__device__ __forceinline__ bool row_insert_unique(uint64_t& key, uint64_t kx, int K, int lane) {
  if (__ballot_sync(kFull, key == kx)) return false;
  const int pos = __popc(__ballot_sync(kFull, key < kx));
  if (pos >= K) return false;
  const uint32_t lo = __shfl_up_sync(kFull, uint32_t(key), 1);
  const uint32_t hi = __shfl_up_sync(kFull, uint32_t(key >> 32), 1);
  const uint64_t prev = (uint64_t(hi) << 32) | lo;
  key = lane < pos ? key : (lane == pos ? kx : prev);
  if (lane >= K) key = kKeyInf;
  return true;
}

// top-K of each bucket -> reverse list rows (ids only); resets the counters
__global__ void rev_select_kernel(int64_t n, int K, int32_t* __restrict__ cnt,
                                  int32_t* __restrict__ fill, const int64_t* __restrict__ off,
                                  const uint64_t* __restrict__ seg, int32_t* __restrict__ rev) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t w = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); w < n; w += nw) {
    const int32_t m = cnt[w];
    uint64_t key = kKeyInf;
    for (int32_t c = 0; c < m; c += 32) {
      const uint64_t x = c + lane < m ? seg[off[w] + c + lane] : kKeyInf;
      unsigned b = __ballot_sync(kFull, x < shfl64(key, K - 1));
      while (b) {
        const int src = __ffs(b) - 1;
        b &= b - 1;
        row_insert_unique(key, shfl64(x, src), K, lane);
      }
    }
    if (lane < K) rev[size_t(w) * K + lane] = key_empty(key) ? -1 : key_id(key);
    __syncwarp();
    if (lane == 0) {
      cnt[w] = 0;
      fill[w] = 0;
    }
  }
}

// proposals: pair distances among S(v) = list(v) u rev(v), rows staged in smem
__host__ __device__ constexpr size_t knn_warp_smem(int d4) {
  return size_t(64) * (d4 + 1) * 16 + 64 * 4;
}

template <bool L2>
__global__ void __launch_bounds__(kKnnWarps * 32)
knn_propose_kernel(const float* __restrict__ X, int64_t n, int d4, int K,
                   const int32_t* __restrict__ ids, const float* __restrict__ dists,
                   const int32_t* __restrict__ rev, int32_t* __restrict__ Pa,
                   float* __restrict__ Pd, int32_t* __restrict__ Pb,
                   unsigned long long* __restrict__ pcount, unsigned long long cap,
                   int* __restrict__ overflow) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int pitch4 = d4 + 1;   // padded row stride (float4): conflict-free own-row reads
  uint8_t* base = smem + size_t(w) * knn_warp_smem(d4);
  float4* stage = reinterpret_cast<float4*>(base);
  int32_t* sS = reinterpret_cast<int32_t*>(base + size_t(64) * pitch4 * 16);
  const float4* X4 = reinterpret_cast<const float4*>(X);
  const int64_t nwarps = int64_t(gridDim.x) * kKnnWarps;
  for (int64_t v = int64_t(blockIdx.x) * kKnnWarps + w; v < n; v += nwarps) {
    // S(v): forward ids, then the reverse ids not already present (R-K2)
    const int32_t f = lane < K ? ids[size_t(v) * K + lane] : -1;
    int32_t r = lane < K ? rev[size_t(v) * K + lane] : -1;
    for (int j = 0; j < K; ++j)
      if (__shfl_sync(kFull, f, j) == r) r = -1;
    const unsigned fm = __ballot_sync(kFull, f >= 0), rm = __ballot_sync(kFull, r >= 0);
    const int nf = __popc(fm), m = nf + __popc(rm);
    if (f >= 0) sS[__popc(fm & lanemask_lt())] = f;
    if (r >= 0) sS[nf + __popc(rm & lanemask_lt())] = r;
    __syncwarp();
    // stage the m rows (coalesced row loads by the whole warp)
    for (int t = 0; t < m; ++t) {
      const int32_t u = sS[t];
      for (int c = lane; c < d4; c += 32) stage[size_t(t) * pitch4 + c] = X4[size_t(u) * d4 + c];
    }
    __syncwarp();
    // lane j owns slots j and j + 32: their K-th keys bound what can enter
    int32_t own[2];
    uint64_t worst[2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int t = lane + 32 * h;
      own[h] = t < m ? sS[t] : -1;
      worst[h] = kKeyInf;
      if (own[h] >= 0) {
        const int32_t wid = ids[size_t(own[h]) * K + K - 1];
        worst[h] = wid >= 0 ? mkkey(dists[size_t(own[h]) * K + K - 1], wid) : kKeyInf;
      }
    }
    for (int b = 0; b < m; ++b) {
      const int32_t ub = sS[b];
      const float4* rb = stage + size_t(b) * pitch4;
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int t = lane + 32 * h;
        bool prop = false;
        uint64_t kx = 0;
        if (t < m && t != b) {
          const float4* ra = stage + size_t(t) * pitch4;
          uint64_t acc = 0;
          for (int c = 0; c < d4; ++c) acc = accum4<L2>(acc, ra[c], rb[c]);
          const float dd = L2 ? hsum2(acc) : 0.f - hsum2(acc);
          kx = mkkey(dd, ub);
          prop = kx < worst[h];
        }
        const unsigned pm = __ballot_sync(kFull, prop);
        if (pm) {
          const int leader = __ffs(pm) - 1;
          unsigned long long at0 = 0;
          if (lane == leader) at0 = atomicAdd(pcount, (unsigned long long)__popc(pm));
          at0 = __shfl_sync(kFull, at0, leader);
          if (prop) {
            const unsigned long long at = at0 + __popc(pm & lanemask_lt());
            if (at < cap) {
              Pa[at] = own[h];
              Pd[at] = key_dist(kx);
              Pb[at] = ub;
            } else {
              *overflow = 1;
            }
          }
        }
      }
    }
    __syncwarp();
  }
}

// Register-tiled form of knn_propose_kernel (same proposals, same arithmetic per
// pair): the rows of S(v) are staged by cp.async (all in flight at once), then the
// m x m pair distances are computed in 4 passes of 4 x 8 tiles per lane -- lane
// (ga = lane % 4, gb = lane / 4) owns a-rows ga + 4 i + 16 p and b-rows gb + 8 j --
// so each staged float4 is loaded once per tile instead of once per pair (the
// one-pair-per-lane form was bound by shared-memory bandwidth: ~4 MB of LDS per v
// at m = 64, d = 128).  Loads are conflict-free with the padded row pitch.
#ifndef GANNS_KNN_TILED
#define GANNS_KNN_TILED 1
#endif
__host__ __device__ constexpr size_t knn_tiled_warp_smem(int d4) {
  return size_t(64) * (d4 + 1) * 16 + 64 * 4 + 64 * 8;
}
template <bool L2>
__global__ void __launch_bounds__(kKnnWarps * 32)
knn_propose_tiled_kernel(const float* __restrict__ X, int64_t n, int d4, int K,
                         const int32_t* __restrict__ ids, const float* __restrict__ dists,
                         const int32_t* __restrict__ rev, int32_t* __restrict__ Pa,
                         float* __restrict__ Pd, int32_t* __restrict__ Pb,
                         unsigned long long* __restrict__ pcount, unsigned long long cap,
                         int* __restrict__ overflow) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int pitch4 = d4 + 1;
  uint8_t* base = smem + size_t(w) * knn_tiled_warp_smem(d4);
  float4* stage = reinterpret_cast<float4*>(base);
  int32_t* sS = reinterpret_cast<int32_t*>(base + size_t(64) * pitch4 * 16);
  uint64_t* sW = reinterpret_cast<uint64_t*>(sS + 64);
  const float4* X4 = reinterpret_cast<const float4*>(X);
  const int ga = lane & 3, gb = lane >> 2;
  const int64_t nwarps = int64_t(gridDim.x) * kKnnWarps;
  for (int64_t v = int64_t(blockIdx.x) * kKnnWarps + w; v < n; v += nwarps) {
    // S(v): forward ids, then the reverse ids not already present (R-K2)
    const int32_t f = lane < K ? ids[size_t(v) * K + lane] : -1;
    int32_t r = lane < K ? rev[size_t(v) * K + lane] : -1;
    for (int j = 0; j < K; ++j)
      if (__shfl_sync(kFull, f, j) == r) r = -1;
    const unsigned fm = __ballot_sync(kFull, f >= 0), rm = __ballot_sync(kFull, r >= 0);
    const int nf = __popc(fm), m = nf + __popc(rm);
    if (f >= 0) sS[__popc(fm & lanemask_lt())] = f;
    if (r >= 0) sS[nf + __popc(rm & lanemask_lt())] = r;
    __syncwarp();
    // stage the m rows: every copy in flight at once
    for (int t = 0; t < m; ++t) {
      const float4* src = X4 + size_t(sS[t]) * d4;
      float4* dst = stage + size_t(t) * pitch4;
      for (int c = lane; c < d4; c += 32)
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst + c)), "l"(src + c)
                     : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    // the K-th key of every a (what a proposal must beat)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int t = lane + 32 * h;
      uint64_t wk = kKeyInf;
      if (t < m) {
        const int32_t a = sS[t];
        const int32_t wid = ids[size_t(a) * K + K - 1];
        wk = wid >= 0 ? mkkey(dists[size_t(a) * K + K - 1], wid) : kKeyInf;
      }
      sW[t] = wk;
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
    __syncwarp();
    for (int p = 0; p * 16 < m; ++p) {
      uint64_t acc[4][8];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = 0;
      int ta[4], tb[8];
#pragma unroll
      for (int i = 0; i < 4; ++i) ta[i] = min(ga + 4 * i + 16 * p, 63);
#pragma unroll
      for (int j = 0; j < 8; ++j) tb[j] = gb + 8 * j;
      for (int c = 0; c < d4; ++c) {
        float4 ra[4], rb[8];
#pragma unroll
        for (int i = 0; i < 4; ++i) ra[i] = stage[size_t(ta[i]) * pitch4 + c];
#pragma unroll
        for (int j = 0; j < 8; ++j) rb[j] = stage[size_t(tb[j]) * pitch4 + c];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = accum4<L2>(acc[i][j], ra[i], rb[j]);
      }
      // proposals of this pass: a = S[t] -> b = S[u] where the key beats a's K-th
      unsigned pm = 0;
      float dd[4][8];
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int t = ga + 4 * i + 16 * p;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int u = tb[j];
          dd[i][j] = L2 ? hsum2(acc[i][j]) : 0.f - hsum2(acc[i][j]);
          const bool ok = t < m && u < m && t != u && mkkey(dd[i][j], sS[u]) < sW[t];
          pm |= ok ? 1u << (i * 8 + j) : 0u;
        }
      }
      const int mine = __popc(pm);
      int incl = mine;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const int y = __shfl_up_sync(kFull, incl, off);
        if (lane >= off) incl += y;
      }
      const int total = __shfl_sync(kFull, incl, 31);
      if (total == 0) continue;
      unsigned long long at0 = 0;
      if (lane == 0) at0 = atomicAdd(pcount, (unsigned long long)total);
      unsigned long long at = __shfl_sync(kFull, at0, 0) + (incl - mine);
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j)
          if (pm & (1u << (i * 8 + j))) {
            if (at < cap) {
              Pa[at] = sS[ga + 4 * i + 16 * p];
              Pd[at] = dd[i][j];
              Pb[at] = sS[tb[j]];
            } else {
              *overflow = 1;
            }
            ++at;
          }
    }
    __syncwarp();
  }
}

__global__ void prop_scatter_kernel(const int32_t* __restrict__ Pa, const float* __restrict__ Pd,
                                    const int32_t* __restrict__ Pb, const unsigned long long* pcount,
                                    const int64_t* __restrict__ off, int32_t* __restrict__ fill,
                                    uint64_t* __restrict__ seg) {
  const int64_t m = int64_t(*pcount);
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int32_t a = Pa[i];
    const int32_t p = atomicAdd(&fill[a], 1);
    seg[off[a] + p] = mkkey(Pd[i], Pb[i]);
  }
}

__global__ void prop_count_kernel(const int32_t* __restrict__ Pa, const unsigned long long* pcount,
                                  int32_t* __restrict__ cnt) {
  const int64_t m = int64_t(*pcount);
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
       i += int64_t(gridDim.x) * blockDim.x)
    atomicAdd(&cnt[Pa[i]], 1);
}

// Step 3 style merge with de-duplication; counts the lists that changed
__global__ void knn_merge_kernel(int64_t n, int K, int32_t* __restrict__ ids,
                                 float* __restrict__ dists, int32_t* __restrict__ cnt,
                                 int32_t* __restrict__ fill, const int64_t* __restrict__ off,
                                 const uint64_t* __restrict__ seg,
                                 unsigned long long* __restrict__ changed) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = int64_t(gridDim.x) * (blockDim.x >> 5);
  for (int64_t a = int64_t(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5); a < n; a += nw) {
    const int32_t m = cnt[a];
    if (m == 0) continue;
    const int32_t id0 = lane < K ? ids[size_t(a) * K + lane] : -1;
    uint64_t key = id0 >= 0 ? mkkey(dists[size_t(a) * K + lane], id0) : kKeyInf;
    bool ch = false;
    for (int32_t c = 0; c < m; c += 32) {
      const uint64_t x = c + lane < m ? seg[off[a] + c + lane] : kKeyInf;
      unsigned b = __ballot_sync(kFull, x < shfl64(key, K - 1));
      while (b) {
        const int src = __ffs(b) - 1;
        b &= b - 1;
        ch |= row_insert_unique(key, shfl64(x, src), K, lane);
      }
    }
    if (ch) {
      if (lane < K) {
        ids[size_t(a) * K + lane] = key_empty(key) ? -1 : key_id(key);
        dists[size_t(a) * K + lane] = key_empty(key) ? __int_as_float(0x7f800000) : key_dist(key);
      }
      if (lane == 0) atomicAdd(changed, 1ull);
    }
    __syncwarp();
    if (lane == 0) {
      cnt[a] = 0;
      fill[a] = 0;
    }
  }
}

template <typename T>
struct Buf {
  T* p = nullptr;
  cudaError_t alloc(size_t count) { return cudaMalloc(&p, std::max<size_t>(count, 1) * sizeof(T)); }
  ~Buf() { if (p) cudaFree(p); }
};

}  // namespace

#define KNN_TRY(...)                                                \
  do {                                                              \
    cudaError_t _e = (__VA_ARGS__);                                 \
    if (_e != cudaSuccess) return cuda_fail(_e, #__VA_ARGS__);      \
  } while (0)

template <bool L2>
static int knn_t(const float* X, int64_t n, int d, int K, const int32_t* init_dev, int max_iters,
                 int32_t* out_ids, int* iters_out, int64_t* changed_last, cudaStream_t s) {
  const int d4 = d / 4;
  const int64_t mrows = 2 * K;
  const unsigned long long cap = (unsigned long long)n * mrows * (mrows - 1);
  Buf<float> dists, Pd;
  Buf<int32_t> rev, cnt, fill, Pa, Pb;
  Buf<int64_t> off;
  Buf<uint64_t> seg;
  Buf<unsigned long long> counters;   // [0] bucket total, [1] proposals, [2] changed
  Buf<int> overflow;
  KNN_TRY(dists.alloc(size_t(n) * K));
  KNN_TRY(rev.alloc(size_t(n) * K));
  KNN_TRY(cnt.alloc(size_t(n)));
  KNN_TRY(fill.alloc(size_t(n)));
  KNN_TRY(off.alloc(size_t(n)));
  KNN_TRY(Pa.alloc(cap));
  KNN_TRY(Pb.alloc(cap));
  KNN_TRY(Pd.alloc(cap));
  KNN_TRY(seg.alloc(std::max<unsigned long long>(cap, (unsigned long long)n * K)));
  KNN_TRY(counters.alloc(3));
  KNN_TRY(overflow.alloc(1));
  KNN_TRY(cudaMemsetAsync(cnt.p, 0, sizeof(int32_t) * n, s));
  KNN_TRY(cudaMemsetAsync(fill.p, 0, sizeof(int32_t) * n, s));
  KNN_TRY(cudaMemsetAsync(overflow.p, 0, sizeof(int), s));
  const unsigned grid = 148 * 16;
  knn_init_kernel<L2><<<grid, 128, 0, s>>>(X, n, d4, K, init_dev, out_ids, dists.p);
  count_launch();
  KNN_TRY(cudaGetLastError());
  const bool tiled = GANNS_KNN_TILED != 0;
  const size_t smem = size_t(kKnnWarps) * (tiled ? knn_tiled_warp_smem(d4) : knn_warp_smem(d4));
  if (smem > 227 * 1024) return fail(GANNS_ENOTSUP, "knn: staged rows exceed shared memory");
  KNN_TRY(cudaFuncSetAttribute(knn_propose_kernel<L2>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               int(smem)));
  KNN_TRY(cudaFuncSetAttribute(knn_propose_tiled_kernel<L2>,
                               cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  int it = 0;
  unsigned long long h[3] = {0, 0, 0};
  for (; it < max_iters;) {
    KNN_TRY(cudaMemsetAsync(counters.p, 0, sizeof(unsigned long long) * 3, s));
    // reverse lists
    bucket_count_kernel<<<grid, 256, 0, s>>>(out_ids, n * K, cnt.p);
    bucket_carve_kernel<<<grid, 256, 0, s>>>(cnt.p, n, off.p, counters.p);
    rev_scatter_kernel<<<grid, 256, 0, s>>>(out_ids, dists.p, n, K, off.p, fill.p, seg.p);
    rev_select_kernel<<<grid, 128, 0, s>>>(n, K, cnt.p, fill.p, off.p, seg.p, rev.p);
    // proposals
    if (tiled)
      knn_propose_tiled_kernel<L2><<<grid, kKnnWarps * 32, smem, s>>>(
          X, n, d4, K, out_ids, dists.p, rev.p, Pa.p, Pd.p, Pb.p, counters.p + 1, cap, overflow.p);
    else
      knn_propose_kernel<L2><<<grid, kKnnWarps * 32, smem, s>>>(X, n, d4, K, out_ids, dists.p,
                                                             rev.p, Pa.p, Pd.p, Pb.p,
                                                             counters.p + 1, cap, overflow.p);
    // bucket by a, merge
    KNN_TRY(cudaMemsetAsync(counters.p, 0, sizeof(unsigned long long), s));
    prop_count_kernel<<<grid, 256, 0, s>>>(Pa.p, counters.p + 1, cnt.p);
    bucket_carve_kernel<<<grid, 256, 0, s>>>(cnt.p, n, off.p, counters.p);
    prop_scatter_kernel<<<grid, 256, 0, s>>>(Pa.p, Pd.p, Pb.p, counters.p + 1, off.p, fill.p, seg.p);
    knn_merge_kernel<<<grid, 128, 0, s>>>(n, K, out_ids, dists.p, cnt.p, fill.p, off.p, seg.p,
                                          counters.p + 2);
    count_launch(9);
    KNN_TRY(cudaGetLastError());
    KNN_TRY(cudaMemcpyAsync(h, counters.p, sizeof(h), cudaMemcpyDeviceToHost, s));
    int of = 0;
    KNN_TRY(cudaMemcpyAsync(&of, overflow.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    KNN_TRY(cudaStreamSynchronize(s));
    if (of) return fail(GANNS_ENOMEM, "knn: proposal buffer overflow");
    ++it;
    if (h[2] == 0) break;
  }
  *iters_out = it;
  *changed_last = int64_t(h[2]);
  return GANNS_OK;
}

int run_knn(const float* X, int64_t n, int d, int metric, int K, const int32_t* init_dev,
            int max_iters, int32_t* out_ids, int* iters_out, int64_t* changed_last,
            cudaStream_t s) {
  return metric == 0 ? knn_t<true>(X, n, d, K, init_dev, max_iters, out_ids, iters_out,
                                   changed_last, s)
                     : knn_t<false>(X, n, d, K, init_dev, max_iters, out_ids, iters_out,
                                    changed_last, s);
}

}  // namespace ganns
