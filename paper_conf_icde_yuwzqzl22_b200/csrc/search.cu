// search.cu -- dispatch of K1, the batched GANNS search kernel (§III-B,
// P:193-216; instances in search_inst.cu), the HNSW bookkeeping kernels, and the
// multi-GPU helpers K6 (shard top-k merge) and the id offset.
//
// K1's launch shape (search_inst.cu): persistent, grid = SMs x resident CTAs of
// kSearchWarps warps; every warp takes queries from a per-launch atomic ticket
// (one warp per query, the paper's n_t = 32) until the batch is
// exhausted.  No other global scratch: the whole search of a query is one fused
// warp program (ganns_dev.cuh) and only the top-k leaves the SM.
#include "ganns_dev.cuh"
#include "ganns_internal.h"

namespace ganns {

cudaError_t launch_search(const SearchLaunch& a, cudaStream_t s) {
  if (a.nq == 0) return cudaSuccess;
  switch (nv4_for(a.d)) {
    case 1: return launch_search_nv<1>(a, s);
#ifndef GANNS_DEV_NV1
    case 2: return launch_search_nv<2>(a, s);
    case 4: return launch_search_nv<4>(a, s);
    case 8: return launch_search_nv<8>(a, s);
#endif
  }
  return cudaErrorInvalidValue;
}

cudaError_t launch_entries(const EntryLaunch& a, cudaStream_t s) {
  if (a.nq == 0) return cudaSuccess;
  switch (nv4_for(a.d)) {
    case 1: return launch_entries_nv<1>(a, s);
#ifndef GANNS_DEV_NV1
    case 2: return launch_entries_nv<2>(a, s);
    case 4: return launch_entries_nv<4>(a, s);
    case 8: return launch_entries_nv<8>(a, s);
#endif
  }
  return cudaErrorInvalidValue;
}

// HNSW bookkeeping: rows of the points in shuffled order, and the
// relabelling of layer 0 back to the original ids.
__global__ void gather_rows_kernel(const float4* __restrict__ X, const int32_t* __restrict__ perm,
                                   int64_t n, int d4, float4* __restrict__ Xp) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n * d4;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = i / d4, c = i % d4;
    Xp[i] = X[size_t(perm[r]) * d4 + c];
  }
}

cudaError_t launch_gather_rows(const float* X, const int32_t* perm, int64_t n, int d, float* Xp,
                               cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  gather_rows_kernel<<<148 * 16, 256, 0, s>>>(reinterpret_cast<const float4*>(X), perm, n, d / 4,
                                              reinterpret_cast<float4*>(Xp));
  count_launch();
  return cudaGetLastError();
}

__global__ void relabel_kernel(const int32_t* __restrict__ in, const int32_t* __restrict__ perm,
                               int64_t n, int d_max, int32_t* __restrict__ out) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n * d_max;
       i += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = i / d_max, c = i % d_max;
    const int32_t u = in[i];
    out[size_t(perm[r]) * d_max + c] = u >= 0 ? perm[u] : -1;
  }
}

cudaError_t launch_relabel(const int32_t* in, const int32_t* perm, int64_t n, int d_max,
                           int32_t* out, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  relabel_kernel<<<148 * 16, 256, 0, s>>>(in, perm, n, d_max, out);
  count_launch();
  return cudaGetLastError();
}

// ---------------------------------------------------------------- K6
// Per query, the k smallest (dist, global id) among W sorted shard lists.  One
// warp per query; each candidate's output position is its rank among all W*k
// candidates (keys are unique: shards hold disjoint id ranges).
__global__ void merge_topk_kernel(const int32_t* __restrict__ ids, const float* __restrict__ dists,
                                  int W, int64_t nq, int k, int32_t* __restrict__ out_ids,
                                  float* __restrict__ out_dists) {
  extern __shared__ uint64_t skeys[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t q = int64_t(blockIdx.x) * kWarpsPerBlock + w;
  if (q >= nq) return;
  const int m = W * k;
  uint64_t* sk = skeys + size_t(w) * m;
  for (int i = lane; i < m; i += 32) {
    int s = i / k, j = i % k;
    size_t off = (size_t(s) * nq + q) * k + j;
    int32_t id = ids[off];
    sk[i] = id < 0 ? kKeyInf : mkkey(dists[off], id);
  }
  for (int i = lane; i < k; i += 32) {
    out_ids[size_t(q) * k + i] = -1;
    out_dists[size_t(q) * k + i] = __int_as_float(0x7f800000);
  }
  __syncwarp();
  for (int i = lane; i < m; i += 32) {
    uint64_t key = sk[i];
    if (key_empty(key)) continue;
    int rank = 0;
    for (int j = 0; j < m; ++j) rank += sk[j] < key ? 1 : 0;
    if (rank < k) {
      out_ids[size_t(q) * k + rank] = key_id(key);
      out_dists[size_t(q) * k + rank] = key_dist(key);
    }
  }
}

cudaError_t launch_merge_topk(const int32_t* ids, const float* dists, int W, int64_t nq, int k,
                              int32_t* out_ids, float* out_dists, cudaStream_t s) {
  if (nq == 0) return cudaSuccess;
  const size_t smem = size_t(kWarpsPerBlock) * W * k * sizeof(uint64_t);
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(merge_topk_kernel,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
  }
  const int64_t blocks = (nq + kWarpsPerBlock - 1) / kWarpsPerBlock;
  merge_topk_kernel<<<unsigned(blocks), kWarpsPerBlock * 32, smem, s>>>(ids, dists, W, nq, k,
                                                                      out_ids, out_dists);
  count_launch();
  return cudaGetLastError();
}

__global__ void offset_ids_kernel(int32_t* ids, int64_t count, int32_t offset) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < count;
       i += int64_t(gridDim.x) * blockDim.x) {
    int32_t v = ids[i];
    if (v >= 0) ids[i] = v + offset;
  }
}

cudaError_t launch_offset_ids(int32_t* ids, int64_t count, int64_t offset, cudaStream_t s) {
  if (count == 0) return cudaSuccess;
  int64_t blocks = (count + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  offset_ids_kernel<<<unsigned(blocks), 256, 0, s>>>(ids, count, int32_t(offset));
  count_launch();
  return cudaGetLastError();
}

}  // namespace ganns
