// ganns_internal.h -- host-side declarations shared by the .cu translation units
// of libganns.so (not part of the public ABI; see include/ganns.h).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <atomic>
#include <cstdint>
#include <string>
#include <vector>

struct ganns_graph {
  int32_t* nbr = nullptr;   // device [n][d_max]
  int64_t n = 0;
  int d = 0;
  int d_max = 0;
  int metric = 0;
  int device = 0;
};

namespace ganns {

constexpr int kWarpsPerBlock = 4;   // warps per CTA of the small helper kernels
#ifndef GANNS_SEARCH_WARPS
#define GANNS_SEARCH_WARPS 2
#endif
#ifndef GANNS_SEARCH_POOL
#define GANNS_SEARCH_POOL 0
#endif
constexpr int kSearchWarps = GANNS_SEARCH_WARPS;   // warps (= concurrent queries) per CTA
constexpr int kSearchPool = GANNS_SEARCH_POOL;     // shared stage buffers per CTA (0: one per warp)
#ifndef GANNS_MIN_BLOCKS
#define GANNS_MIN_BLOCKS (24 / GANNS_SEARCH_WARPS)
#endif
constexpr int kMinBlocksPerSM = GANNS_MIN_BLOCKS; // register budget: <= 85 regs/thread (24 warps per SM);
                                    // the TMA stage (8 KB/warp at d=128) allows ~22 warps
#ifndef GANNS_MIN_BLOCKS_WIDE
#define GANNS_MIN_BLOCKS_WIDE (16 / GANNS_SEARCH_WARPS)
#endif
// d > 128 (NV4 >= 2): register budget 128/thread (<= 16 warps per SM).  The 2-round
// TMA stage is 16 rows x d x 4 B = 8.4-16 KB per warp for d in (128, 256], plus N;
// at the bench's C4 point (d = 200, l = 288, 13 KB + 2.3 KB per warp) shared memory
// already caps residency at 14 warps, so 128 registers cost nothing there and remove
// the spills of the 80-register budget (268 B/thread, 566 MB of DRAM writes per
// launch).  For d ~ 132-176 with small l, shared memory would allow ~20 warps and
// this cap (16) may cost occupancy; only d = 200 was measured.
constexpr int kMinBlocksWide = GANNS_MIN_BLOCKS_WIDE;

// cudaFuncSetAttribute state is per device: run `set` once per device ordinal
// (bit d of `done`); concurrent first calls may both run `set`, which is idempotent.
template <class F>
inline cudaError_t once_per_device(std::atomic<uint64_t>& done, F&& set) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return set();
  const uint64_t bit = uint64_t(1) << dev;
  if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
  e = set();
  if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
  return e;
}

// Stream-ordered scratch from the device's default memory pool.  The pool's release
// threshold is raised once per device, so freed blocks stay mapped for the next
// build: a cudaMalloc/cudaFree of the build scratch cost 2 ms typically and up to
// 1 s of host time (profiles/r02/build_phases_host_gap.log), the pool 0.02 ms.
cudaError_t pool_alloc(void** p, size_t bytes, cudaStream_t s);
// GANNS_PROFILE builds: the current device's phase counters (8 x u64), else nullptr
constexpr int kProfSlots = 16;   // GANNS_PROFILE counters (ganns_dev.cuh, ganns_profile_read_n)
unsigned long long* prof_buffer();
void pool_free(void* p, cudaStream_t s);

void set_error(const std::string& msg);
int fail(int status, const std::string& msg);
int cuda_fail(cudaError_t e, const char* what);
void count_launch(uint64_t n = 1);
// TMA tensor map of the point rows (2-D {d, n}, box {d, 1}) for tile::gather4.
cudaError_t encode_row_tmap(const float* X, int64_t n, int d, CUtensorMap* out);
cudaError_t zero_tmap(CUtensorMap* out);

// Template selectors.
inline int nv4_for(int d) {
  int d4 = d / 4;
  return d4 <= 32 ? 1 : d4 <= 64 ? 2 : d4 <= 128 ? 4 : d4 <= 256 ? 8 : -1;
}
inline int tpl_for(int d_max) { return d_max <= 32 ? 1 : d_max <= 64 ? 2 : d_max <= 128 ? 4 : -1; }

struct UpperLayersHost {
  int top = 0;
  const int32_t* nbr[16] = {nullptr};
  int64_t n[16] = {0};
};

struct SearchLaunch {
  const int32_t* nbr;
  const float* X;
  int64_t n;
  int d, d_max, metric;
  const float* Q;
  int64_t nq;
  int k, l, e;
  int32_t entry;
  int32_t* out_ids;
  float* out_dists;
  uint32_t* stats;
  int32_t* ticket;      // device scratch counter for the persistent scheduler
  const int32_t* entries = nullptr;   // per-query entry vertices (HNSW), nullable
  // HNSW with the descent fused into K1 (d <= 256): upper layers over the permuted
  // rows Xp [np][d]; a query enters layer 0 at perm[vertex its descent reaches]
  const UpperLayersHost* upper = nullptr;
  const float* Xp = nullptr;
  int64_t np = 0;
  const int32_t* perm = nullptr;
  uint32_t* dstats = nullptr;   // HNSW: nullable [nq][2] descent iterations / comps
};
// HNSW: per-query layer-0 entry = perm[greedy descent through the upper layers]
struct EntryLaunch {
  UpperLayersHost upper;
  const float* Xp;      // permuted points, prefix [0, n_1)
  int64_t np;           // rows of Xp
  int d, d_max, metric;
  const float* Q;
  int64_t nq;
  const int32_t* perm;
  int32_t* entries;
  uint32_t* dstats = nullptr;   // nullable [nq][2] descent iterations / comps
};
cudaError_t launch_entries(const EntryLaunch& a, cudaStream_t s);
template <int NV4>
cudaError_t launch_entries_nv(const EntryLaunch& a, cudaStream_t s);
cudaError_t launch_gather_rows(const float* X, const int32_t* perm, int64_t n, int d, float* Xp,
                               cudaStream_t s);
cudaError_t launch_relabel(const int32_t* in, const int32_t* perm, int64_t n, int d_max,
                           int32_t* out, cudaStream_t s);
int32_t* ticket_slot(cudaStream_t stream);   // the search kernel's ticket counter of `stream`
cudaError_t launch_search(const SearchLaunch& a, cudaStream_t s);
template <int NV4>
cudaError_t launch_search_nv(const SearchLaunch& a, cudaStream_t s);

struct BuildArgs {
  const float* X;
  int64_t n;
  int d, metric, d_max, d_min, l_build, e_build;
  int l_local = 0, e_local = 0;   // Phase-1 searches (0: l_build / e_build)
  int64_t group_size;
  int max_rounds;       // < 0: all
  int32_t* out_nbr;     // device [n][d_max]
  uint64_t stats[4];    // out: iterations, distance computations, searches, rounds
  UpperLayersHost upper;   // HNSW: finished layers above `layer` (top = 0: plain NSW)
  int layer = 0;
};
// One Algorithm-2 construction, step by step (build.cu drives it; the per-instance
// operations come from build_inst.cu).  Device scratch is owned by the state.
struct BuildState {
  BuildArgs a{};
  int64_t S = 0, ngroups = 0;
  float* gdist = nullptr;      // [n][d_max] distance half of the build-form rows
  int32_t* gpid = nullptr;     // G' [n][d_min]
  float* gpd = nullptr;
  int32_t* Eu = nullptr;       // E of one round [s][d_min] (fixed slots)
  float* Ed = nullptr;
  int32_t* indeg = nullptr;    // GatherScatter counters [n]
  int32_t* fill = nullptr;
  int32_t* segoff = nullptr;
  int32_t* touched = nullptr;  // [s * d_min]
  uint64_t* seg = nullptr;     // [s * d_min]
  int32_t* counters = nullptr; // [4]: GatherScatter counters of even / odd rounds
  unsigned long long* stats = nullptr;   // [3] iterations, comps, searches
  CUtensorMap tmap;
  cudaStream_t stream = nullptr;         // the scratch is stream-ordered on this stream
  void* dev = nullptr;                   // instance-private block (build_inst.cu)
  void (*dev_free)(void*) = nullptr;
  int device = 0;
  // operations of the (NV4, TPL, L2) instance
  int (*phase1)(BuildState&, int64_t g0, int64_t g1, cudaStream_t) = nullptr;
  int (*round_search)(BuildState&, int64_t i, int64_t v0, int64_t v1, int32_t* f_ids,
                      float* f_dists, cudaStream_t) = nullptr;
  int (*round_merge)(BuildState&, int64_t i, cudaStream_t) = nullptr;
  int (*round_apply)(BuildState&, int64_t i, const int32_t* f_ids, const float* f_dists,
                     cudaStream_t) = nullptr;
  // staged-API bookkeeping: groups whose rows are final for Phase 1 (built here or
  // imported), and the next Phase-2 round
  std::vector<uint8_t> group_ready;
  int64_t next_round = 1;
  ~BuildState();
};
int build_begin(BuildState& st, cudaStream_t s);   // scratch + instance operations
template <int NV4>
int build_begin_nv(BuildState& st, cudaStream_t s);
int run_build(BuildArgs& a, cudaStream_t s);       // the whole construction on one GPU

int run_knn(const float* X, int64_t n, int d, int metric, int K, const int32_t* init_dev,
            int max_iters, int32_t* out_ids, int* iters_out, int64_t* changed_last,
            cudaStream_t s);

cudaError_t launch_merge_topk(const int32_t* ids, const float* dists, int W, int64_t nq, int k,
                              int32_t* out_ids, float* out_dists, cudaStream_t s);
cudaError_t launch_offset_ids(int32_t* ids, int64_t count, int64_t offset, cudaStream_t s);

}  // namespace ganns
