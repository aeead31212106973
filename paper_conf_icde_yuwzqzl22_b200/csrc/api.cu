// api.cu -- the C ABI of libganns.so (include/ganns.h): argument validation,
// graph handles, error reporting, the host-buffer pipeline and save/load.
// Every compute step runs in the kernels of search.cu / build.cu.
#include "../../include/ganns.h"
#include "ganns_internal.h"

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <exception>
#include <mutex>
#include <new>
#include <unordered_map>
#include <vector>

namespace ganns {

static thread_local std::string g_last_error;
static std::atomic<uint64_t> g_launches{0};

void set_error(const std::string& msg) { g_last_error = msg; }
int fail(int status, const std::string& msg) {
  g_last_error = msg;
  return status;
}
int cuda_fail(cudaError_t e, const char* what) {
  return fail(GANNS_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
void count_launch(uint64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

cudaError_t pool_alloc(void** p, size_t bytes, cudaStream_t s) {
  static std::atomic<uint64_t> raised{0};
  cudaError_t e = once_per_device(raised, [] {
    int dev = 0;
    cudaMemPool_t mp;
    cudaError_t r = cudaGetDevice(&dev);
    if (r == cudaSuccess) r = cudaDeviceGetDefaultMemPool(&mp, dev);
    uint64_t thr = ~uint64_t(0);
    if (r == cudaSuccess) r = cudaMemPoolSetAttribute(mp, cudaMemPoolAttrReleaseThreshold, &thr);
    return r;
  });
  if (e != cudaSuccess) return e;
  return cudaMallocAsync(p, bytes, s);
}

unsigned long long* prof_buffer() {
#if GANNS_PROFILE
  static std::mutex mu;
  static unsigned long long* buf[64] = {nullptr};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lock(mu);
  if (!buf[dev]) {
    if (cudaMalloc(&buf[dev], kProfSlots * sizeof(unsigned long long)) != cudaSuccess) return nullptr;
    cudaMemset(buf[dev], 0, kProfSlots * sizeof(unsigned long long));
  }
  return buf[dev];
#else
  return nullptr;
#endif
}

void pool_free(void* p, cudaStream_t s) {
  if (p) cudaFreeAsync(p, s);
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no link-time
// dependency on libcuda).  Maps are cached per (pointer, n, d).
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
struct TmapCacheEntry {
  const float* X = nullptr;
  int64_t n = 0;
  int d = 0;
  CUtensorMap map;
};
static std::mutex g_tmap_mu;
static TmapCacheEntry g_tmap_cache[8];
static int g_tmap_next = 0;

cudaError_t zero_tmap(CUtensorMap* out) {
  std::memset(out, 0, sizeof(*out));
  return cudaSuccess;
}

cudaError_t encode_row_tmap(const float* X, int64_t n, int d, CUtensorMap* out) {
  std::lock_guard<std::mutex> lock(g_tmap_mu);
  for (auto& e : g_tmap_cache)
    if (e.X == X && e.n == n && e.d == d) {
      *out = e.map;
      return cudaSuccess;
    }
  static EncodeTiledFn enc = nullptr;
  if (!enc) {
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", reinterpret_cast<void**>(&enc),
                                cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess || !enc)
      return cudaErrorNotSupported;
  }
  const cuuint64_t dims[2] = {cuuint64_t(d), cuuint64_t(n)};
  const cuuint64_t strides[1] = {cuuint64_t(d) * 4};
  const cuuint32_t box[2] = {cuuint32_t(d), 1};
  const cuuint32_t es[2] = {1, 1};
  CUresult r = enc(out, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(X), dims, strides,
                   box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return cudaErrorInvalidValue;
  TmapCacheEntry& e = g_tmap_cache[g_tmap_next];
  g_tmap_next = (g_tmap_next + 1) % 8;
  e.X = X;
  e.n = n;
  e.d = d;
  e.map = *out;
  return cudaSuccess;
}

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

static int check_graph(const ganns_graph* g) {
  if (g == nullptr || g->nbr == nullptr) return fail(GANNS_EINVAL, "graph is NULL");
  return GANNS_OK;
}

// Pipeline state for ganns_search_host: two streams and double-buffered device
// staging, grown on demand (one set per device, guarded by a mutex).
struct HostPipe {
  int device = -1;
  cudaStream_t st[2] = {nullptr, nullptr};
  cudaEvent_t ev = nullptr;
  float* dq[2] = {nullptr, nullptr};
  int32_t* dids[2] = {nullptr, nullptr};
  float* ddst[2] = {nullptr, nullptr};
  size_t cap_q = 0, cap_r = 0;
};
static std::mutex g_pipe_mu;
static HostPipe g_pipes[64];

// Ticket counters for the persistent search kernel: one device int per (device,
// stream).  A launch resets its stream's counter with a memset on that stream, so
// consecutive launches on one stream are ordered and launches on different
// streams never share a counter.  Up to kTicketSlots streams per device get
// their own slot; beyond that, slots are shared round-robin (two launches in
// flight on two streams that share a slot would race: documented limit).
constexpr int kTicketSlots = 4096;
static std::mutex g_ticket_mu;
static int32_t* g_tickets[64] = {nullptr};
static std::unordered_map<cudaStream_t, int32_t> g_ticket_of[64];

int32_t* ticket_slot(cudaStream_t stream) {
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return nullptr;
  std::lock_guard<std::mutex> lock(g_ticket_mu);
  if (!g_tickets[dev] && cudaMalloc(&g_tickets[dev], sizeof(int32_t) * kTicketSlots) != cudaSuccess) {
    g_tickets[dev] = nullptr;
    return nullptr;
  }
  auto& m = g_ticket_of[dev];
  auto it = m.find(stream);
  if (it == m.end())
    it = m.emplace(stream, int32_t(m.size() % kTicketSlots)).first;
  return g_tickets[dev] + it->second;
}


// H2D, search, D2H of one batch on `stream` (no sync); `search` enqueues the search
// on the device copies.
template <class SEARCH>
int host_async(int d, const float* queries_host, int64_t nq, int k, float* queries_dev,
                      int32_t* ids_dev, float* dists_dev, int32_t* out_ids_host,
                      float* out_dists_host, void* stream, SEARCH&& search) {
  if (nq < 0) return fail(GANNS_EINVAL, "nq < 0");
  if (nq == 0) return GANNS_OK;
  if (!queries_host || !queries_dev || !ids_dev || !dists_dev || !out_ids_host || !out_dists_host)
    return fail(GANNS_EINVAL, "NULL buffer");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t err = cudaMemcpyAsync(queries_dev, queries_host, sizeof(float) * size_t(nq) * d,
                                    cudaMemcpyHostToDevice, s);
  if (err != cudaSuccess) return cuda_fail(err, "H2D queries");
  if (int rc = search()) return rc;
  err = cudaMemcpyAsync(out_ids_host, ids_dev, sizeof(int32_t) * size_t(nq) * k,
                        cudaMemcpyDeviceToHost, s);
  if (err == cudaSuccess)
    err = cudaMemcpyAsync(out_dists_host, dists_dev, sizeof(float) * size_t(nq) * k,
                          cudaMemcpyDeviceToHost, s);
  return err == cudaSuccess ? GANNS_OK : cuda_fail(err, "D2H results");
}

// R-C14: automatic group size = clamp(1.5 sqrt n rounded to a multiple of 256, 256,
// 8192) -- 1536 at n = 1M.  The build takes ~ s * t_insert (Phase 1, s sequential
// insertions per group) + (n / s) * t_round (Phase 2): measured on C2 (B200, l_build
// 128, l_local 64) 0.72 s at s = 1024, 0.65 s at 1536, 0.72 s at 2048, with the same
// search recall at every s.
int64_t auto_group_size(int64_t n) {
  const double t = 1.5 * std::sqrt(double(std::max<int64_t>(n, 1)));
  const int64_t s = int64_t(std::llround(t / 256.0)) * 256;
  return std::min<int64_t>(8192, std::max<int64_t>(256, s));
}

}  // namespace ganns

using namespace ganns;

extern "C" {

const char* ganns_last_error(void) { return g_last_error.c_str(); }
uint64_t ganns_kernel_launches(void) { return g_launches.load(); }

int ganns_profile_read_n(uint64_t* out, int count, int reset) {
  unsigned long long* p = prof_buffer();
  if (!p) return fail(GANNS_ENOTSUP, "library built without GANNS_PROFILE");
  if (!out) return fail(GANNS_EINVAL, "out is NULL");
  if (count < 0 || count > kProfSlots) return fail(GANNS_EINVAL, "count out of range");
  cudaError_t e = cudaDeviceSynchronize();
  if (e == cudaSuccess) e = cudaMemcpy(out, p, size_t(count) * sizeof(uint64_t), cudaMemcpyDeviceToHost);
  if (e == cudaSuccess && reset) e = cudaMemset(p, 0, kProfSlots * sizeof(uint64_t));
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "ganns_profile_read");
}

int ganns_profile_read(uint64_t* out, int reset) { return ganns_profile_read_n(out, 8, reset); }

int ganns_graph_info(const ganns_graph* g, int64_t* n, int* d, int* d_max, int* metric) {
  if (int rc = check_graph(g)) return rc;
  if (n) *n = g->n;
  if (d) *d = g->d;
  if (d_max) *d_max = g->d_max;
  if (metric) *metric = g->metric;
  return GANNS_OK;
}

int ganns_graph_device_ptr(const ganns_graph* g, const int32_t** nbr) {
  if (int rc = check_graph(g)) return rc;
  if (!nbr) return fail(GANNS_EINVAL, "nbr is NULL");
  *nbr = g->nbr;
  return GANNS_OK;
}

void ganns_graph_free(ganns_graph* g) {
  if (!g) return;
  if (g->nbr) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(g->device);
    // like cudaFree, wait for the device; the rows go back to the pool (no unmap:
    // a cudaFree of a 128 MB graph cost up to 0.46 s of host time)
    cudaDeviceSynchronize();
    pool_free(g->nbr, nullptr);
    cudaSetDevice(cur);
  }
  delete g;
}

static int validate_common(int64_t n, int d, int metric, int d_max) {
  if (n < 2 || n >= (int64_t(1) << 31)) return fail(GANNS_EINVAL, "n must be in [2, 2^31)");
  if (d < 4 || d % 4 != 0 || d > 1024) return fail(GANNS_EINVAL, "d must be a multiple of 4 in [4, 1024]");
  if (metric < 0 || metric > 2) return fail(GANNS_EINVAL, "unknown metric");
  if (d_max < 2 || d_max > 128) return fail(GANNS_EINVAL, "degree must be in [2, 128]");
  return GANNS_OK;
}

// The rows come from the device pool, ordered on `s` (the legacy stream for the
// synchronous entry points); every entry point that returns a graph synchronises
// before the caller may use it on another stream.
static int new_graph(int64_t n, int d, int d_max, int metric, ganns_graph** out,
                     cudaStream_t s = nullptr) {
  ganns_graph* g = new (std::nothrow) ganns_graph();
  if (!g) return fail(GANNS_ENOMEM, "host allocation failed");
  g->n = n;
  g->d = d;
  g->d_max = d_max;
  g->metric = metric;
  cudaGetDevice(&g->device);
  cudaError_t e = pool_alloc(reinterpret_cast<void**>(&g->nbr), sizeof(int32_t) * size_t(n) * d_max, s);
  if (e != cudaSuccess) {
    delete g;
    return fail(GANNS_ENOMEM, std::string("cudaMallocAsync(graph): ") + cudaGetErrorString(e));
  }
  *out = g;
  return GANNS_OK;
}

int ganns_graph_from_adjacency(const int32_t* nbr_host, int64_t n, int d_max, int d, int metric,
                               int device, ganns_graph** out) {
  if (!nbr_host || !out) return fail(GANNS_EINVAL, "NULL argument");
  if (int rc = validate_common(n, d, metric, d_max)) return rc;
  std::vector<int32_t> seen;   // row stamp per id
  try {
    seen.assign(size_t(n), -1);
  } catch (const std::exception&) {
    return fail(GANNS_ENOMEM, "host allocation failed (adjacency check)");
  }
  for (int64_t v = 0; v < n; ++v) {
    for (int j = 0; j < d_max; ++j) {
      int32_t u = nbr_host[size_t(v) * d_max + j];
      if (u < -1 || u >= n) return fail(GANNS_EINVAL, "adjacency id out of range");
      if (u < 0) continue;
      if (seen[u] == int32_t(v)) return fail(GANNS_EINVAL, "adjacency row repeats an id");
      seen[u] = int32_t(v);
    }
  }
  int cur = 0;
  cudaGetDevice(&cur);
  if (cudaSetDevice(device) != cudaSuccess) return fail(GANNS_EINVAL, "bad device");
  int rc = new_graph(n, d, d_max, metric, out);
  if (rc == GANNS_OK) {
    cudaError_t e = cudaMemcpy((*out)->nbr, nbr_host, sizeof(int32_t) * size_t(n) * d_max,
                               cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      ganns_graph_free(*out);
      *out = nullptr;
      rc = cuda_fail(e, "cudaMemcpy(adjacency)");
    }
  }
  cudaSetDevice(cur);
  return rc;
}

int ganns_graph_adjacency(const ganns_graph* g, int32_t* out_host) {
  if (int rc = check_graph(g)) return rc;
  if (!out_host) return fail(GANNS_EINVAL, "out is NULL");
  cudaError_t e = cudaMemcpy(out_host, g->nbr, sizeof(int32_t) * size_t(g->n) * g->d_max,
                             cudaMemcpyDeviceToHost);
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "cudaMemcpy(adjacency)");
}

int ganns_graph_save(const ganns_graph* g, const char* path) {
  if (int rc = check_graph(g)) return rc;
  if (!path) return fail(GANNS_EINVAL, "path is NULL");
  std::vector<int32_t> h;
  try {
    h.resize(size_t(g->n) * g->d_max);
  } catch (const std::exception&) {
    return fail(GANNS_ENOMEM, "host allocation failed (graph save)");
  }
  if (int rc = ganns_graph_adjacency(g, h.data())) return rc;
  FILE* f = std::fopen(path, "wb");
  if (!f) return fail(GANNS_EIO, std::string("cannot open ") + path);
  char magic[8] = {'G', 'A', 'N', 'N', 'S', 'G', '0', '1'};
  int64_t n = g->n;
  int32_t meta[4] = {g->d, g->d_max, g->metric, 0};
  bool ok = std::fwrite(magic, 1, 8, f) == 8 && std::fwrite(&n, 8, 1, f) == 1 &&
            std::fwrite(meta, 4, 4, f) == 4 && std::fwrite(h.data(), 4, h.size(), f) == h.size();
  ok = (std::fclose(f) == 0) && ok;
  return ok ? GANNS_OK : fail(GANNS_EIO, std::string("write failed: ") + path);
}

int ganns_graph_load(const char* path, int device, ganns_graph** out) {
  if (!path || !out) return fail(GANNS_EINVAL, "NULL argument");
  FILE* f = std::fopen(path, "rb");
  if (!f) return fail(GANNS_EIO, std::string("cannot open ") + path);
  char magic[8];
  int64_t n = 0;
  int32_t meta[4];
  bool ok = std::fread(magic, 1, 8, f) == 8 && std::memcmp(magic, "GANNSG01", 8) == 0 &&
            std::fread(&n, 8, 1, f) == 1 && std::fread(meta, 4, 4, f) == 4;
  // validate the header before allocating: sizes, dimension, metric, and the
  // file length must match exactly (a corrupt header never reaches the allocator)
  ok = ok && n >= 2 && n < (int64_t(1) << 31) && meta[1] >= 2 && meta[1] <= 128 &&
       meta[0] >= 4 && meta[0] <= 1024 && meta[0] % 4 == 0 && meta[2] >= 0 && meta[2] <= 2;
  const int64_t header = 8 + 8 + 16;
  if (ok) {
    ok = std::fseek(f, 0, SEEK_END) == 0 &&
         std::ftell(f) == header + int64_t(4) * n * meta[1] && std::fseek(f, header, SEEK_SET) == 0;
  }
  if (!ok) {
    std::fclose(f);
    return fail(GANNS_EIO, std::string("bad graph header or size: ") + path);
  }
  std::vector<int32_t> h;
  try {
    h.resize(size_t(n) * meta[1]);
  } catch (const std::exception&) {
    std::fclose(f);
    return fail(GANNS_ENOMEM, "host allocation failed (graph load)");
  }
  ok = std::fread(h.data(), 4, h.size(), f) == h.size();
  std::fclose(f);
  if (!ok) return fail(GANNS_EIO, std::string("truncated graph file: ") + path);
  return ganns_graph_from_adjacency(h.data(), n, meta[1], meta[0], meta[2], device, out);
}

static int validate_search(const ganns_graph* g, const float* points, const float* queries,
                           int64_t nq, int k, int l, const ganns_search_params* p,
                           const void* out_ids, const void* out_dists, int* e_out,
                           int32_t* entry_out) {
  if (int rc = check_graph(g)) return rc;
  // the persistent kernel's int32 ticket reaches nq + (resident warps): keep headroom
  if (nq < 0 || nq > (int64_t(1) << 31) - (int64_t(1) << 24))
    return fail(GANNS_EINVAL, "nq must be in [0, 2^31 - 2^24]");
  if (k < 1 || k >= g->n) return fail(GANNS_EINVAL, "k must be in [1, n)");
  if (l < k || l > 1024) return fail(GANNS_EINVAL, "l must be in [k, 1024]");
  int e = p ? p->e : 0;
  if (e < 0 || e > l) return fail(GANNS_EINVAL, "e must be in [0, l]");
  int64_t entry = p ? p->entry : 0;
  if (entry < 0 || entry >= g->n) return fail(GANNS_EINVAL, "entry out of range");
  if (nq > 0 && (!points || !queries || !out_ids || !out_dists))
    return fail(GANNS_EINVAL, "NULL pointer");
  if (!aligned16(points) || !aligned16(queries)) return fail(GANNS_EINVAL, "points/queries not 16-byte aligned");
  *e_out = e == 0 ? l : e;
  *entry_out = int32_t(entry);
  return GANNS_OK;
}

int ganns_search_ex(const ganns_graph* g, const float* points, const float* queries, int64_t nq,
                    int k, int l, const ganns_search_params* p, int32_t* out_ids,
                    float* out_dists, void* stream) {
  int e = 0;
  int32_t entry = 0;
  if (int rc = validate_search(g, points, queries, nq, k, l, p, out_ids, out_dists, &e, &entry))
    return rc;
  if (nq == 0) return GANNS_OK;
  int32_t* tk = ticket_slot(static_cast<cudaStream_t>(stream));
  if (!tk) return fail(GANNS_ENOMEM, "ticket allocation failed");
  SearchLaunch a{g->nbr, points, g->n, g->d, g->d_max, g->metric, queries, nq, k, l, e, entry,
                 out_ids, out_dists, p ? p->stats : nullptr, tk};
  cudaError_t err = launch_search(a, static_cast<cudaStream_t>(stream));
  return err == cudaSuccess ? GANNS_OK : cuda_fail(err, "search kernel launch");
}

int ganns_search(const ganns_graph* g, const float* points, const float* queries, int64_t nq,
                 int k, int l, int32_t* out_ids, float* out_dists, void* stream) {
  return ganns_search_ex(g, points, queries, nq, k, l, nullptr, out_ids, out_dists, stream);
}

int ganns_search_host(const ganns_graph* g, const float* points, const float* queries_host,
                      int64_t nq, int k, int l, const ganns_search_params* p,
                      int32_t* out_ids_host, float* out_dists_host, void* stream) {
  int e = 0;
  int32_t entry = 0;
  if (int rc = validate_search(g, points, queries_host, nq, k, l, p, out_ids_host,
                               out_dists_host, &e, &entry))
    return rc;
  if (p && p->stats) return fail(GANNS_EINVAL, "stats are not supported by ganns_search_host");
  if (nq == 0) return GANNS_OK;
  int dev = 0;
  cudaGetDevice(&dev);
  if (dev < 0 || dev >= 64) return fail(GANNS_ENOTSUP, "device ordinal >= 64");
  std::lock_guard<std::mutex> lock(g_pipe_mu);
  HostPipe& P = g_pipes[dev];
  if (P.device != dev) {
    for (int i = 0; i < 2; ++i)
      if (cudaStreamCreateWithFlags(&P.st[i], cudaStreamNonBlocking) != cudaSuccess)
        return fail(GANNS_ECUDA, "cudaStreamCreate failed");
    if (cudaEventCreateWithFlags(&P.ev, cudaEventDisableTiming) != cudaSuccess)
      return fail(GANNS_ECUDA, "cudaEventCreate failed");
    P.device = dev;
  }
  // chunking: every search launch pays a drain tail of about one query latency,
  // so chunks must be large (>= 64K queries) for the H2D/search/D2H overlap to
  // win; smaller batches go in one chunk (copies are ~5% of the search time).
  int64_t chunk = std::max<int64_t>(65536, (nq + 3) / 4);
  if (chunk > nq) chunk = nq;
  const size_t need_q = size_t(chunk) * g->d, need_r = size_t(chunk) * k;
  if (need_q > P.cap_q || need_r > P.cap_r) {
    for (int i = 0; i < 2; ++i) {
      cudaFree(P.dq[i]);
      cudaFree(P.dids[i]);
      cudaFree(P.ddst[i]);
      P.dq[i] = nullptr;
      P.dids[i] = nullptr;
      P.ddst[i] = nullptr;
    }
    P.cap_q = P.cap_r = 0;
    for (int i = 0; i < 2; ++i) {
      if (cudaMalloc(&P.dq[i], need_q * sizeof(float)) != cudaSuccess ||
          cudaMalloc(&P.dids[i], need_r * sizeof(int32_t)) != cudaSuccess ||
          cudaMalloc(&P.ddst[i], need_r * sizeof(float)) != cudaSuccess)
        return fail(GANNS_ENOMEM, "cudaMalloc(search_host staging)");
    }
    P.cap_q = need_q;
    P.cap_r = need_r;
  }
  cudaStream_t user = static_cast<cudaStream_t>(stream);
  cudaError_t err = cudaEventRecord(P.ev, user);
  for (int i = 0; i < 2 && err == cudaSuccess; ++i) err = cudaStreamWaitEvent(P.st[i], P.ev, 0);
  for (int64_t q0 = 0, c = 0; q0 < nq && err == cudaSuccess; q0 += chunk, ++c) {
    const int64_t m = std::min(chunk, nq - q0);
    const int b = int(c & 1);
    cudaStream_t s = P.st[b];
    err = cudaMemcpyAsync(P.dq[b], queries_host + size_t(q0) * g->d, sizeof(float) * m * g->d,
                          cudaMemcpyHostToDevice, s);
    if (err != cudaSuccess) break;
    int32_t* tk = ticket_slot(s);
    if (!tk) return fail(GANNS_ENOMEM, "ticket allocation failed");
    SearchLaunch a{g->nbr, points, g->n, g->d, g->d_max, g->metric, P.dq[b], m, k, l, e, entry,
                   P.dids[b], P.ddst[b], nullptr, tk};
    err = launch_search(a, s);
    if (err != cudaSuccess) break;
    err = cudaMemcpyAsync(out_ids_host + size_t(q0) * k, P.dids[b], sizeof(int32_t) * m * k,
                          cudaMemcpyDeviceToHost, s);
    if (err == cudaSuccess)
      err = cudaMemcpyAsync(out_dists_host + size_t(q0) * k, P.ddst[b], sizeof(float) * m * k,
                            cudaMemcpyDeviceToHost, s);
  }
  for (int i = 0; i < 2; ++i) {
    cudaError_t e2 = cudaStreamSynchronize(P.st[i]);
    if (err == cudaSuccess) err = e2;
  }
  return err == cudaSuccess ? GANNS_OK : cuda_fail(err, "ganns_search_host");
}


int ganns_search_host_async(const ganns_graph* g, const float* points, const float* queries_host,
                            int64_t nq, int k, int l, const ganns_search_params* p,
                            float* queries_dev, int32_t* ids_dev, float* dists_dev,
                            int32_t* out_ids_host, float* out_dists_host, void* stream) {
  if (int rc = check_graph(g)) return rc;
  return host_async(g->d, queries_host, nq, k, queries_dev, ids_dev, dists_dev, out_ids_host,
                    out_dists_host, stream, [&] {
                      return ganns_search_ex(g, points, queries_dev, nq, k, l, p, ids_dev,
                                             dists_dev, stream);
                    });
}

// Arguments of Algorithm 2 (validated; defaults applied) -> BuildArgs.
static int build_args(const float* points, int64_t n, int d, int metric, int degree,
                      const ganns_build_params* p, BuildArgs* out) {
  if (!points) return fail(GANNS_EINVAL, "NULL argument");
  if (int rc = validate_common(n, d, metric, degree)) return rc;
  if (!aligned16(points)) return fail(GANNS_EINVAL, "points not 16-byte aligned");
  int d_min = p && p->d_min > 0 ? p->d_min : degree / 2;
  if (d_min < 1) d_min = 1;
  int l_build = p && p->l_build > 0 ? p->l_build : 64;
  int e_build = p && p->e_build > 0 ? p->e_build : l_build;
  if (d_min > degree) return fail(GANNS_EINVAL, "d_min > degree");
  if (d_min >= n) return fail(GANNS_EINVAL, "d_min must be < n");
  if (l_build < d_min || l_build > 1024) return fail(GANNS_EINVAL, "l_build must be in [d_min, 1024]");
  if (e_build < 1 || e_build > l_build) return fail(GANNS_EINVAL, "e_build must be in [1, l_build]");
  const int l_local = p && p->l_local > 0 ? p->l_local : l_build;
  if (l_local < d_min || l_local > l_build) return fail(GANNS_EINVAL, "l_local must be in [d_min, l_build]");
  if (p && p->group_size < 0) return fail(GANNS_EINVAL, "group_size < 0");
  int64_t S = p && p->group_size > 0 ? p->group_size : 0;
  if (S == 0) S = auto_group_size(n);
  if (S > n) S = n;
  BuildArgs a{};
  a.X = points;
  a.n = n;
  a.d = d;
  a.metric = metric == GANNS_COSINE ? GANNS_IP : metric;   // symmetric keys inside the build
  a.d_max = degree;
  a.d_min = d_min;
  a.l_build = l_build;
  a.e_build = e_build;
  a.l_local = l_local;
  a.e_local = std::min(e_build, l_local);
  a.group_size = S;
  a.max_rounds = p ? (p->stop_after_phase1 ? 0 : (p->max_rounds > 0 ? p->max_rounds : -1)) : -1;
  *out = a;
  return GANNS_OK;
}

int ganns_build(const float* points, int64_t n, int d, int metric, int degree,
                const ganns_build_params* p, void* stream, ganns_graph** out) {
  if (!points || !out) return fail(GANNS_EINVAL, "NULL argument");
  BuildArgs a{};
  if (int rc = build_args(points, n, d, metric, degree, p, &a)) return rc;
  int rc = new_graph(n, d, degree, metric, out, static_cast<cudaStream_t>(stream));
  if (rc) return rc;
  a.out_nbr = (*out)->nbr;
  rc = run_build(a, static_cast<cudaStream_t>(stream));
  if (rc) {
    ganns_graph_free(*out);
    *out = nullptr;
    return rc;
  }
  if (p && p->stats)
    for (int i = 0; i < 4; ++i) p->stats[i] = a.stats[i];
  return GANNS_OK;
}

// ------------------------------------------------ staged Algorithm 2 (NEXT-2)
}  // extern "C"

struct ganns_build_state {
  ganns::BuildState st;
  ganns_graph* graph = nullptr;   // the rows being built (becomes the result)
  int64_t rounds_applied = 0;
};

namespace {
int check_state(const ganns_build_state* s) {
  if (!s || !s->graph || !s->st.phase1) return fail(GANNS_EINVAL, "build state is NULL or finished");
  return GANNS_OK;
}
int64_t group_lo(const BuildState& st, int64_t g) { return std::min(g * st.S, st.a.n); }
}  // namespace

extern "C" {

int ganns_build_begin(const float* points, int64_t n, int d, int metric, int degree,
                      const ganns_build_params* p, void* stream, ganns_build_state** out) {
  if (!points || !out) return fail(GANNS_EINVAL, "NULL argument");
  BuildArgs a{};
  if (int rc = build_args(points, n, d, metric, degree, p, &a)) return rc;
  ganns_build_state* s = new (std::nothrow) ganns_build_state();
  if (!s) return fail(GANNS_ENOMEM, "host allocation failed");
  int rc = new_graph(n, d, degree, metric, &s->graph, static_cast<cudaStream_t>(stream));
  if (rc) {
    delete s;
    return rc;
  }
  a.out_nbr = s->graph->nbr;
  s->st.a = a;
  rc = build_begin(s->st, static_cast<cudaStream_t>(stream));
  if (rc) {
    ganns_build_abort(s);
    return rc;
  }
  s->st.group_ready.assign(size_t(s->st.ngroups), 0);
  *out = s;
  return GANNS_OK;
}

int ganns_build_info(const ganns_build_state* s, int64_t* group_size, int64_t* ngroups,
                     int* d_min, int* d_max) {
  if (int rc = check_state(s)) return rc;
  if (group_size) *group_size = s->st.S;
  if (ngroups) *ngroups = s->st.ngroups;
  if (d_min) *d_min = s->st.a.d_min;
  if (d_max) *d_max = s->st.a.d_max;
  return GANNS_OK;
}

int ganns_build_phase1(ganns_build_state* s, int64_t g0, int64_t g1, void* stream) {
  if (int rc = check_state(s)) return rc;
  BuildState& st = s->st;
  if (g0 < 0 || g1 > st.ngroups || g0 > g1) return fail(GANNS_EINVAL, "groups must satisfy 0 <= g0 <= g1 <= ngroups");
  if (s->rounds_applied > 0) return fail(GANNS_EINVAL, "Phase 1 after a Phase-2 round");
  if (int rc = st.phase1(st, g0, g1, static_cast<cudaStream_t>(stream))) return rc;
  for (int64_t g = g0; g < g1; ++g) st.group_ready[size_t(g)] = 1;
  return GANNS_OK;
}

int ganns_build_rows(ganns_build_state* s, int64_t v0, int64_t v1, int32_t* ids, float* dists,
                     int32_t* pids, float* pdists, int to_state, void* stream) {
  if (int rc = check_state(s)) return rc;
  BuildState& st = s->st;
  if (v0 < 0 || v1 > st.a.n || v0 > v1) return fail(GANNS_EINVAL, "rows must satisfy 0 <= v0 <= v1 <= n");
  if (v1 > v0 && (!ids || !dists || !pids || !pdists)) return fail(GANNS_EINVAL, "NULL buffer");
  const size_t m = size_t(v1 - v0), dmax = size_t(st.a.d_max), dm = size_t(st.a.d_min);
  const cudaMemcpyKind k = cudaMemcpyDeviceToDevice;
  cudaStream_t cs = static_cast<cudaStream_t>(stream);
  int32_t* gid = s->graph->nbr + size_t(v0) * dmax;
  float* gd = st.gdist + size_t(v0) * dmax;
  int32_t* gpi = st.gpid + size_t(v0) * dm;
  float* gpd = st.gpd + size_t(v0) * dm;
  cudaError_t e;
  if (to_state) {
    e = cudaMemcpyAsync(gid, ids, 4 * m * dmax, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(gd, dists, 4 * m * dmax, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(gpi, pids, 4 * m * dm, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(gpd, pdists, 4 * m * dm, k, cs);
  } else {
    e = cudaMemcpyAsync(ids, gid, 4 * m * dmax, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dists, gd, 4 * m * dmax, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(pids, gpi, 4 * m * dm, k, cs);
    if (e == cudaSuccess) e = cudaMemcpyAsync(pdists, gpd, 4 * m * dm, k, cs);
  }
  if (e != cudaSuccess) return cuda_fail(e, "ganns_build_rows");
  if (to_state)   // whole groups covered by imported rows are ready for Phase 2
    for (int64_t g = 0; g < st.ngroups; ++g)
      if (group_lo(st, g) >= v0 && group_lo(st, g + 1) <= v1) st.group_ready[size_t(g)] = 1;
  return GANNS_OK;
}

int ganns_build_round_search(ganns_build_state* s, int64_t i, int64_t v0, int64_t v1,
                             int32_t* f_ids, float* f_dists, void* stream) {
  if (int rc = check_state(s)) return rc;
  BuildState& st = s->st;
  if (i < 1 || i >= st.ngroups) return fail(GANNS_EINVAL, "round must be in [1, ngroups)");
  if (i != s->rounds_applied + 1) return fail(GANNS_EINVAL, "rounds must be applied in order");
  for (int64_t g = 0; g <= i; ++g)
    if (!st.group_ready[size_t(g)]) return fail(GANNS_EINVAL, "Phase 1 of a group <= i is missing");
  const int64_t lo = group_lo(st, i), hi = group_lo(st, i + 1);
  if (v0 < lo || v1 > hi || v0 > v1) return fail(GANNS_EINVAL, "vertices must lie in P_i");
  if (v1 > v0 && (!f_ids || !f_dists)) return fail(GANNS_EINVAL, "NULL buffer");
  return st.round_search(st, i, v0, v1, f_ids, f_dists, static_cast<cudaStream_t>(stream));
}

int ganns_build_round_apply(ganns_build_state* s, int64_t i, const int32_t* f_ids,
                            const float* f_dists, void* stream) {
  if (int rc = check_state(s)) return rc;
  BuildState& st = s->st;
  if (i < 1 || i >= st.ngroups) return fail(GANNS_EINVAL, "round must be in [1, ngroups)");
  if (i != s->rounds_applied + 1) return fail(GANNS_EINVAL, "rounds must be applied in order");
  if (!f_ids || !f_dists) return fail(GANNS_EINVAL, "NULL buffer");
  for (int64_t g = 0; g <= i; ++g)
    if (!st.group_ready[size_t(g)]) return fail(GANNS_EINVAL, "Phase 1 of a group <= i is missing");
  if (int rc = st.round_apply(st, i, f_ids, f_dists, static_cast<cudaStream_t>(stream))) return rc;
  s->rounds_applied = i;
  return GANNS_OK;
}

int ganns_build_finish(ganns_build_state* s, void* stream, uint64_t* stats, ganns_graph** out) {
  if (int rc = check_state(s)) return rc;
  if (!out) return fail(GANNS_EINVAL, "NULL argument");
  cudaStream_t cs = static_cast<cudaStream_t>(stream);
  unsigned long long hs[3];
  cudaError_t e = cudaMemcpyAsync(hs, s->st.stats, sizeof(hs), cudaMemcpyDeviceToHost, cs);
  if (e == cudaSuccess) e = cudaStreamSynchronize(cs);
  if (e != cudaSuccess) return cuda_fail(e, "ganns_build_finish");
  if (stats) {
    stats[0] = hs[0];
    stats[1] = hs[1];
    stats[2] = hs[2];
    stats[3] = uint64_t(s->rounds_applied);
  }
  *out = s->graph;
  s->graph = nullptr;
  s->st.stream = cs;   // the scratch returns to the pool in stream order
  delete s;
  return GANNS_OK;
}

void ganns_build_abort(ganns_build_state* s) {
  if (!s) return;
  if (s->graph) ganns_graph_free(s->graph);
  s->graph = nullptr;
  delete s;
}


// ---------------------------------------------------------------- HNSW
}  // extern "C"

struct ganns_hnsw {
  ganns_graph* base = nullptr;          // layer 0, original ids
  int nlayers = 0;
  int64_t layer_n[16] = {0};
  int32_t* upper[16] = {nullptr};       // device, layers 1..nlayers-1, shuffled ids
  int32_t* perm = nullptr;              // device [n]
  float* Xp = nullptr;                  // device [layer_n[1]][d], rows of the upper points
  int d = 0, d_max = 0, metric = 0, device = 0;
  int32_t entry0 = 0;                   // perm[0]: the entry when there is no upper layer
};

extern "C" {

void ganns_hnsw_free(ganns_hnsw* h) {
  if (!h) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(h->device);
  // like ganns_graph_free: wait for the device, return the index memory to the pool
  cudaDeviceSynchronize();
  for (auto* p : h->upper) pool_free(p, nullptr);
  pool_free(h->perm, nullptr);
  pool_free(h->Xp, nullptr);
  cudaSetDevice(cur);
  ganns_graph_free(h->base);
  delete h;
}

int ganns_build_hnsw(const float* points, int64_t n, int d, int metric, int degree,
                     const int8_t* levels_host, const ganns_build_params* p, void* stream,
                     ganns_hnsw** out) {
  if (!points || !out || !levels_host) return fail(GANNS_EINVAL, "NULL argument");
  if (int rc = validate_common(n, d, metric, degree)) return rc;
  if (!aligned16(points)) return fail(GANNS_EINVAL, "points not 16-byte aligned");
  const int d_min = p && p->d_min > 0 ? p->d_min : std::max(1, degree / 2);
  const int l_build = p && p->l_build > 0 ? p->l_build : 64;
  const int e_build = p && p->e_build > 0 ? p->e_build : l_build;
  if (d_min > degree || d_min >= n) return fail(GANNS_EINVAL, "bad d_min");
  if (l_build < d_min || l_build > 1024) return fail(GANNS_EINVAL, "l_build must be in [d_min, 1024]");
  if (e_build < 1 || e_build > l_build) return fail(GANNS_EINVAL, "e_build must be in [1, l_build]");
  const int l_local = p && p->l_local > 0 ? p->l_local : l_build;
  if (l_local < d_min || l_local > l_build) return fail(GANNS_EINVAL, "l_local must be in [d_min, l_build]");
  // (1) shuffled ids: points by level descending, ties by id (stable counting sort)
  int top = 0;
  for (int64_t v = 0; v < n; ++v) {
    if (levels_host[v] < 0 || levels_host[v] >= 16) return fail(GANNS_EINVAL, "level outside [0, 16)");
    top = std::max(top, int(levels_host[v]));
  }
  std::vector<int32_t> perm(static_cast<size_t>(n));
  std::vector<int64_t> cntl(17, 0);
  for (int64_t v = 0; v < n; ++v) cntl[levels_host[v]]++;
  int64_t layer_n[16] = {0};
  for (int j = top; j >= 0; --j) layer_n[j] = cntl[j] + (j < top ? layer_n[j + 1] : 0);
  {
    std::vector<int64_t> pos(17, 0);
    for (int j = top; j >= 0; --j) pos[j] = (j < top ? pos[j + 1] + cntl[j + 1] : 0);
    for (int64_t v = 0; v < n; ++v) perm[pos[levels_host[v]]++] = int32_t(v);
  }
  ganns_hnsw* h = new (std::nothrow) ganns_hnsw();
  if (!h) return fail(GANNS_ENOMEM, "host allocation failed");
  cudaGetDevice(&h->device);
  h->nlayers = top + 1;
  h->d = d;
  h->d_max = degree;
  h->metric = metric;
  for (int j = 0; j <= top; ++j) h->layer_n[j] = layer_n[j];
  h->entry0 = perm[0];
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  float* Xfull = nullptr;
  int32_t* layer0_shuffled = nullptr;
  int rc = GANNS_OK;
  uint64_t tot[4] = {0, 0, 0, 0};
  auto cleanup = [&](int code) {
    pool_free(Xfull, s);
    pool_free(layer0_shuffled, s);
    if (code) ganns_hnsw_free(h);
    return code;
  };
  // index memory from the stream-ordered pool (as graph rows: cudaMalloc/cudaFree of
  // index-sized buffers cost variable host time inside the build)
  if (pool_alloc(reinterpret_cast<void**>(&h->perm), sizeof(int32_t) * n, s) != cudaSuccess ||
      pool_alloc(reinterpret_cast<void**>(&Xfull), sizeof(float) * size_t(n) * d, s) != cudaSuccess ||
      pool_alloc(reinterpret_cast<void**>(&layer0_shuffled), sizeof(int32_t) * size_t(n) * degree,
                 s) != cudaSuccess)
    return cleanup(fail(GANNS_ENOMEM, "cudaMalloc(hnsw scratch)"));
  cudaError_t e = cudaMemcpyAsync(h->perm, perm.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess) e = launch_gather_rows(points, h->perm, n, d, Xfull, s);
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "hnsw permute"));
  // (2) layers top-down, each Algorithm 2 on its prefix
  UpperLayersHost U;
  U.top = top;
  for (int j = top; j >= 0; --j) {
    int32_t* dst = layer0_shuffled;
    if (j >= 1) {
      if (pool_alloc(reinterpret_cast<void**>(&h->upper[j]), sizeof(int32_t) * size_t(layer_n[j]) * degree,
                     s) != cudaSuccess)
        return cleanup(fail(GANNS_ENOMEM, "cudaMalloc(hnsw layer)"));
      dst = h->upper[j];
    }
    BuildArgs a{};
    a.X = Xfull;
    a.n = layer_n[j];
    a.d = d;
    a.metric = metric == GANNS_COSINE ? GANNS_IP : metric;
    a.d_max = degree;
    a.d_min = d_min;
    a.l_build = l_build;
    a.e_build = e_build;
    a.l_local = l_local;   // every layer's Phase-1 searches (R-C13)
    a.e_local = std::min(e_build, l_local);
    int64_t S = p && p->group_size > 0 ? p->group_size : 0;
    if (S == 0) S = auto_group_size(layer_n[j]);
    a.group_size = std::max<int64_t>(1, std::min<int64_t>(S, layer_n[j]));
    a.max_rounds = -1;
    a.out_nbr = dst;
    a.upper = U;
    a.upper.top = j < top ? top : 0;   // layers above j are finished
    a.layer = j;
    rc = run_build(a, s);
    if (rc) return cleanup(rc);
    for (int i = 0; i < 4; ++i) tot[i] += a.stats[i];
    if (j >= 1) {
      U.nbr[j] = h->upper[j];
      U.n[j] = layer_n[j];
    }
  }
  // (3) recover the original ids of layer 0
  ganns_graph* base = nullptr;
  rc = new_graph(n, d, degree, metric, &base, s);
  if (rc) return cleanup(rc);
  h->base = base;
  e = launch_relabel(layer0_shuffled, h->perm, n, degree, base->nbr, s);
  if (e == cudaSuccess && top >= 1) {
    if (pool_alloc(reinterpret_cast<void**>(&h->Xp), sizeof(float) * size_t(layer_n[1]) * d, s) !=
        cudaSuccess)
      return cleanup(fail(GANNS_ENOMEM, "cudaMalloc(hnsw upper rows)"));
    e = cudaMemcpyAsync(h->Xp, Xfull, sizeof(float) * size_t(layer_n[1]) * d,
                        cudaMemcpyDeviceToDevice, s);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cleanup(cuda_fail(e, "hnsw finalize"));
  if (p && p->stats)
    for (int i = 0; i < 4; ++i) p->stats[i] = tot[i];
  *out = h;
  return cleanup(GANNS_OK);
}

int ganns_hnsw_search(const ganns_hnsw* h, const float* points, const float* queries, int64_t nq,
                      int k, int l, const ganns_search_params* p, int32_t* out_ids,
                      float* out_dists, void* stream) {
  if (!h || !h->base) return fail(GANNS_EINVAL, "hnsw is NULL");
  int e = 0;
  int32_t entry = 0;
  if (int rc = validate_search(h->base, points, queries, nq, k, l, p, out_ids, out_dists, &e, &entry))
    return rc;
  if (nq == 0) return GANNS_OK;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  const ganns_graph* g = h->base;
  if (h->nlayers > 1 && nv4_for(h->d) <= 2) {
    // d <= 256: the descent runs inside K1, one launch (search_inst.cu: HnswUpper)
    UpperLayersHost up;
    up.top = h->nlayers - 1;
    for (int j = 1; j < h->nlayers; ++j) {
      up.nbr[j] = h->upper[j];
      up.n[j] = h->layer_n[j];
    }
    int32_t* tk = ticket_slot(s);
    if (!tk) return fail(GANNS_ENOMEM, "ticket allocation failed");
    SearchLaunch a{g->nbr, points, g->n, g->d, g->d_max, g->metric, queries, nq, k, l, e, entry,
                   out_ids, out_dists, p ? p->stats : nullptr, tk};
    a.upper = &up;
    a.Xp = h->Xp;
    a.np = h->layer_n[1];
    a.perm = h->perm;
    a.dstats = p ? p->descent_stats : nullptr;
    cudaError_t err = launch_search(a, s);
    return err == cudaSuccess ? GANNS_OK : cuda_fail(err, "hnsw search");
  }
  int32_t* entries = nullptr;
  if (cudaMallocAsync(&entries, sizeof(int32_t) * nq, s) != cudaSuccess)
    return fail(GANNS_ENOMEM, "cudaMallocAsync(entries)");
  cudaError_t err = cudaSuccess;
  if (h->nlayers > 1) {
    EntryLaunch ea;
    ea.upper.top = h->nlayers - 1;
    for (int j = 1; j < h->nlayers; ++j) {
      ea.upper.nbr[j] = h->upper[j];
      ea.upper.n[j] = h->layer_n[j];
    }
    ea.Xp = h->Xp;
    ea.np = h->layer_n[1];
    ea.d = h->d;
    ea.d_max = h->d_max;
    ea.metric = h->metric;
    ea.Q = queries;
    ea.nq = nq;
    ea.perm = h->perm;
    ea.entries = entries;
    ea.dstats = p ? p->descent_stats : nullptr;
    err = launch_entries(ea, s);
  } else {
    entry = h->entry0;   // a single layer: every query enters at perm[0]
    cudaFreeAsync(entries, s);
    entries = nullptr;
    if (p && p->descent_stats)   // no descent
      err = cudaMemsetAsync(p->descent_stats, 0, sizeof(uint32_t) * 2 * size_t(nq), s);
  }
  if (err != cudaSuccess) {
    if (entries) cudaFreeAsync(entries, s);
    return cuda_fail(err, "hnsw entries");
  }
  int32_t* tk = ticket_slot(s);
  if (!tk) return fail(GANNS_ENOMEM, "ticket allocation failed");
  SearchLaunch a{g->nbr, points, g->n, g->d, g->d_max, g->metric, queries, nq, k, l, e, entry,
                 out_ids, out_dists, p ? p->stats : nullptr, tk};
  a.entries = entries;
  err = launch_search(a, s);
  if (entries) cudaFreeAsync(entries, s);
  return err == cudaSuccess ? GANNS_OK : cuda_fail(err, "hnsw search");
}

int ganns_hnsw_search_host_async(const ganns_hnsw* h, const float* points,
                                 const float* queries_host, int64_t nq, int k, int l,
                                 const ganns_search_params* p, float* queries_dev,
                                 int32_t* ids_dev, float* dists_dev, int32_t* out_ids_host,
                                 float* out_dists_host, void* stream) {
  if (!h || !h->base) return fail(GANNS_EINVAL, "hnsw is NULL");
  return host_async(h->d, queries_host, nq, k, queries_dev, ids_dev, dists_dev, out_ids_host,
                    out_dists_host, stream, [&] {
                      return ganns_hnsw_search(h, points, queries_dev, nq, k, l, p, ids_dev,
                                               dists_dev, stream);
                    });
}

int ganns_hnsw_info(const ganns_hnsw* h, int* nlayers, int64_t* layer_n) {
  if (!h) return fail(GANNS_EINVAL, "hnsw is NULL");
  if (nlayers) *nlayers = h->nlayers;
  if (layer_n)
    for (int j = 0; j < h->nlayers; ++j) layer_n[j] = h->layer_n[j];
  return GANNS_OK;
}

int ganns_hnsw_layer(const ganns_hnsw* h, int layer, int32_t* out_host) {
  if (!h || !out_host) return fail(GANNS_EINVAL, "NULL argument");
  if (layer < 0 || layer >= h->nlayers) return fail(GANNS_EINVAL, "layer out of range");
  if (layer == 0) return ganns_graph_adjacency(h->base, out_host);
  cudaError_t e = cudaMemcpy(out_host, h->upper[layer], sizeof(int32_t) * size_t(h->layer_n[layer]) * h->d_max,
                             cudaMemcpyDeviceToHost);
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "cudaMemcpy(layer)");
}

int ganns_hnsw_perm(const ganns_hnsw* h, int32_t* out_host) {
  if (!h || !out_host) return fail(GANNS_EINVAL, "NULL argument");
  cudaError_t e = cudaMemcpy(out_host, h->perm, sizeof(int32_t) * size_t(h->layer_n[0]),
                             cudaMemcpyDeviceToHost);
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "cudaMemcpy(perm)");
}

int ganns_hnsw_base(const ganns_hnsw* h, const ganns_graph** base) {
  if (!h || !base) return fail(GANNS_EINVAL, "NULL argument");
  *base = h->base;
  return GANNS_OK;
}

int ganns_build_knn(const float* points, int64_t n, int d, int metric, int K,
                    const int32_t* init_host, int max_iters, void* stream, ganns_graph** out,
                    int* iters_out, int64_t* changed_last) {
  if (!points || !init_host || !out) return fail(GANNS_EINVAL, "NULL argument");
  if (int rc = validate_common(n, d, metric, 2)) return rc;
  if (K < 1 || K > 32 || K >= n) return fail(GANNS_EINVAL, "K must be in [1, min(32, n-1)]");
  if (max_iters < 0) return fail(GANNS_EINVAL, "max_iters < 0");
  if (!aligned16(points)) return fail(GANNS_EINVAL, "points not 16-byte aligned");
  for (int64_t v = 0; v < n; ++v)
    for (int j = 0; j < K; ++j) {
      const int32_t u = init_host[size_t(v) * K + j];
      if (u < 0 || u >= n || u == v) return fail(GANNS_EINVAL, "init: ids must be in [0, n) and != row");
      for (int i = 0; i < j; ++i)
        if (init_host[size_t(v) * K + i] == u) return fail(GANNS_EINVAL, "init: repeated id in a row");
    }
  int rc = new_graph(n, d, K, metric, out);
  if (rc) return rc;
  int32_t* init_dev = nullptr;
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaMalloc(&init_dev, sizeof(int32_t) * size_t(n) * K);
  if (e == cudaSuccess)
    e = cudaMemcpy(init_dev, init_host, sizeof(int32_t) * size_t(n) * K, cudaMemcpyHostToDevice);
  if (e != cudaSuccess) {
    cudaFree(init_dev);
    ganns_graph_free(*out);
    *out = nullptr;
    return cuda_fail(e, "knn init upload");
  }
  int it = 0;
  int64_t ch = 0;
  rc = run_knn(points, n, d, metric == GANNS_COSINE ? GANNS_IP : metric, K, init_dev, max_iters,
               (*out)->nbr, &it, &ch, s);
  cudaFree(init_dev);
  if (rc) {
    ganns_graph_free(*out);
    *out = nullptr;
    return rc;
  }
  if (iters_out) *iters_out = it;
  if (changed_last) *changed_last = ch;
  return GANNS_OK;
}

int ganns_merge_topk(const int32_t* shard_ids, const float* shard_dists, int W, int64_t nq, int k,
                     int32_t* out_ids, float* out_dists, void* stream) {
  if (W < 1 || k < 1 || nq < 0) return fail(GANNS_EINVAL, "bad W / k / nq");
  if (size_t(W) * k * kWarpsPerBlock * 8 > 200 * 1024) return fail(GANNS_ENOTSUP, "W*k too large");
  if (nq > 0 && (!shard_ids || !shard_dists || !out_ids || !out_dists))
    return fail(GANNS_EINVAL, "NULL pointer");
  cudaError_t e = launch_merge_topk(shard_ids, shard_dists, W, nq, k, out_ids, out_dists,
                                    static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "merge_topk launch");
}

int ganns_offset_ids(int32_t* ids, int64_t count, int64_t offset, void* stream) {
  if (count < 0 || (count > 0 && !ids)) return fail(GANNS_EINVAL, "bad ids/count");
  if (offset < 0 || offset >= (int64_t(1) << 31)) return fail(GANNS_EINVAL, "offset out of range");
  cudaError_t e = launch_offset_ids(ids, count, offset, static_cast<cudaStream_t>(stream));
  return e == cudaSuccess ? GANNS_OK : cuda_fail(e, "offset_ids launch");
}

}  // extern "C"
