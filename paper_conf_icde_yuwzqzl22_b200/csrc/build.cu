// build.cu -- host driver of the GGraphCon construction (Algorithm 2):
// the one-GPU build (ganns_build) and the state the staged multi-GPU build
// (ganns_build_begin ... ganns_build_finish, NEXT-2) advances step by step.  The
// kernels and their per-instance operations are in build_inst.cu.
#include "ganns_dev.cuh"
#include "../../include/ganns.h"
#include "ganns_internal.h"

#include <algorithm>

namespace ganns {

BuildState::~BuildState() {
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(device);
  for (void* p : {static_cast<void*>(gdist), static_cast<void*>(gpid), static_cast<void*>(gpd),
                  static_cast<void*>(Eu), static_cast<void*>(Ed), static_cast<void*>(indeg),
                  static_cast<void*>(fill), static_cast<void*>(segoff),
                  static_cast<void*>(touched), static_cast<void*>(seg),
                  static_cast<void*>(counters), static_cast<void*>(stats)})
    pool_free(p, stream);
  cudaSetDevice(cur);
  if (dev && dev_free) dev_free(dev);
}

int build_begin(BuildState& st, cudaStream_t s) {
  cudaGetDevice(&st.device);
  st.stream = s;
  switch (nv4_for(st.a.d)) {
    case 1: return build_begin_nv<1>(st, s);
#ifndef GANNS_DEV_NV1
    case 2: return build_begin_nv<2>(st, s);
    case 4: return build_begin_nv<4>(st, s);
    case 8: return build_begin_nv<8>(st, s);
#endif
  }
  return fail(GANNS_ENOTSUP, "unsupported dimension");
}

// One GPU: Phase 1 for every group at once, then the t rounds of Phase 2 with the
// fused round search (rows, E slots and in-degrees written by K3 itself).
int run_build(BuildArgs& a, cudaStream_t s) {
  BuildState st;
  st.a = a;
  if (int rc = build_begin(st, s)) return rc;
  if (int rc = st.phase1(st, 0, st.ngroups, s)) return rc;
  int64_t rounds = 0;
  const int64_t last = a.max_rounds < 0 ? st.ngroups - 1
                                         : std::min<int64_t>(st.ngroups - 1, a.max_rounds);
  for (int64_t i = 1; i <= last; ++i) {
    const int64_t lo = i * st.S, hi = std::min(lo + st.S, a.n);
    if (int rc = st.round_search(st, i, lo, hi, nullptr, nullptr, s)) return rc;
    if (int rc = st.round_merge(st, i, s)) return rc;
    ++rounds;
  }
  unsigned long long hs[3];
  cudaError_t e = cudaMemcpyAsync(hs, st.stats, sizeof(hs), cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "build stats");
  a.stats[0] = hs[0];
  a.stats[1] = hs[1];
  a.stats[2] = hs[2];
  a.stats[3] = uint64_t(rounds);
  return 0;
}

}  // namespace ganns
