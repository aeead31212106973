// Probe of the sm_100a TMA tile::gather4 semantics (box dims, smem layout, OOB
// rows, tx byte count).  Standalone: nvcc -gencode arch=compute_100a,code=sm_100a
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*,
                             CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion,
                             CUtensorMapFloatOOBfill);

__global__ void k(const __grid_constant__ CUtensorMap map, int r0, int r1, int r2, int r3, int ncols,
                  float* out, int* done) {
  __shared__ alignas(128) float buf[4 * 256];
  __shared__ alignas(8) uint64_t mbar;
  uint32_t sb = uint32_t(__cvta_generic_to_shared(buf)), mb = uint32_t(__cvta_generic_to_shared(&mbar));
  for (int i = threadIdx.x; i < 4 * 256; i += 32) buf[i] = -7.f;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("fence.proxy.async.shared::cta;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(4 * ncols * 4));
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
        ::"r"(sb), "l"(&map), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(mb) : "memory");
    uint32_t ok = 0;
    for (int it = 0; it < 1000000 && !ok; ++it)
      asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                   : "=r"(ok) : "r"(mb) : "memory");
    *done = ok;
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 4 * 256; i += 32) out[i] = buf[i];
}

int main() {
  const int n = 1000, d = 128;
  std::vector<float> h(size_t(n) * d);
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < d; ++j) h[size_t(i) * d + j] = float(i * 1000 + j);
  float* X;
  cudaMalloc(&X, h.size() * 4);
  cudaMemcpy(X, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  EncodeFn enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  printf("entry point %p\n", (void*)enc);
  for (int box1 : {1, 4}) {
    CUtensorMap map;
    cuuint64_t dims[2] = {cuuint64_t(d), cuuint64_t(n)};
    cuuint64_t strides[1] = {cuuint64_t(d) * 4};
    cuuint32_t box[2] = {cuuint32_t(d), cuuint32_t(box1)};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, X, dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("box1=%d encode=%d\n", box1, int(r));
    if (r) continue;
    float* out;
    int* done;
    cudaMalloc(&out, 4 * 256 * 4);
    cudaMalloc(&done, 4);
    k<<<1, 32>>>(map, 5, 900, 3, 2000000000, d, out, done);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<float> ho(4 * 256);
    int hd = 0;
    cudaMemcpy(ho.data(), out, ho.size() * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(&hd, done, 4, cudaMemcpyDeviceToHost);
    printf("  kernel=%s done=%d\n", cudaGetErrorString(e), hd);
    for (int rr = 0; rr < 4; ++rr)
      printf("  row%d: %g %g ... %g | next %g\n", rr, ho[rr * d], ho[rr * d + 1], ho[rr * d + d - 1],
             ho[rr * d + d < 4 * 256 ? rr * d + d : 0]);
    cudaFree(out);
    cudaFree(done);
  }
  return 0;
}
