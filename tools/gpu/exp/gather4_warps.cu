// Microbenchmark: does the TMA tile::gather4 issue rate scale with the number of issuing
// WARPS?  64 gather4 (256 rows of 96 B) per item, 4 items in flight, 148 CTAs of 512
// threads; the 64 gather4 of an item are spread over W warps x (64 / W) lanes (W = 1..16).
// Row indices are precomputed in registers (issue cost only).  L2-resident source.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void wait(uint64_t* bar, uint32_t ph) {
  asm volatile("{\n.reg .pred P1;\nW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W;\n}\n" ::"r"(su(bar)), "r"(ph) : "memory");
}
__global__ void k_tma(const __grid_constant__ CUtensorMap tm, const int* __restrict__ rows, int R, long long* out, int items,
                      int nwarps, int per_lane) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[4];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar[i])), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int lanes = 64 / nwarps / per_lane;   // issuing lanes per warp
  const bool issuer = warp < nwarps && lane < lanes;
  const int base = (warp * lanes + lane) * per_lane;   // first gather4 (of 64) of this thread
  int rr[4];
#pragma unroll
  for (int t = 0; t < 4; ++t) rr[t] = rows[(blockIdx.x * 7919 + threadIdx.x * 4 + t) % R];
  long long t0 = clock64();
  for (int it = 0; it < items; ++it) {
    const int b = it & 3;
    if (it >= 4) wait(&bar[b], ((it >> 2) - 1) & 1);
    __syncthreads();
    if (threadIdx.x == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar[b])), "r"(256 * 96) : "memory");
    __syncthreads();
    if (issuer)
      for (int g = 0; g < per_lane; ++g) {
        const int gg = base + g;
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(
                su(sm + b * 32768 + gg * 4 * 128)),
            "l"((uint64_t)&tm), "r"(0), "r"((rr[0] + it * 13 + g) % R), "r"((rr[1] + it * 7) % R), "r"((rr[2] + 3 * g) % R),
            "r"((rr[3] + it * 5) % R), "r"(su(&bar[b]))
            : "memory");
      }
  }
  for (int it = items - 4; it < items; ++it) wait(&bar[it & 3], (it >> 2) & 1);
  long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}
int main() {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  EncodeTiledFn fn = (EncodeTiledFn)p;
  cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  long long* dout;
  cudaMalloc(&dout, 148 * 8);
  std::vector<long long> h(148);
  const int items = 200;
  for (int R : {200000, 4000000}) {
    uint8_t* d;
    cudaMalloc(&d, (size_t)R * 96 + 4096);
    cudaMemset(d, 1, (size_t)R * 96);
    std::vector<int> rows(R);
    uint32_t x = 12345;
    for (int i = 0; i < R; ++i) { x = x * 1664525u + 1013904223u; rows[i] = (x >> 8) % R; }
    int* drows;
    cudaMalloc(&drows, (size_t)R * 4);
    cudaMemcpy(drows, rows.data(), (size_t)R * 4, cudaMemcpyHostToDevice);
    CUtensorMap tm;
    cuuint64_t dims[2] = {48, (cuuint64_t)R};
    cuuint64_t str[1] = {96};
    cuuint32_t box[2] = {48, 1};
    cuuint32_t es[2] = {1, 1};
    fn(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
       CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    struct C { int w, per; };
    for (C c : {C{1, 2}, C{2, 1}, C{4, 1}, C{4, 2}, C{4, 4}, C{8, 1}, C{8, 2}, C{8, 8}, C{16, 1}, C{16, 4}}) {
      for (int rep = 0; rep < 2; ++rep) k_tma<<<148, 512, 140000>>>(tm, drows, R, dout, items, c.w, c.per);
      cudaDeviceSynchronize();
      cudaMemcpy(h.data(), dout, 148 * 8, cudaMemcpyDeviceToHost);
      double m = 0;
      for (auto v : h) m += v;
      m /= 148;
      printf("R=%7d warps %2d lanes %2d per-lane %d: %6.0f cycles per 256-row item (%5.2f per row, %5.1f per gather4)  %s\n", R,
             c.w, 64 / c.w / c.per, c.per, m / items, m / items / 256, m / items / 64, cudaGetErrorString(cudaGetLastError()));
    }
    cudaFree(d);
    cudaFree(drows);
  }
  return 0;
}
