// Microbenchmark: issue rate of TMA tile::gather4 vs cp.async (LDGSTS) for 1024 random 128-B rows
// per CTA (one item set = 256 rows into 32 KB), L2-resident source; 148 CTAs.
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
__global__ void k_tma(const __grid_constant__ CUtensorMap tm, const int* rows, int R, long long* out, int iters, int issuers, int rowbytes) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[4];
  if (threadIdx.x == 0) { for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar[i])), "r"(1)); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  __syncthreads();
  // per issuer: its gather4 row indices precomputed in registers (no loads in the loop)
  int rr[4];
  for (int t = 0; t < 4; ++t) rr[t] = rows[(blockIdx.x * 977 + threadIdx.x * 4 + t) % R];
  const int per = 64 / issuers;
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const int b = it & 3;
    if (it >= 4) wait(&bar[b], ((it >> 2) - 1) & 1);
    __syncthreads();
    if (threadIdx.x == 0) asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar[b])), "r"(256 * rowbytes) : "memory");
    __syncthreads();
    if (threadIdx.x < issuers)
      for (int g = 0; g < per; ++g) {
        const int gg = threadIdx.x * per + g;
        asm volatile("cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
            ::"r"(su(sm + b * 32768 + gg * 4 * rowbytes)), "l"((uint64_t)&tm), "r"(0), "r"(rr[0] + g), "r"(rr[1] + it), "r"(rr[2] + 3 * g), "r"((rr[3] + it * 7) % R), "r"(su(&bar[b])) : "memory");
      }
  }
  for (int it = iters - 4; it < iters; ++it) wait(&bar[it & 3], (it >> 2) & 1);
  long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}
__global__ void k_cpa(const uint8_t* src, const int* rows, int R, long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  long long t0 = clock64();
  for (int it = 0; it < iters; ++it) {
    // 256 rows x 8 chunks over blockDim threads
    for (int q = threadIdx.x; q < 256 * 8; q += blockDim.x) {
      const int r = q >> 3, c = q & 7;
      const int row = rows[((blockIdx.x * 977 + it * 256 + r)) % R];
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su(sm + r * 128 + ((c ^ (r & 7)) << 4))), "l"(src + (size_t)row * 128 + c * 16) : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncthreads();
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
}
int main() {
  void* p = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  EncodeTiledFn fn = (EncodeTiledFn)p;
  cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  long long* dout; cudaMalloc(&dout, 148 * 8);
  std::vector<long long> h(148);
  const int iters = 200;
  for (int R : {200000, 4000000}) {
    uint8_t* d; cudaMalloc(&d, (size_t)R * 128); cudaMemset(d, 1, (size_t)R * 128);
    std::vector<int> rows(R); uint32_t x = 12345; for (int i = 0; i < R; ++i) { x = x * 1664525u + 1013904223u; rows[i] = (x >> 8) % R; }
    int* drows; cudaMalloc(&drows, (size_t)R * 4); cudaMemcpy(drows, rows.data(), (size_t)R * 4, cudaMemcpyHostToDevice);
    struct V { const char* name; CUtensorMapDataType dt; int cols; int pitch; int box; CUtensorMapSwizzle sw; int rowbytes; };
    V vs[3] = {{"bf16 128B sw128", CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 64, 128, 64, CU_TENSOR_MAP_SWIZZLE_128B, 128},
               {"bf16  96B sw128", CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 48, 96, 48, CU_TENSOR_MAP_SWIZZLE_128B, 128},
               {"u8    48B none ", CU_TENSOR_MAP_DATA_TYPE_UINT8, 48, 48, 48, CU_TENSOR_MAP_SWIZZLE_NONE, 48}};
    for (auto& v : vs) {
      CUtensorMap tm;
      cuuint64_t dims[2] = {(cuuint64_t)v.cols, (cuuint64_t)R}; cuuint64_t str[1] = {(cuuint64_t)v.pitch};
      cuuint32_t box[2] = {(cuuint32_t)v.box, 1}; cuuint32_t es[2] = {1, 1};
      CUresult cr = fn(&tm, v.dt, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, v.sw,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (cr) { printf("%s encode error %d\n", v.name, (int)cr); continue; }
      // landed bytes per row: for the 96-B box with SW128 the smem row still takes 128 B of space but 96 B land
      const int landed = v.box * (v.dt == CU_TENSOR_MAP_DATA_TYPE_UINT8 ? 1 : 2);
      for (int issuers : {16, 64}) {
        for (int rep = 0; rep < 2; ++rep) k_tma<<<148, 128, 140000>>>(tm, drows, R, dout, iters, issuers, landed);
        cudaDeviceSynchronize();
        cudaMemcpy(h.data(), dout, 148 * 8, cudaMemcpyDeviceToHost);
        double m = 0; for (auto v2 : h) m += v2; m /= 148;
        printf("R=%7d %s issuers %2d: %6.0f cycles per 256-row item (%5.1f per gather4)  %s\n", R, v.name, issuers, m / iters,
               m / iters / 64, cudaGetErrorString(cudaGetLastError()));
      }
    }
    cudaFree(d); cudaFree(drows);
  }
  return 0;
}
