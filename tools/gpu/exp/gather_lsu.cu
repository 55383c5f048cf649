// Microbenchmark: random 96-B row gather into a SWIZZLE_128B smem tile, LSU path
// (LDG.128 -> registers -> STS, software-pipelined one tile ahead) vs TMA tile::gather4
// with 2/4/8 issuing warps.  148 CTAs, 1024-row tiles, L2-resident (19 MB) and
// DRAM-resident (384 MB) sources.  Row indices are read from global memory each tile
// (as the real gather reads queue entries).
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
constexpr int TROWS = 1024;   // rows per tile
// LSU: NT threads; tile rows split over threads as (row, chunk) pairs: 1024 x 6 = 6144 16-B chunks
template <int NT>
__global__ void k_lsu(const uint4* __restrict__ src, const int* __restrict__ rows, int R, long long* out, int tiles) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);   // one 128 KB tile buffer
  constexpr int PER = TROWS * 6 / NT;
  uint4 v[PER];
  int ridx[PER];
  const int tid = threadIdx.x;
  long long t0 = clock64();
  // prologue: tile 0 loads
#pragma unroll
  for (int u = 0; u < PER; ++u) {
    const int q = tid + u * NT, r = q / 6;
    ridx[u] = rows[(blockIdx.x * 7919 + r) % R];
  }
#pragma unroll
  for (int u = 0; u < PER; ++u) { const int q = tid + u * NT, c = q % 6; v[u] = src[(size_t)ridx[u] * 6 + c]; }
  for (int t = 0; t < tiles; ++t) {
    // indices of tile t+1 (independent of the loads in flight)
#pragma unroll
    for (int u = 0; u < PER; ++u) {
      const int q = tid + u * NT, r = q / 6;
      ridx[u] = rows[(blockIdx.x * 7919 + (t + 1) * TROWS + r) % R];
    }
    __syncthreads();   // the previous tile's consumer (none here) is done with the buffer
#pragma unroll
    for (int u = 0; u < PER; ++u) {
      const int q = tid + u * NT, r = q / 6, c = q % 6;
      *reinterpret_cast<uint4*>(sm + r * 128 + ((c ^ (r & 7)) << 4)) = v[u];
    }
#pragma unroll
    for (int u = 0; u < PER; ++u) { const int q = tid + u * NT, c = q % 6; v[u] = src[(size_t)ridx[u] * 6 + c]; }
  }
  __syncthreads();
  long long t1 = clock64();
  if (tid == 0) out[blockIdx.x] = (t1 - t0) + (long long)sm[5];
}
// TMA gather4: 1024-row tile = 4 items of 256 rows (32 KB each), 4 item buffers in flight.
// 'issuers' threads issue 64/issuers... (256 gather4 per tile / issuers each)
__global__ void k_tma(const __grid_constant__ CUtensorMap tm, const int* __restrict__ rows, int R, long long* out, int tiles,
                      int issuers) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar[4];
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar[i])), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int per = 64 / issuers > 0 ? 64 / issuers : 1;   // gather4 per issuer per item
  long long t0 = clock64();
  const int items = tiles * 4;
  for (int it = 0; it < items; ++it) {
    const int b = it & 3;
    // row indices of this item (loaded from global, like queue entries)
    int rr[4][4];
    if (threadIdx.x < issuers && threadIdx.x * per < 64) {
#pragma unroll
      for (int g = 0; g < 4; ++g)
        if (g < per)
#pragma unroll
          for (int t = 0; t < 4; ++t) rr[g][t] = rows[(blockIdx.x * 7919 + it * 256 + (threadIdx.x * per + g) * 4 + t) % R];
    }
    if (it >= 4) wait(&bar[b], ((it >> 2) - 1) & 1);
    __syncthreads();
    if (threadIdx.x == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar[b])), "r"(256 * 96) : "memory");
    __syncthreads();
    if (threadIdx.x < issuers && threadIdx.x * per < 64) {
#pragma unroll
      for (int g = 0; g < 4; ++g)
        if (g < per) {
          const int gg = threadIdx.x * per + g;
          asm volatile(
              "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(
                  su(sm + b * 32768 + gg * 4 * 128)),
              "l"((uint64_t)&tm), "r"(0), "r"(rr[g][0]), "r"(rr[g][1]), "r"(rr[g][2]), "r"(rr[g][3]), "r"(su(&bar[b]))
              : "memory");
        }
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
  cudaFuncSetAttribute(k_lsu<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  cudaFuncSetAttribute(k_lsu<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  cudaFuncSetAttribute(k_lsu<512>, cudaFuncAttributeMaxDynamicSharedMemorySize, 140000);
  long long* dout;
  cudaMalloc(&dout, 148 * 8);
  std::vector<long long> h(148);
  const int tiles = 50;
  auto report = [&](const char* name, int R) {
    cudaDeviceSynchronize();
    cudaMemcpy(h.data(), dout, 148 * 8, cudaMemcpyDeviceToHost);
    double m = 0;
    for (auto v2 : h) m += v2;
    m /= 148;
    printf("R=%7d %-28s %7.0f cycles per 1024-row tile (%5.2f per row)  %s\n", R, name, m / tiles, m / tiles / TROWS,
           cudaGetErrorString(cudaGetLastError()));
  };
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
    for (int rep = 0; rep < 2; ++rep) { k_lsu<128><<<148, 128, 140000>>>((const uint4*)d, drows, R, dout, tiles); }
    report("LSU 128 thr", R);
    for (int rep = 0; rep < 2; ++rep) { k_lsu<256><<<148, 256, 140000>>>((const uint4*)d, drows, R, dout, tiles); }
    report("LSU 256 thr", R);
    for (int rep = 0; rep < 2; ++rep) { k_lsu<512><<<148, 512, 140000>>>((const uint4*)d, drows, R, dout, tiles); }
    report("LSU 512 thr", R);
    CUtensorMap tm;
    cuuint64_t dims[2] = {48, (cuuint64_t)R};
    cuuint64_t str[1] = {96};
    cuuint32_t box[2] = {48, 1};
    cuuint32_t es[2] = {1, 1};
    CUresult cr = fn(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (cr) printf("encode error %d\n", (int)cr);
    for (int issuers : {16, 32, 64}) {
      for (int rep = 0; rep < 2; ++rep) k_tma<<<148, 256, 140000>>>(tm, drows, R, dout, tiles, issuers);
      char name[64];
      snprintf(name, sizeof name, "TMA gather4 %d issuers", issuers);
      report(name, R);
    }
    cudaFree(d);
    cudaFree(drows);
  }
  return 0;
}
