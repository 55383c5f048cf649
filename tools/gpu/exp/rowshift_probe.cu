// Experiment: does a SWIZZLE_128B K-major smem descriptor whose start address is shifted
// by whole 128-B rows (not 1024-B aligned) read the rows from that start, with the
// descriptor's base-offset field (bits 49..51) = (start >> 7) & 7?  (Needed to take a k3
// convolution's three taps as row-shifted views of ONE tile instead of three copies.)
// A: 136 rows x 64 bf16 in SW128 layout, A[r][k] = r + k / 64 (distinct per row);
// B = identity 64 x 64; D = A rows shift .. shift + 127 for shift in {0, 1, 2, 3, 7, 8}.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

#include "../../../paper_conf_sc_pandeylfhl22_b200/csrc/tc_common.cuh"
using namespace psim::tc;

__device__ uint64_t desc_shift(uint32_t saddr, int use_base_offset) {
  uint64_t d = sw128_desc(saddr);
  if (use_base_offset) d |= (uint64_t)((saddr >> 7) & 7) << 49;
  return d;
}

__global__ void k(const __nv_bfloat16* A, const __nv_bfloat16* B, int shift, int use_bo, float* D) {
  __shared__ __align__(1024) uint8_t sA[136 * 128];
  __shared__ __align__(1024) uint8_t sB[64 * 128];
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int idx = tid; idx < 136 * 8; idx += blockDim.x) st_sw128(sA, idx / 8, idx % 8, reinterpret_cast<const uint4*>(A)[idx]);
  for (int idx = tid; idx < 64 * 8; idx += blockDim.x) st_sw128(sB, idx / 8, idx % 8, reinterpret_cast<const uint4*>(B)[idx]);
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  if (warp == 0) tmem_alloc(&slot, 64);
  fence_async_smem();
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = slot;
  if (tid == 0) {
    const uint32_t a0 = smem_u32(sA) + shift * 128;
    for (int kk = 0; kk < 4; ++kk)
      mma_bf16(tmem, desc_shift(a0 + 32 * kk, use_bo), sw128_desc(smem_u32(sB) + 32 * kk), idesc_bf16(128, 64), kk > 0);
    mma_commit(&bar);
  }
  __syncwarp();
  mbar_wait(&bar, 0);
  fence_after();
  uint32_t r[32];
  tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16), r);
  tmem_wait_ld();
  for (int i = 0; i < 32; ++i) D[(warp * 32 + lane) * 64 + i] = __uint_as_float(r[i]);
  tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16) + 32, r);
  tmem_wait_ld();
  for (int i = 0; i < 32; ++i) D[(warp * 32 + lane) * 64 + 32 + i] = __uint_as_float(r[i]);
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 64);
}

int main() {
  std::vector<__nv_bfloat16> A(136 * 64), B(64 * 64);
  for (int r = 0; r < 136; ++r)
    for (int c = 0; c < 64; ++c) A[r * 64 + c] = __float2bfloat16((float)(r + (c % 2) * 0.5f));
  for (int n = 0; n < 64; ++n)
    for (int c = 0; c < 64; ++c) B[n * 64 + c] = __float2bfloat16(n == c ? 1.f : 0.f);
  __nv_bfloat16 *dA, *dB;
  float* dD;
  cudaMalloc(&dA, A.size() * 2); cudaMalloc(&dB, B.size() * 2); cudaMalloc(&dD, 128 * 64 * 4);
  cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
  for (int use_bo = 0; use_bo < 2; ++use_bo)
    for (int shift : {0, 1, 2, 3, 7, 8}) {
      cudaMemset(dD, 0, 128 * 64 * 4);
      k<<<1, 128>>>(dA, dB, shift, use_bo, dD);
      cudaError_t e = cudaDeviceSynchronize();
      if (e != cudaSuccess) { printf("shift %d bo %d: %s\n", shift, use_bo, cudaGetErrorString(e)); return 1; }
      std::vector<float> D(128 * 64);
      cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
      int bad = 0, first_bad = -1;
      for (int m = 0; m < 128; ++m)
        for (int c = 0; c < 64; ++c) {
          const float want = (float)(m + shift) + (c % 2) * 0.5f;
          if (D[m * 64 + c] != want) { if (!bad) first_bad = m * 64 + c; ++bad; }
        }
      printf("shift %d base_offset %d: %s (%d mismatches; D[0][0..3] = %g %g %g %g; D[1][0] = %g)\n", shift, use_bo,
             bad ? "WRONG" : "exact", bad, D[0], D[1], D[2], D[3], D[64]);
      (void)first_bad;
    }
  return 0;
}
