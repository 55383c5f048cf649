// Experiment: tcgen05.mma kind::f16 with the A operand in TMEM (written by tcgen05.st as
// packed bf16x2, two K elements per 32-bit column) and B from a SWIZZLE_128B K-major smem
// tile.  M = 128, N = 64, K = 64 (4 MMAs of K = 16 reading A columns 8i .. 8i + 7).
// Checks D against a CPU reference.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cmath>
#include <vector>
#include "../../../paper_conf_sc_pandeylfhl22_b200/csrc/tc_common.cuh"
using namespace psim::tc;

__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
__device__ __forceinline__ void mma_bf16_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(acc));
}

__global__ void k(const __nv_bfloat16* A, const __nv_bfloat16* B, float* D) {
  __shared__ __align__(1024) uint8_t sB[64 * 128];
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  // B [64 N][64 K] bf16 -> SW128 K-major atom
  for (int idx = tid; idx < 64 * 8; idx += blockDim.x) {
    const int r = idx / 8, c = idx % 8;
    st_sw128(sB, r, c, reinterpret_cast<const uint4*>(B)[idx]);
  }
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  if (warp == 0) tmem_alloc(&slot, 128);
  fence_async_smem();
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = slot;
  // A row m = lane 32 w + lane: columns 64 .. 95 hold A[m][0..63] as bf16x2
  {
    const int m = warp * 32 + lane;
    uint32_t r[16];
    for (int half = 0; half < 2; ++half) {
      for (int i = 0; i < 16; ++i) {
        const __nv_bfloat16 lo = A[m * 64 + half * 32 + 2 * i], hi = A[m * 64 + half * 32 + 2 * i + 1];
        r[i] = (uint32_t)__bfloat16_as_ushort(lo) | ((uint32_t)__bfloat16_as_ushort(hi) << 16);
      }
      tmem_st16(tmem + ((uint32_t)(warp * 32) << 16) + 64 + half * 16, r);
    }
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  if (tid == 0) {
    const uint32_t id = idesc_bf16(128, 64);
    for (int kk = 0; kk < 4; ++kk)
      mma_bf16_ts(tmem, tmem + 64 + 8 * kk, sw128_desc(smem_u32(sB) + 32 * kk), id, kk > 0);
    mma_commit(&bar);
  }
  mbar_wait(&bar, 0);
  fence_after();
  {
    uint32_t r0[32], r1[32];
    tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16), r0);
    tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16) + 32, r1);
    tmem_wait_ld();
    const int m = warp * 32 + lane;
    for (int i = 0; i < 32; ++i) { D[m * 64 + i] = __uint_as_float(r0[i]); D[m * 64 + 32 + i] = __uint_as_float(r1[i]); }
  }
  fence_before();
  __syncthreads();
  if (warp == 0) { fence_after(); tmem_dealloc(tmem, 128); }
}
int main() {
  std::vector<__nv_bfloat16> A(128 * 64), B(64 * 64);
  std::vector<float> Af(128 * 64), Bf(64 * 64);
  uint32_t x = 7;
  auto rnd = [&]() { x = x * 1664525u + 1013904223u; return ((x >> 9) % 2001) / 1000.0f - 1.0f; };
  for (int i = 0; i < 128 * 64; ++i) { A[i] = __float2bfloat16(rnd()); Af[i] = __bfloat162float(A[i]); }
  for (int i = 0; i < 64 * 64; ++i) { B[i] = __float2bfloat16(rnd()); Bf[i] = __bfloat162float(B[i]); }
  __nv_bfloat16 *dA, *dB; float* dD;
  cudaMalloc(&dA, A.size() * 2); cudaMalloc(&dB, B.size() * 2); cudaMalloc(&dD, 128 * 64 * 4);
  cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
  k<<<1, 128>>>(dA, dB, dD);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<float> D(128 * 64);
  cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
  double maxerr = 0;
  for (int m = 0; m < 128; ++m)
    for (int n = 0; n < 64; ++n) {
      double ref = 0;
      for (int kk = 0; kk < 64; ++kk) ref += (double)Af[m * 64 + kk] * Bf[n * 64 + kk];
      maxerr = fmax(maxerr, fabs(ref - D[m * 64 + n]));
    }
  printf("tmem-A MMA: %s, max |err| = %g (D[0]=%g)\n", cudaGetErrorString(e), maxerr, D[0]);
  return 0;
}
