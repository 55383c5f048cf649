// gemm_simt.cu -- CUDA-core GEMM for the fp32 path (PSIM_FP32, parity stage
// S2 at 1e-3) and the reference bf16-operand path the tensor-core kernel is
// checked against: C[M][N] = act(A[M][K] . W[N][K]^T + b[N]), fp32 accumulate.
// 64x64 output tile per 256-thread block, 4x4 per thread, K step 16.
#include "internal.h"

namespace psim {

template <typename TA>
__device__ __forceinline__ float ldf(const TA* p);
template <>
__device__ __forceinline__ float ldf<float>(const float* p) { return __ldg(p); }
template <>
__device__ __forceinline__ float ldf<__nv_bfloat16>(const __nv_bfloat16* p) { return __bfloat162float(*p); }

template <typename TA, typename TC>
__global__ void __launch_bounds__(256) gemm_simt_kernel(const TA* __restrict__ A, const TA* __restrict__ W,
                                                        const float* __restrict__ bias, TC* __restrict__ C,
                                                        int64_t M, int N, int K, bool relu) {
  __shared__ float As[16][64 + 4];
  __shared__ float Ws[16][64 + 4];
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  const int64_t m0 = (int64_t)blockIdx.x * 64;
  const int n0 = blockIdx.y * 64;
  float acc[4][4] = {};
  for (int k0 = 0; k0 < K; k0 += 16) {
    // 64x16 tiles of A and W: 1024 elements each, 4 per thread
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const int idx = threadIdx.x + 256 * r;
      const int row = idx >> 4, kk = idx & 15;
      const int64_t gm = m0 + row;
      As[kk][row] = (gm < M && k0 + kk < K) ? ldf<TA>(A + gm * K + k0 + kk) : 0.f;
      const int gn = n0 + row;
      Ws[kk][row] = (gn < N && k0 + kk < K) ? ldf<TA>(W + (int64_t)gn * K + k0 + kk) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < 16; ++kk) {
      float a[4], w[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { a[i] = As[kk][ty * 4 + i]; w[i] = Ws[kk][tx * 4 + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], w[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int64_t gm = m0 + ty * 4 + i;
    if (gm >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int gn = n0 + tx * 4 + j;
      if (gn >= N) continue;
      float v = acc[i][j] + bias[gn];
      if (relu) v = fmaxf(v, 0.f);
      if constexpr (sizeof(TC) == 4) C[gm * N + gn] = v;
      else C[gm * N + gn] = __float2bfloat16_rn(v);
    }
  }
}

void launch_gemm_simt_f32(const float* A, const float* W, const float* b, float* C, int64_t M, int N,
                          int K, bool relu, cudaStream_t st) {
  dim3 grid((unsigned)((M + 63) / 64), (unsigned)((N + 63) / 64));
  gemm_simt_kernel<float, float><<<grid, 256, 0, st>>>(A, W, b, C, M, N, K, relu);
}

void launch_gemm_simt_bf16(const __nv_bfloat16* A, const __nv_bfloat16* W, const float* b, void* C,
                           bool c_is_f32, int64_t M, int N, int K, bool relu, cudaStream_t st) {
  dim3 grid((unsigned)((M + 63) / 64), (unsigned)((N + 63) / 64));
  if (c_is_f32)
    gemm_simt_kernel<__nv_bfloat16, float><<<grid, 256, 0, st>>>(A, W, b, (float*)C, M, N, K, relu);
  else
    gemm_simt_kernel<__nv_bfloat16, __nv_bfloat16><<<grid, 256, 0, st>>>(A, W, b, (__nv_bfloat16*)C, M, N, K, relu);
}

}  // namespace psim
