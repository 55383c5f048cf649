// gemm_tc.cu -- tcgen05 / TMEM / TMA GEMM for the lowered CNN layers (sm_100a).
//
//   C[M][N] = act(A[M][K] . W[N][K]^T + b[N])     A, W bf16 K-major; fp32 accumulate
//
// The convolutions of the SimNet-style CNN (k = s = 2) are plain GEMMs on the
// row-pair reshape of the previous activation, and FC1 is a GEMM on the
// position-major flattening, so every layer but the
// 3-output head runs here ("efficient use of Tensor Core").
//
// Kernel shape: persistent, one CTA per SM, 192 threads = 6 warps:
//   warp 0      TMA producer: A tile 128x64 and W tile BNx64 per k-block into an
//               S-stage smem ring (SWIZZLE_128B, mbarrier complete_tx)
//   warp 1      TMEM allocator + single-thread tcgen05.mma issuer
//               (M=128, N=BN, K=16 per instruction), commits to mbarriers
//   warps 2..5  epilogue: tcgen05.ld 32x32b -> +bias (+ residual), ReLU -> bf16/fp32 -> global
// Stride-1 convolutions (RB7's k = 3, pad 1 residual convs) run on the same
// kernel with no im2col: K-block kb of tap t = kb / (Cin/64) loads the A tile
// at row offset t - 1 (TMA zero-fills rows -1 and M), and the activations are
// laid out with one zero pad row before and after each sub-trace's positions
// (period P = positions + 2), which the epilogue keeps zero.
// Two TMEM accumulators (2*BN columns) let the epilogue of tile i overlap the
// MMAs of tile i+1.
#include <cuda.h>

#include "internal.h"
#include "tc_common.cuh"

namespace psim {

// PTX helpers (mbarrier, TMA, tcgen05 descriptors / MMA / TMEM): tc_common.cuh

constexpr int kBM = 128, kBK = 64;

template <int BN>
struct TcCfg {
  static constexpr int A_BYTES = kBM * kBK * 2;
  static constexpr int B_BYTES = BN * kBK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES = (196 * 1024) / STAGE;
  static constexpr int SMEM = STAGES * STAGE + 1024 /*align*/ + 256 /*barriers*/;
  static constexpr int TMEM_COLS = 2 * BN;   // two accumulators; power of 2 >= 32
};

template <int BN>
__global__ void __launch_bounds__(192, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const float* __restrict__ bias, void* __restrict__ C, int64_t M, int K, int relu, int c_f32,
                   int taps, const __nv_bfloat16* __restrict__ resid, int pad_period) {
  using Cfg = TcCfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);   // 1024-B aligned; stays in the shared window (LDS/STS, not generic LD/ST)
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Cfg::STAGES * Cfg::STAGE);
  uint64_t* empty = full + Cfg::STAGES;
  uint64_t* tfull = empty + Cfg::STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t n_tiles = (M + kBM - 1) / kBM;
  const int nk = K / kBK;

  if (threadIdx.x == 0) {
    for (int s = 0; s < Cfg::STAGES; ++s) { tc::mbar_init(full + s, 1); tc::mbar_init(empty + s, 1); }
    for (int a = 0; a < 2; ++a) { tc::mbar_init(tfull + a, 1); tc::mbar_init(tempty + a, 4); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmB)) : "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(tc::smem_u32(tmem_slot)),
                 "r"(Cfg::TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc::fence_before();
  __syncthreads();
  tc::fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {   // ---------------- TMA producer ----------------
      int stage = 0;
      uint32_t phase = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const int m0 = (int)(tile * kBM);
        const int kpt = nk / taps;          // K-blocks per tap
        for (int kb = 0; kb < nk; ++kb) {
          tc::mbar_wait(empty + stage, phase ^ 1);
          uint8_t* sa = smem + stage * Cfg::STAGE;
          uint8_t* sb = sa + Cfg::A_BYTES;
          tc::mbar_expect_tx(full + stage, Cfg::STAGE);
          const int tap = kb / kpt;
          // taps == 1: plain GEMM; taps == 3: rows shifted by tap - 1 (zero-filled outside [0, M))
          tc::tma_load_2d(sa, &tmA, full + stage, (kb - tap * kpt) * kBK, m0 + (taps > 1 ? tap - 1 : 0));
          tc::tma_load_2d(sb, &tmB, full + stage, kb * kBK, 0);
          if (++stage == Cfg::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {   // ---------------- MMA issuer ----------------
      constexpr uint32_t idesc = tc::idesc_bf16(kBM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
        const int acc = it & 1;
        const uint32_t use = (uint32_t)(it >> 1);
        tc::mbar_wait(tempty + acc, (use & 1) ^ 1);
        tc::fence_after();
        const uint32_t tmem_d = tmem_base + acc * BN;
        for (int kb = 0; kb < nk; ++kb) {
          tc::mbar_wait(full + stage, phase);
          tc::fence_after();
          const uint32_t sa = tc::smem_u32(smem + stage * Cfg::STAGE);
          const uint32_t sb = sa + Cfg::A_BYTES;
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k)
            tc::mma_bf16(tmem_d, tc::sw128_desc(sa + 32 * k), tc::sw128_desc(sb + 32 * k), idesc, (kb | k) != 0);
          tc::mma_commit(empty + stage);   // frees the smem stage when these MMAs finish
          if (++stage == Cfg::STAGES) { stage = 0; phase ^= 1; }
        }
        tc::mma_commit(tfull + acc);       // accumulator ready for the epilogue
      }
    }
  } else {   // ---------------- epilogue (warps 2..5) ----------------
    const int quad = warp & 3;             // TMEM lanes 32*quad .. 32*quad+31
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
      const int acc = it & 1;
      const uint32_t use = (uint32_t)(it >> 1);
      tc::mbar_wait(tfull + acc, use & 1);
      tc::fence_after();
      const int64_t row = tile * kBM + quad * 32 + lane;
      bool pad_row = false;
      if (pad_period) {
        const int pr = (int)(row % pad_period);
        pad_row = pr == 0 || pr == pad_period - 1;
      }
#pragma unroll 1
      for (int c0 = 0; c0 < BN; c0 += 32) {
        uint32_t r[32];
        tc::tmem_ld32(tmem_base + ((uint32_t)(quad * 32) << 16) + acc * BN + c0, r);
        if (row < M) {
          float v[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = __uint_as_float(r[j]) + __ldg(bias + c0 + j);
          if (resid) {   // residual block: y = relu(x + conv_b(...)) (R11)
            const uint4* rs = reinterpret_cast<const uint4*>(resid + row * BN + c0);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const uint4 u = __ldg(rs + j);
              const uint32_t w4[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                v[8 * j + 2 * q] += __uint_as_float(w4[q] << 16);
                v[8 * j + 2 * q + 1] += __uint_as_float(w4[q] & 0xFFFF0000u);
              }
            }
          }
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            if (relu) v[j] = fmaxf(v[j], 0.f);
            if (pad_row) v[j] = 0.f;
          }
          if (c_f32) {
            float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(C) + row * BN + c0);
#pragma unroll
            for (int j = 0; j < 8; ++j) dst[j] = make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
          } else {
            uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(C) + row * BN + c0);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              uint32_t p[4];
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                __nv_bfloat162 h2 = __floats2bfloat162_rn(v[8 * j + 2 * q], v[8 * j + 2 * q + 1]);
                p[q] = *reinterpret_cast<uint32_t*>(&h2);
              }
              dst[j] = make_uint4(p[0], p[1], p[2], p[3]);
            }
          }
        }
      }
      tc::fence_before();
      __syncwarp();
      if (lane == 0) tc::mbar_arrive(tempty + acc);
    }
  }
  tc::fence_before();
  __syncthreads();
  if (warp == 1) {
    tc::fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(Cfg::TMEM_COLS));
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  }
  return fn;
}

// 2-D bf16 tensor [rows][cols] row-major, box [box_rows][64 cols], SWIZZLE_128B
static bool make_map(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  EncodeTiledFn fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {(cuuint32_t)kBK, box_rows};
  cuuint32_t es[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool gemm_tc_supported(int N, int K) { return (N == 64 || N == 128 || N == 256) && K % kBK == 0 && K > 0; }

void* pretile_weight_tc(const __nv_bfloat16* W, int, int, cudaStream_t) {
  // TMA reads the [N][K] K-major weight in place; no repacking is needed.
  return const_cast<__nv_bfloat16*>(W);
}

static int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <int BN>
static void launch_bn(const CUtensorMap& ma, const CUtensorMap& mb, const float* b, void* C, int64_t M, int K,
                      bool relu, bool c_f32, int taps, const __nv_bfloat16* resid, int pad_period, cudaStream_t st) {
  using Cfg = TcCfg<BN>;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_tc_kernel<BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    attr = true;
  }
  const int64_t tiles = (M + kBM - 1) / kBM;
  const int grid = (int)std::min<int64_t>(tiles, num_sms());
  gemm_tc_kernel<BN><<<grid, 192, Cfg::SMEM, st>>>(ma, mb, b, C, M, K, relu ? 1 : 0, c_f32 ? 1 : 0, taps, resid,
                                                   pad_period);
}

void launch_gemm_tc(const __nv_bfloat16* A, const void* Wtc, const float* b, void* C, bool c_is_f32, int64_t M,
                    int N, int K, bool relu, cudaStream_t st, int taps, const __nv_bfloat16* resid, int pad_period) {
  CUtensorMap ma, mb;
  if (taps < 1 || K % (taps * kBK) != 0 || (resid && (c_is_f32 || N != 64 && N != 128 && N != 256)) ||
      !make_map(&ma, A, (uint64_t)M, (uint64_t)(K / taps), kBM) || !make_map(&mb, Wtc, (uint64_t)N, (uint64_t)K, N)) {
    // leave an error for the caller's cudaGetLastError check
    cudaLaunchKernel((const void*)nullptr, dim3(1), dim3(1), nullptr, 0, st);
    return;
  }
  if (N == 64) launch_bn<64>(ma, mb, b, C, M, K, relu, c_is_f32, taps, resid, pad_period, st);
  else if (N == 128) launch_bn<128>(ma, mb, b, C, M, K, relu, c_is_f32, taps, resid, pad_period, st);
  else launch_bn<256>(ma, mb, b, C, M, K, relu, c_is_f32, taps, resid, pad_period, st);
}

}  // namespace psim
