// rb7_stem.cu -- the RB7 model's gather + stem convolution fused on tcgen05 (sm_100a):
//
//   act0[b][q] = relu(b_s + W_s . [X_b(2q - 2) | X_b(2q - 1)])     q = 0 .. 57 (pad-row layout,
//                                                                   q = 0 and 57 kept zero)
//
// X_b(R) is input row R of sub-trace b (R6, R2): R = 0 the current instruction
// (attributes, time features 0), 1 <= R <= k the queue entry k - R (its attributes and age /
// remaining-to-complete / remaining-to-retire), otherwise zero.  The layer-wise path writes
// the whole 116 x 64 input of every sub-trace to HBM and the stem GEMM reads it back; here a
// tile of two sub-traces (116 stem rows, M = 128) builds its A operand -- row (b, q) = the two
// input rows 2q - 2, 2q - 1 side by side, K = 128, the layer-wise feature order -- straight
// into shared memory (SWIZZLE_128B, two K-atoms), one builder thread per row.
//
// Roles (288 threads, ~82 KB smem: two CTAs per SM): warps 0..3 builders (double-buffered A),
// warp 4 TMEM allocator + weight TMA + MMA issuer (8 x K16, N = 64), warps 5..8 epilogue
// (bias, ReLU, pad rows zero, bf16, 128-B rows to act0).
#include <cuda.h>

#include "internal.h"
#include "tc_common.cuh"

namespace psim {

using namespace tc;

namespace st {
constexpr int P = 58;                   // stem positions per sub-trace in the pad-row layout
constexpr int TROWS = 2 * P;            // real rows of a tile (two sub-traces)
constexpr int W_OFF = 0;                // stem weight [64][128] bf16: two K-atoms [64][64] (16 KB)
constexpr int A_OFF = 16 * 1024;        // 2 stages x two K-atoms [128][64] (32 KB each)
constexpr int BIAS_OFF = A_OFF + 2 * 32 * 1024;
constexpr int BAR_OFF = BIAS_OFF + 256;
constexpr int SMEM = BAR_OFF + 256 + 1024;
constexpr int THREADS = 288;
}  // namespace st
static_assert(st::SMEM <= 113 * 1024, "rb7_stem: two CTAs per SM");

struct StemArgs {
  GatherArgs g;              // trace rows, sub-trace state, queue (item_rows / row_off unused)
  const float* bias;         // [64]
  __nv_bfloat16* y;          // [n * 58][64]
};

__global__ void __launch_bounds__(st::THREADS, 2)
    rb7_stem_kernel(StemArgs a, const __grid_constant__ CUtensorMap tmW) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + st::BAR_OFF);
  uint64_t* wbar = bars;           // weight + bias landed
  uint64_t* afull = bars + 1;      // [2] 4 builder warps
  uint64_t* aempty = bars + 3;     // [2] commit
  uint64_t* dfull = bars + 5;      // [2] commit
  uint64_t* dempty = bars + 7;     // [2] 4 epilogue warps
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 9);
  float* sbias = reinterpret_cast<float*>(sm + st::BIAS_OFF);
  const GatherArgs& g = a.g;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint64_t n = g.n;
  const uint64_t n_tiles = (n + 1) / 2;
  if (threadIdx.x == 0) {
    mbar_init(wbar, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(afull + i, 4); mbar_init(aempty + i, 1);
      mbar_init(dfull + i, 1); mbar_init(dempty + i, 4);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 4) tmem_alloc(tmem_slot, 128);   // two accumulators of 64 columns
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp < 4) {   // ---------------- builders: thread = A row (b, q) ----------------
    const int m = warp * 32 + lane;
    const int bl = m / st::P, q = m % st::P;
    const uint64_t qn = g.qn ? g.qn : g.n;
    const bool vec = ((g.stride | reinterpret_cast<uintptr_t>(g.trace)) & 15) == 0;
    uint32_t it = 0;
    for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
      const int s = it & 1;
      const uint64_t b = 2 * tile + bl;
      bool live = m < st::TROWS && b < n;
      int64_t ws = 0, clock = 0;
      int k = 0;
      if (live) {
        ws = g.ws[b];
        live = g.step < g.e[b] - ws;                               // sub-trace still running
        k = g.count[b];
        clock = g.clock[b];
      }
      uint4 out[2][8];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int R = 2 * q - 2 + h;                               // input row (PAPER.md:93 order)
        float v[64];
#pragma unroll
        for (int c = 0; c < 64; ++c) v[c] = 0.f;
        if (live && R >= 0 && R <= k && R < kRows) {
          int64_t row;
          if (R == 0) {
            row = ws + g.step;
          } else {
            const uint4 en = g.q[(uint64_t)(k - R) * qn + b];     // newest first (R6)
            row = en.x;
            const int c = en.z & 0xFFFF, sv = en.z >> 16;
            const int age = (int)((uint32_t)clock - en.y);          // R2, clamped (R7)
            v[0] = (float)min(age, kTimeMax);
            v[1] = (float)min(max(0, c - age), kTimeMax);
            v[2] = (float)min(c + sv - age, kTimeMax);
          }
          const uint8_t* ar = g.trace + (row - g.row_lo) * g.stride;
          if (vec) {
            const uint4* a4 = reinterpret_cast<const uint4*>(ar);
            const uint4 w0 = __ldg(a4), w1 = __ldg(a4 + 1), w2 = __ldg(a4 + 2);
            const uint32_t w[12] = {w0.x, w0.y, w0.z, w0.w, w1.x, w1.y, w1.z, w1.w, w2.x, w2.y, w2.z, w2.w};
#pragma unroll
            for (int j = 0; j < kFeat - 3; ++j) v[3 + j] = (float)((w[j >> 2] >> ((j & 3) * 8)) & 0xFFu);
          } else {
#pragma unroll
            for (int j = 0; j < kFeat - 3; ++j) v[3 + j] = (float)__ldg(ar + j);
          }
        }
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          uint32_t p[4];
#pragma unroll
          for (int t = 0; t < 4; ++t) {
            __nv_bfloat162 h2 = __floats2bfloat162_rn(v[8 * c + 2 * t], v[8 * c + 2 * t + 1]);   // RNE (R16)
            p[t] = *reinterpret_cast<uint32_t*>(&h2);
          }
          out[h][c] = make_uint4(p[0], p[1], p[2], p[3]);
        }
      }
      wait_empty(aempty + s, it >> 1);
      uint8_t* A = sm + st::A_OFF + s * 32768;
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int c = 0; c < 8; ++c) st_sw128(A + h * 16384, m, c, out[h][c]);   // K-atom h = input row 2q - 2 + h
      fence_async_smem();
      __syncwarp();
      if (lane == 0) mbar_arrive(afull + s);
    }
  } else if (warp == 4) {   // ---------------- weights + MMA ----------------
    if (lane == 0) {
      mbar_expect_tx(wbar, 16384 + 256);
      tma_load_2d(sm + st::W_OFF, &tmW, wbar, 0, 0);
      tma_load_2d(sm + st::W_OFF + 8192, &tmW, wbar, 64, 0);
      bulk_g2s(sbias, a.bias, 256, wbar);
      mbar_wait(wbar, 0);
      const uint32_t sbase = smem_u32(sm);
      constexpr uint32_t idesc = idesc_bf16(128, 64);
      uint32_t it = 0;
      for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
        const int s = it & 1;
        wait_full(afull + s, it >> 1);
        wait_empty(dempty + s, it >> 1);
        fence_after();
#pragma unroll
        for (int k = 0; k < 8; ++k)
          mma_bf16(tmem + s * 64, sw128_desc(sbase + st::A_OFF + s * 32768 + (k >> 2) * 16384 + (k & 3) * 32),
                   sw128_desc(sbase + st::W_OFF + (k >> 2) * 8192 + (k & 3) * 32), idesc, k > 0);
        mma_commit(aempty + s);
        mma_commit(dfull + s);
      }
    }
  } else {   // ---------------- epilogue (warps 5..8): thread = stem row ----------------
    const int qd = warp & 3;
    const int m = qd * 32 + lane;
    const uint32_t lane_base = (uint32_t)(qd * 32) << 16;
    const int bl = m / st::P, q = m % st::P;
    mbar_wait(wbar, 0);
    uint32_t it = 0;
    for (uint64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
      const int s = it & 1;
      wait_full(dfull + s, it >> 1);
      fence_after();
      uint32_t r0[32], r1[32], pk[32];
      tmem_ld32_nowait(tmem + lane_base + s * 64, r0);
      tmem_ld32_nowait(tmem + lane_base + s * 64 + 32, r1);
      tmem_wait_ld();
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(dempty + s);
      bias_relu_pack32(r0, sbias, pk);
      bias_relu_pack32(r1, sbias + 32, pk + 16);
      const uint64_t b = 2 * tile + bl;
      if (m < st::TROWS && b < n) {
        const bool pad = q == 0 || q == st::P - 1;
        uint4* dst = reinterpret_cast<uint4*>(a.y + (b * st::P + q) * 64);
#pragma unroll
        for (int c = 0; c < 8; ++c)
          dst[c] = pad ? make_uint4(0, 0, 0, 0) : make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 4) {
    fence_after();
    tmem_dealloc(tmem, 128);
  }
}

typedef CUresult (*EncodeTiledFnSt)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

void launch_rb7_stem(const GatherArgs& g, const __nv_bfloat16* w, const float* bias, __nv_bfloat16* y, cudaStream_t stm) {
  static bool attr = false;
  static EncodeTiledFnSt fn = nullptr;
  if (!attr) {
    cudaFuncSetAttribute(rb7_stem_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, st::SMEM);
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFnSt>(p);
    attr = true;
  }
  CUtensorMap mw;
  cuuint64_t dims[2] = {128, 64};
  cuuint64_t strides[1] = {256};
  cuuint32_t box[2] = {64, 64};
  cuuint32_t es[2] = {1, 1};
  if (!fn || fn(&mw, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<__nv_bfloat16*>(w), dims, strides, box, es,
                CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
    cudaLaunchKernel((const void*)nullptr, dim3(1), dim3(1), nullptr, 0, stm);   // error for the caller
    return;
  }
  StemArgs a{g, bias, y};
  const uint64_t tiles = (g.n + 1) / 2;
  const int grid = (int)std::min<uint64_t>(tiles, 2 * (uint64_t)sm_count());
  if (tiles) rb7_stem_kernel<<<grid, st::THREADS, st::SMEM, stm>>>(a, mw);
}

}  // namespace psim
