// gemm_sp.cu -- 2:4 structured-sparse tcgen05 GEMM for the lowered CNN layers (sm_100a),
// the paper's "2:4 structured sparsity" inference optimisation (PAPER.md:157 [IV-B],
// :261 [VI-B, Fig. 13]) on the layer-wise path.
//
//   C[M][N] = act(X[M][K] . W[N][K]^T + b[N])     W 2:4-sparse along K (magnitude-pruned
//                                                  weights, R22), X bf16 dense
//
// tcgen05.mma.sp takes the SPARSE operand as A, so the layer is computed transposed:
// D^T[N out][M rows] = Wc (A: compressed [N][K/2], M-dim = output channels, 128 per MMA)
// x X^T (B: the activation tile, K-major [128 rows][K], exactly the dense kernel's A tile).
// Per 32 logical K the MMA reads 16 stored weights per row and one 32-bit TMEM metadata
// word per lane: for lane L = 16 b + i of the 128-row weight tile, i < 8: nibbles 0-3 =
// row L groups 0-3, nibbles 4-7 = row L + 8 groups 0-3; i >= 8: nibbles 0-3 = row L - 8
// groups 4-7, nibbles 4-7 = row L groups 4-7 (a group = 4 logical K, nibble = idx0 |
// idx1 << 2 of its two kept elements, stored in that order).  Metadata columns are
// addressed in even pairs with sparse_id2 selecting the odd column.  (Layout established
// on the B200 by tools/gpu/exp/sparse_probe.cu, profiles/r02_sparse_probe.md.)
//
// Kernel shape (as gemm_tc.cu): persistent, one CTA per SM, 192 threads: warp 0 TMA
// producer (per k-block of 128 logical K: Wc tile [MH*128][64 stored] + X tile 2 x
// [128][64]), warp 1 TMEM allocator + MMA issuer (MH x 4 sparse MMAs per k-block, M = 128,
// N = 128 rows, K = 32), warps 2..5 epilogue (thread = output channel: D^T lanes; bias,
// ReLU, stores of 32 consecutive channels of a row per warp instruction).  The metadata of
// all k-blocks stays resident in TMEM columns 256.. (loaded once per launch).
#include <cuda.h>

#include "internal.h"
#include "tc_common.cuh"

namespace psim {

using namespace tc;

namespace sp {
constexpr int BN = 128;              // activation rows per tile (the MMA's N)
constexpr int KB = 128;              // logical K per k-block (64 stored weights per row)
constexpr int META_COL = 256;        // first TMEM column of the metadata
}  // namespace sp

template <int MH>   // weight tiles of 128 output channels (1: N <= 128, 2: N <= 256)
struct SpCfg {
  static constexpr int A_BYTES = MH * 128 * 128;   // compressed weights [MH*128][64] bf16
  static constexpr int B_BYTES = 2 * sp::BN * 128; // activations [128][128 logical K] bf16, two SW128 atoms
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES = (192 * 1024) / STAGE;
  static constexpr int SMEM = STAGES * STAGE + 1024 + 256 + 4 * 32 * 33 * 4;   // + epilogue transpose stages
  static constexpr int ACC_COLS = MH * sp::BN;
  static constexpr int NACC = MH == 1 ? 2 : 1;     // double-buffered accumulators when they fit next to the metadata
};

__device__ __forceinline__ void mma_bf16_sp(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                            uint32_t tmem_e, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%5], %3, p;\n}\n" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(acc), "r"(tmem_e));
}
__device__ __forceinline__ void tmem_st1(uint32_t taddr, uint32_t v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(v) : "memory");
}

template <int MH>
__global__ void __launch_bounds__(192, 1)
    gemm_sp_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmW,
                   const uint32_t* __restrict__ meta, int meta_cols, const float* __restrict__ bias,
                   void* __restrict__ C, int64_t M, int K, int n_out, int relu, int c_f32) {
  using Cfg = SpCfg<MH>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (tc::smem_u32(smem_raw) & 1023u)) & 1023u);   // 1024-B aligned; stays in the shared window (LDS/STS, not generic LD/ST)
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + Cfg::STAGES * Cfg::STAGE);
  uint64_t* empty = full + Cfg::STAGES;
  uint64_t* tfull = empty + Cfg::STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t n_tiles = (M + sp::BN - 1) / sp::BN;
  const int nk = K / sp::KB;
  const int steps = K / 32;   // metadata columns per weight tile

  if (threadIdx.x == 0) {
    for (int s = 0; s < Cfg::STAGES; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(tfull + a, 1); mbar_init(tempty + a, 4); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) tmem_alloc(tmem_slot, 512);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp >= 2) {   // metadata of every (weight tile, K step) into TMEM, lane = weight row
    const int q = warp & 3;
    for (int c = 0; c < meta_cols; ++c)
      tmem_st1(tmem + ((uint32_t)(32 * q) << 16) + sp::META_COL + c, __ldg(meta + (size_t)c * 128 + 32 * q + lane));
    tmem_wait_st();
  }
  fence_before();
  __syncthreads();
  fence_after();

  if (warp == 0) {
    if (lane == 0) {   // ---------------- TMA producer ----------------
      int stage = 0;
      uint32_t phase = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) {
        const int r0 = (int)(tile * sp::BN);
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(empty + stage, phase ^ 1);
          uint8_t* sa = smem + stage * Cfg::STAGE;
          uint8_t* sb = sa + Cfg::A_BYTES;
          mbar_expect_tx(full + stage, Cfg::STAGE);
          tma_load_2d(sa, &tmW, full + stage, kb * 64, 0);                  // stored columns kb*64 .. +63
          tma_load_2d(sb, &tmX, full + stage, kb * sp::KB, r0);             // logical K kb*128 .. +63
          tma_load_2d(sb + sp::BN * 128, &tmX, full + stage, kb * sp::KB + 64, r0);
          if (++stage == Cfg::STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {   // ---------------- MMA issuer ----------------
      const uint32_t idesc0 = idesc_bf16(128, sp::BN) | (1u << 2);   // sparse A
      int stage = 0;
      uint32_t phase = 0;
      int it = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
        const int acc = it % Cfg::NACC;
        const uint32_t use = (uint32_t)(it / Cfg::NACC);
        wait_empty(tempty + acc, use);
        fence_after();
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(full + stage, phase);
          fence_after();
          const uint32_t sa = smem_u32(smem + stage * Cfg::STAGE);
          const uint32_t sb = sa + Cfg::A_BYTES;
#pragma unroll
          for (int h = 0; h < MH; ++h)
#pragma unroll
            for (int s = 0; s < 4; ++s) {
              const int idx = h * steps + kb * 4 + s;                      // metadata column
              mma_bf16_sp(tmem + acc * Cfg::ACC_COLS + h * sp::BN,
                          sw128_desc(sa + h * 128 * 128 + 32 * s),         // 16 stored weights per K step
                          sw128_desc(sb + (s >> 1) * sp::BN * 128 + (s & 1) * 64),   // 32 logical K
                          idesc0 | (uint32_t)(idx & 1), tmem + sp::META_COL + (idx & ~1), (kb | s) != 0);
            }
          mma_commit(empty + stage);
          if (++stage == Cfg::STAGES) { stage = 0; phase ^= 1; }
        }
        mma_commit(tfull + acc);
      }
    }
  } else {   // ---------------- epilogue (warps 2..5): thread = output channel ----------------
    // D^T lane = output channel, column = row.  Each 32 x 32 block (32 channels of this warp's
    // quadrant x 32 rows) goes through a per-warp smem stage (fp32, padded rows) so that lane j
    // then writes row j's 32 channels as contiguous 16-B stores (64 B bf16 / 128 B fp32 per lane).
    const int q = warp & 3;
    float* stg = reinterpret_cast<float*>(smem + Cfg::STAGES * Cfg::STAGE + 256) + (warp - 2) * 32 * 33;
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
      const int acc = it % Cfg::NACC;
      wait_full(tfull + acc, (uint32_t)(it / Cfg::NACC));
      fence_after();
#pragma unroll 1
      for (int h = 0; h < MH; ++h) {
        const int c0 = h * 128 + 32 * q;                         // first channel of this warp's block
        if (c0 >= n_out) continue;                               // (warp-uniform) padding channels
        const int c = c0 + lane;
        const float b = c < n_out ? __ldg(bias + c) : 0.f;
#pragma unroll 1
        for (int r0 = 0; r0 < sp::BN; r0 += 32) {
          uint32_t r[32];
          tmem_ld32_nowait(tmem + ((uint32_t)(32 * q) << 16) + acc * Cfg::ACC_COLS + h * sp::BN + r0, r);
          tmem_wait_ld();
#pragma unroll
          for (int j = 0; j < 32; ++j) {                         // stage[row j][channel lane]
            float v = __uint_as_float(r[j]) + b;
            stg[j * 33 + lane] = relu ? fmaxf(v, 0.f) : v;
          }
          __syncwarp();
          const int64_t row = tile * sp::BN + r0 + lane;         // lane = row now
          if (row < M) {
            const float* src = stg + lane * 33;
            if (c_f32) {
              float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(C) + row * n_out + c0);
#pragma unroll
              for (int u = 0; u < 8; ++u) dst[u] = make_float4(src[4 * u], src[4 * u + 1], src[4 * u + 2], src[4 * u + 3]);
            } else {
              uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(C) + row * n_out + c0);
#pragma unroll
              for (int u = 0; u < 4; ++u) {
                uint32_t p4[4];
#pragma unroll
                for (int t = 0; t < 4; ++t) {
                  __nv_bfloat162 h2 = __floats2bfloat162_rn(src[8 * u + 2 * t], src[8 * u + 2 * t + 1]);
                  p4[t] = *reinterpret_cast<uint32_t*>(&h2);
                }
                dst[u] = make_uint4(p4[0], p4[1], p4[2], p4[3]);
              }
            }
          }
          __syncwarp();                                          // stage reused by the next block
        }
      }
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(tempty + acc);
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem, 512);
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFnSp)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFnSp encode_fn_sp() {
  static EncodeTiledFnSp fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFnSp>(p);
  }
  return fn;
}
// bf16 [rows][cols] row-major, box [box_rows][64 cols], SWIZZLE_128B (rows past the end read zero)
static bool map_sp(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  EncodeTiledFnSp fn = encode_fn_sp();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {64, box_rows};
  cuuint32_t es[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

int sparse24_compress(const uint16_t* W, int N, int K, std::vector<uint16_t>* wc, std::vector<uint32_t>* meta,
                      int* mh) {
  if (K % sp::KB != 0 || N < 1 || N > 256) return -1;
  const int MH = N <= 128 ? 1 : 2;
  const int Np = MH * 128, steps = K / 32;
  wc->assign((size_t)Np * (K / 2), 0);
  std::vector<uint8_t> nib((size_t)Np * (K / 4), 0x4);   // (0, 1) for all-zero groups and padding rows
  for (int r = 0; r < N; ++r)
    for (int g = 0; g < K / 4; ++g) {
      int idx[2], n = 0;
      for (int t = 0; t < 4; ++t)
        if ((W[(size_t)r * K + 4 * g + t] & 0x7FFF) != 0) {   // nonzero (either sign of zero counts as zero)
          if (n == 2) return -2;                               // more than 2 of 4: not 2:4 sparse
          idx[n++] = t;
        }
      for (int t = 0; n < 2 && t < 4; ++t)                     // fewer than 2: fill with zero positions
        if (!(n == 1 && idx[0] == t)) idx[n++] = t;
      if (idx[0] > idx[1]) std::swap(idx[0], idx[1]);
      (*wc)[(size_t)r * (K / 2) + 2 * g] = W[(size_t)r * K + 4 * g + idx[0]];
      (*wc)[(size_t)r * (K / 2) + 2 * g + 1] = W[(size_t)r * K + 4 * g + idx[1]];
      nib[(size_t)r * (K / 4) + g] = (uint8_t)(idx[0] | (idx[1] << 2));
    }
  // TMEM words: column (h * steps + s), lane L (see the header comment)
  meta->assign((size_t)MH * steps * 128, 0);
  auto nibs4 = [&](int row, int s, int g0) -> uint32_t {
    uint32_t v = 0;
    for (int t = 0; t < 4; ++t) v |= (uint32_t)nib[(size_t)row * (K / 4) + s * 8 + g0 + t] << (4 * t);
    return v;
  };
  for (int h = 0; h < MH; ++h)
    for (int s = 0; s < steps; ++s)
      for (int L = 0; L < 128; ++L) {
        const int b = L / 16, i = L % 16, base = h * 128 + 16 * b;
        const uint32_t w = i < 8 ? (nibs4(base + i, s, 0) | (nibs4(base + i + 8, s, 0) << 16))
                                 : (nibs4(base + i - 8, s, 4) | (nibs4(base + i, s, 4) << 16));
        (*meta)[((size_t)h * steps + s) * 128 + L] = w;
      }
  *mh = MH;
  return 0;
}

static int num_sms_sp() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <int MH>
static void launch_mh(const CUtensorMap& mx, const CUtensorMap& mw, const uint32_t* meta, int meta_cols,
                      const float* b, void* C, int64_t M, int K, int n_out, bool relu, bool c_f32, cudaStream_t st) {
  using Cfg = SpCfg<MH>;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_sp_kernel<MH>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM);
    attr = true;
  }
  const int64_t tiles = (M + sp::BN - 1) / sp::BN;
  const int grid = (int)std::min<int64_t>(tiles, num_sms_sp());
  gemm_sp_kernel<MH><<<grid, 192, Cfg::SMEM, st>>>(mx, mw, meta, meta_cols, b, C, M, K, n_out, relu ? 1 : 0,
                                                   c_f32 ? 1 : 0);
}

void launch_gemm_sp(const __nv_bfloat16* X, const __nv_bfloat16* Wc, const uint32_t* meta, int mh, const float* b,
                    void* C, bool c_is_f32, int64_t M, int N, int K, bool relu, cudaStream_t st) {
  CUtensorMap mx, mw;
  if (K % sp::KB != 0 || (mh != 1 && mh != 2) || !map_sp(&mx, X, (uint64_t)M, (uint64_t)K, sp::BN) ||
      !map_sp(&mw, Wc, (uint64_t)mh * 128, (uint64_t)K / 2, (uint32_t)mh * 128)) {
    cudaLaunchKernel((const void*)nullptr, dim3(1), dim3(1), nullptr, 0, st);   // error for the caller
    return;
  }
  const int meta_cols = mh * (K / 32);
  if (mh == 1) launch_mh<1>(mx, mw, meta, meta_cols, b, C, M, K, N, relu, c_is_f32, st);
  else launch_mh<2>(mx, mw, meta, meta_cols, b, C, M, K, N, relu, c_is_f32, st);
}

}  // namespace psim
