// resblock.cu -- one fused residual block of the RB7 model (config 5; R11) on
// tcgen05 tensor cores (sm_100a):
//
//   y = relu(x + conv_b(relu(conv_a(x))))      conv_a, conv_b: Conv1d k = 3, stride 1, pad 1,
//                                              64 -> 64 channels, over the pad-row layout
//
// The layer-wise path runs the two convolutions as separate GEMMs and round-trips the inner
// activation (and the block input, for the residual) through HBM.  Here a tile of TWO
// sub-traces -- 2 x 58 pad-row positions = 116 rows of the [n * 58][64] activation, padded
// to the MMA's M = 128 -- is self-contained: each sub-trace's pad rows (positions 0 and 57,
// kept zero) are exactly the zero padding of both convolutions, so the halo never leaves the
// tile.  One TMA load brings the tile's 130 input rows (r0 - 1 .. r0 + 128; rows outside the
// tensor read as zero); conv_a's three taps are SWIZZLE_128B descriptors of that tile starting
// at rows 0 / 1 / 2 (a descriptor may start at any 128-B row: the swizzle follows the address,
// tools/gpu/exp/rowshift_probe.cu); its ReLU'd output goes into one 130-row buffer (row m + 1)
// whose row-shifted descriptors are conv_b's taps; the residual x is the input tile's row
// m + 1.  Only x is read and y written per block; ~100 KB of smem: two CTAs per SM.
//
// Roles (320 threads): warp 0 TMA producer (weights once, then the 3 tap tiles per tile,
// two stages), warp 1 TMEM allocator + MMA issuer (order a(0) a(1) b(0) a(2) b(1) ...: the
// next tile's conv_a overlaps this tile's epilogues), warps 2..5 epilogue A (thread = tile
// row = TMEM lane): relu(acc + b_a), pad rows zeroed, bf16, three shifted smem copies;
// warps 6..9 epilogue B: relu(acc + b_b + x), pad rows zeroed, bf16 -> y in HBM (A of the
// next tile overlaps B of this one).  Results are bit-identical to the layer-wise GEMMs
// (same bf16 operands, same K order in the tensor core).
#include <cuda.h>

#include "internal.h"
#include "tc_common.cuh"

namespace psim {

using namespace tc;

namespace rb {
constexpr int P = 58;                        // pad-row positions per sub-trace (56 + 2)
constexpr int TROWS = 2 * P;                 // tile rows that are real (two sub-traces)
constexpr int XROWS = 130;                   // a tile's input rows r0 - 1 .. r0 + 128 (the taps' halo)
constexpr int XSTAGE = 17 * 1024;            // one SW128 tile of 130 rows x 128 B (1024-aligned stages)
constexpr int W_OFF = 0;                     // W_a, W_b: [64 N][192 K] bf16 as 3 K-atoms of [64][64] each
constexpr int X_OFF = 48 * 1024;             // 2 stages
constexpr int ACT_OFF = X_OFF + 2 * XSTAGE;  // relu(conv_a) at rows 1..128 (row 0 and 129 zero)
constexpr int BIAS_OFF = ACT_OFF + XSTAGE;   // b_a[64], b_b[64] fp32
constexpr int BAR_OFF = BIAS_OFF + 512;
constexpr int SMEM = BAR_OFF + 256 + 1024;   // ~100 KB: two CTAs per SM
constexpr int THREADS = 320;                 // warp 0 TMA, 1 MMA, 2..5 epilogue A, 6..9 epilogue B
}  // namespace rb
static_assert(rb::SMEM <= 232448, "resblock smem over the 227 KB opt-in limit");

__global__ void __launch_bounds__(rb::THREADS, 2)
    resblock_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ CUtensorMap tmWa,
                    const __grid_constant__ CUtensorMap tmWb, const float* __restrict__ ba,
                    const float* __restrict__ bb, __nv_bfloat16* __restrict__ y, int64_t M) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + rb::BAR_OFF);
  uint64_t* wbar = bars + 0;         // weights + biases landed
  uint64_t* xfull = bars + 1;        // [2] 3 tap tiles landed (complete_tx)
  uint64_t* xempty = bars + 3;       // [2] 4 epilogue warps: residual read (stage free)
  uint64_t* dafull = bars + 5;       // [2] commit: conv_a accumulated
  uint64_t* daempty = bars + 7;      // [2] 4: conv_a accumulator drained
  uint64_t* actfull = bars + 9;      //     4: shifted copies written
  uint64_t* actempty = bars + 10;    //     commit: conv_b finished reading them
  uint64_t* dbfull = bars + 11;      // [2] commit: conv_b accumulated
  uint64_t* dbempty = bars + 13;     // [2] 4: conv_b accumulator drained
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 16);
  float* sbias = reinterpret_cast<float*>(sm + rb::BIAS_OFF);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t n_tiles = (M + rb::TROWS - 1) / rb::TROWS;
  if (threadIdx.x == 0) {
    mbar_init(wbar, 1);
    for (int i = 0; i < 2; ++i) {
      mbar_init(xfull + i, 1); mbar_init(xempty + i, 4);
      mbar_init(dafull + i, 1); mbar_init(daempty + i, 4);
      mbar_init(dbfull + i, 1); mbar_init(dbempty + i, 4);
    }
    mbar_init(actfull, 4); mbar_init(actempty, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) tmem_alloc(tmem_slot, 256);   // D_a x2 (64 cols each), D_b x2
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {   // ---------------- TMA producer ----------------
      mbar_expect_tx(wbar, 2 * 3 * 8192 + 512);
      for (int t = 0; t < 3; ++t) {
        tma_load_2d(sm + rb::W_OFF + t * 8192, &tmWa, wbar, t * 64, 0);
        tma_load_2d(sm + rb::W_OFF + 24576 + t * 8192, &tmWb, wbar, t * 64, 0);
      }
      bulk_g2s(sbias, ba, 256, wbar);
      bulk_g2s(sbias + 64, bb, 256, wbar);
      uint32_t it = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
        const int s = it & 1;
        wait_empty(xempty + s, it >> 1);
        mbar_expect_tx(xfull + s, rb::XROWS * 128);
        // rows r0 - 1 .. r0 + 128 (row -1 / rows >= M zero-filled): tap t of output row m reads
        // smem row m + t, so the three taps are row-shifted descriptors of this one tile (a
        // SWIZZLE_128B descriptor may start at any 128-B row: the swizzle follows the address)
        tma_load_2d(sm + rb::X_OFF + s * rb::XSTAGE, &tmX, xfull + s, 0, (int)(tile * rb::TROWS) - 1);
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {   // ---------------- MMA issuer ----------------
      mbar_wait(wbar, 0);
      const uint32_t sbase = smem_u32(sm);
      constexpr uint32_t idesc = idesc_bf16(128, 64);
      auto conv_a = [&](uint32_t i) {
        const int s = i & 1;
        wait_full(xfull + s, i >> 1);
        wait_empty(daempty + s, i >> 1);
        fence_after();
        for (int t = 0; t < 3; ++t)
          for (int k = 0; k < 4; ++k)
            mma_bf16(tmem + s * 64, sw128_desc(sbase + rb::X_OFF + s * rb::XSTAGE + t * 128 + 32 * k),
                     sw128_desc(sbase + rb::W_OFF + t * 8192 + 32 * k), idesc, (t | k) != 0);
        mma_commit(dafull + s);
      };
      auto conv_b = [&](uint32_t i) {
        const int s = i & 1;
        wait_full(actfull, i);
        wait_empty(dbempty + s, i >> 1);
        fence_after();
        for (int t = 0; t < 3; ++t)
          for (int k = 0; k < 4; ++k)
            mma_bf16(tmem + 128 + s * 64, sw128_desc(sbase + rb::ACT_OFF + t * 128 + 32 * k),
                     sw128_desc(sbase + rb::W_OFF + 24576 + t * 8192 + 32 * k), idesc, (t | k) != 0);
        mma_commit(actempty);
        mma_commit(dbfull + s);
      };
      uint32_t ntl = 0;
      for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x) ++ntl;
      if (ntl > 0) conv_a(0);
      for (uint32_t i = 0; i < ntl; ++i) {
        if (i + 1 < ntl) conv_a(i + 1);
        conv_b(i);
      }
    }
  } else {   // ---------------- epilogues: warps 2..5 A, warps 6..9 B; thread = tile row ----------------
    const bool roleA = warp < 6;                           // A of tile i + 1 overlaps B of tile i
    const int q = warp & 3;
    const int m = q * 32 + lane;                           // tile row = TMEM lane
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    const int pos = m % rb::P;
    mbar_wait(wbar, 0);
    uint32_t it = 0;
    for (int64_t tile = blockIdx.x; tile < n_tiles; tile += gridDim.x, ++it) {
      const int s = it & 1;
      const int64_t row = tile * rb::TROWS + m;
      const bool zero = m >= rb::TROWS || row >= M || pos == 0 || pos == rb::P - 1;   // pad / junk rows
      uint32_t pk[32];
      if (roleA) {
      // ---- A: relu(conv_a + b_a) -> bf16 -> conv_b's three row-shifted A operands
      wait_full(dafull + s, it >> 1);
      fence_after();
      {
        uint32_t r0[32], r1[32];
        tmem_ld32_nowait(tmem + lane_base + s * 64, r0);
        tmem_ld32_nowait(tmem + lane_base + s * 64 + 32, r1);
        tmem_wait_ld();
        bias_relu_pack32(r0, sbias, pk);
        bias_relu_pack32(r1, sbias + 32, pk + 16);
      }
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(daempty + s);
      if (zero)
        for (int c = 0; c < 32; ++c) pk[c] = 0u;
      wait_empty(actempty, it);                            // conv_b of the previous tile done with them
      uint8_t* act = sm + rb::ACT_OFF;
      // activation row m at buffer row m + 1: conv_b's tap t of output row m reads buffer row
      // m + t = activation row m + t - 1; row 0 (activation row -1 = the previous tile's last pad
      // row) is zero, row 129 feeds only junk rows
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        st_sw128(act, m + 1, c, make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]));
        if (m == 0) st_sw128(act, 0, c, make_uint4(0, 0, 0, 0));
        if (m == 127) st_sw128(act, 129, c, make_uint4(0, 0, 0, 0));
      }
      fence_async_smem();                                  // visible to the tensor core
      __syncwarp();
      if (lane == 0) mbar_arrive(actfull);
      continue;
      }
      // ---- B: relu(conv_b + b_b + x) -> y
      wait_full(dbfull + s, it >> 1);
      fence_after();
      const uint8_t* xt = sm + rb::X_OFF + s * rb::XSTAGE;   // residual x row m = tile row m + 1
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {                      // channels 32 hf .. 32 hf + 31 (register budget)
        uint32_t r0[32];
        tmem_ld32_nowait(tmem + lane_base + 128 + s * 64 + 32 * hf, r0);
        tmem_wait_ld();
        uint32_t xv[16];
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          const int cc = 4 * hf + c;
          const uint4 u = *reinterpret_cast<const uint4*>(xt + (m + 1) * 128 + ((cc ^ ((m + 1) & 7)) << 4));
          xv[4 * c] = u.x; xv[4 * c + 1] = u.y; xv[4 * c + 2] = u.z; xv[4 * c + 3] = u.w;
        }
#pragma unroll
        for (int c = 0; c < 16; ++c) {                      // channels 32 hf + 2c, + 1
          const float x0 = __uint_as_float(xv[c] << 16), x1 = __uint_as_float(xv[c] & 0xFFFF0000u);
          pk[16 * hf + c] = pack_bf16_relu(__uint_as_float(r0[2 * c]) + sbias[64 + 32 * hf + 2 * c] + x0,
                                           __uint_as_float(r0[2 * c + 1]) + sbias[65 + 32 * hf + 2 * c] + x1);
        }
      }
      fence_before();
      __syncwarp();
      if (lane == 0) { mbar_arrive(dbempty + s); mbar_arrive(xempty + s); }   // accumulator drained, X stage free
      if (m < rb::TROWS && row < M) {
        uint4* dst = reinterpret_cast<uint4*>(y + row * 64);
#pragma unroll
        for (int c = 0; c < 8; ++c)
          dst[c] = zero ? make_uint4(0, 0, 0, 0) : make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    tmem_dealloc(tmem, 256);
  }
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFnRb)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFnRb encode_fn_rb() {
  static EncodeTiledFnRb fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFnRb>(p);
  }
  return fn;
}
static bool map_rb(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  EncodeTiledFnRb fn = encode_fn_rb();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {64, box_rows};
  cuuint32_t es[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

void launch_resblock(const __nv_bfloat16* x, const __nv_bfloat16* wa, const float* ba, const __nv_bfloat16* wb,
                     const float* bb, __nv_bfloat16* y, int64_t M, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(resblock_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, rb::SMEM);
    attr = true;
  }
  CUtensorMap mx, mwa, mwb;
  if (M % rb::P != 0 || !map_rb(&mx, x, (uint64_t)M, 64, rb::XROWS) || !map_rb(&mwa, wa, 64, 192, 64) ||
      !map_rb(&mwb, wb, 64, 192, 64)) {
    cudaLaunchKernel((const void*)nullptr, dim3(1), dim3(1), nullptr, 0, st);   // error for the caller
    return;
  }
  const int64_t tiles = (M + rb::TROWS - 1) / rb::TROWS;
  const int grid = (int)std::min<int64_t>(tiles, 2 * (int64_t)sm_count());   // two CTAs per SM
  resblock_kernel<<<grid, rb::THREADS, rb::SMEM, st>>>(mx, mwa, mwb, ba, bb, y, M);
}

}  // namespace psim
