// fused_c3.cu -- the padding-aware fused step of the C3 ("3C+2F") model on
// tcgen05 tensor cores (sm_100a).  Two kernels per lockstep step:
//
//  conv_stack_kernel   gather + conv1 + conv2 + conv3 for every VALID block
//                      (sub-trace b, conv3 position p < P_b), never materialising
//                      the 112x64 input in HBM; output a4[b][p][128] bf16.
//  fc1_head_kernel     fc1 over the P_tile computed positions (+ the constant
//                      table T[P_b] for the all-padding positions), ReLU, fc2,
//                      rounding and the warp-level queue update; emits the
//                      block list of the next step.
//
// Padding awareness generalises the paper's custom first convolution, which
// "dynamically adjusts the dimensions of the convolution channel to perform
// computation only over the non-paddings": with k = s = 2
// convolutions a conv3 position p sees input rows 8p..8p+7 only, so every
// position with 8p > k (all padding: PAPER.md:267, > 68% of rows) has the
// same conv3 output c3 = conv3(conv2(conv1(0))), and its fc1 contribution is
// folded into T[P] = b_fc1 + sum_{p >= P} Wfc1[:, p] c3 (R18).
// P_b = ceil((k_b + 1) / 8).  Exact in real arithmetic; the oracle stays dense.
//
// conv_stack_kernel roles (640 threads, five warpgroups, registers rebalanced with
// setmaxnreg): warps 0..3 = EG-A (conv1 epilogue: TMEM -> bias, ReLU, bf16 -> A2 back
// into TMEM, and the epilogue of conv2 position 0), warps 4..7 = EG-B (conv2
// position 1 -> A3 in TMEM, conv3 epilogue -> a4 rows, staged in smem and stored
// coalesced), warp 8 = TMEM allocator and MMA issuer (the whole warp runs the loop,
// one elected lane issues; it also streams W3), warps 9..11 idle, warps 12..19 = row
// builders + TMA row issuers (each lane builds one input row per item: block entry
// {id, k, ws, Clock} -> queue entry -> trace row index + time features, software-
// pipelined in registers; trace rows by tile::gather4 straight into the SWIZZLE_128B X
// tile, evict_first).
// W1/W2 stay resident in smem (48 KB); W3 (64 KB) is streamed one K-half (32 KB) at
// a time from L2, alternating with the conv3 MMAs.  Per 128-block tile the MMA
// order is
//   c1(0) c1(1) [c3(prev,1)] c2(0,0) c2(0,1) c1(2) c1(3) c3(0) c2(1,0) c2(1,1)
// with K-split accumulation; the conv2 / conv3 A operands live in TMEM.
#include "internal.h"
#include "sim_common.cuh"
#include "tc_common.cuh"

namespace psim {

using namespace tc;

// ------------------------------------------------------------ smem layout
namespace cs {
constexpr int TILE = 128;
constexpr int W1_OFF = 0;                    // 2 atoms [64][64]   8 KB each
constexpr int W2_OFF = W1_OFF + 16 * 1024;   // 2 atoms [128][64] 16 KB each
constexpr int W3_OFF = W2_OFF + 32 * 1024;   // 2 atoms [128][64]: ONE K-half of W3, streamed by TMA
                                             // (halves alternate with the conv3 MMAs, from L2)
constexpr int NX = 2;                        // X slots: gathered items in flight
constexpr int X_OFF = W3_OFF + 32 * 1024;    // NX slots x 2 atoms [128][64]
constexpr int STG_OFF = X_OFF + NX * 32 * 1024;   // conv3 epilogue staging: 2 groups x 4 warps x [32 rows][128 B]
                                                  // (EG-B: channels 0..63 of a4 rows, EG-A: 64..127)
constexpr int BE_OFF = STG_OFF + 32 * 1024;  // uint4 [3 tiles][256 issuer lanes]: block entries staged by cp.async
constexpr int ER = 8, ED = 4;                // queue-entry ring: items staged ED ahead in ER slots
constexpr int ER_OFF = BE_OFF + 12 * 1024;   // uint4 [ER items][256 issuer lanes]: queue entries staged by cp.async
constexpr int BAR_OFF = ER_OFF + ER * 4096;  // mbarriers
constexpr int BIAS_OFF = BAR_OFF + 512;      // b1[64] b2[128] b3[128] fp32
constexpr int SMEM = BIAS_OFF + 1280 + 1024; // + alignment slack (<= 227 KB)
static_assert(SMEM <= 232448, "conv_stack smem over the 227 KB opt-in limit");
// C1 x2 (64 fp32 each), C2 x2 (128 fp32 each), C3 (128 fp32).  The conv2 / conv3 A operands
// (bf16 activations of conv1 / conv2) are written back by the epilogues into the first
// 32 / 64 columns of the slot they were read from (packed bf16x2) and read by the MMA
// from TMEM: no smem traffic for A2 / A3.
constexpr int TMEM_C1 = 0, TMEM_C2 = 128, TMEM_C3 = 384, TMEM_COLS = 512;
// warps 0-3 EG-A (conv1 epi + conv2 position 0 epi), 4-7 EG-B (conv2 position 1 + conv3
// epi + a4 stores), 8 MMA + W3 stream, 9-11 idle, 12-19 row builders + TMA row issuers (8 warps x
// 8 lanes: the gather4 issue rate scales with issuing warps).  Five warpgroups; registers
// rebalanced with setmaxnreg (each SM sub-partition holds one warp of every warpgroup):
// EG-A 136 + EG-B 136 + MMA 96 + issuers 56 + 56 = 480 (= the launch allocation, 96 per thread:
// setmaxnreg only moves registers between the warps of a CTA; a larger sum deadlocks the inc).
constexpr int THREADS = 640;
constexpr int MMA_WARP = 8, GATHER_WARP0 = 12, NISSUE = 8;
constexpr int REG_EPI = 136, REG_MMA = 96, REG_ISSUE = 56;   // 136 + 136 + 96 + 56 + 56 = 480 = 640 x 96 / 128
static_assert(2 * REG_EPI + REG_MMA + 2 * REG_ISSUE <= THREADS * 96 / 128, "setmaxnreg over the CTA's allocation");

}  // namespace cs

// Epilogue split (experiment): EG-B's conv3 epilogue (TMEM -> bias, ReLU, bf16 -> staged, coalesced a4
// stores) takes about as long as a whole tile, so the conv2 position-1 epilogue runs on EG-A
// (after its conv1 epilogues of the tile) instead of EG-B
constexpr bool kEgaConv2Pos1 = false;   // measured neutral (A/B 554.5 vs 555.2 MIPS, G=8 238.2 vs 239.1)

struct ConvArgs {
  const uint4* blocks;       // block entries {b << 4 | p, k, ws lo, Clock lo} of this step
  const uint32_t* nblocks;   // count of this step's list
  uint32_t* next_count;      // the other step parity's counter, reset here
  const __nv_bfloat16* trace16;   // [rows + 1][48] bf16 operand rows (attributes at cols 0..46), row `rows` zero
  uint32_t zero_row;         // gather row index of the padding rows of the input (kPadRow: out of bounds, TMA zero fill)
  int64_t row_lo;
  const int64_t* ws;
  const int64_t* clock;
  const int32_t* count;
  const uint4* q;
  int64_t step;
  uint64_t qn;               // sub-traces (entry stride of the entry-major queue)
  int rows_keep;             // gathered rows evict_last (small slices: the live context window fits L2)
  const __nv_bfloat16* w1;   // [64][128]
  const __nv_bfloat16* w2;   // [128][128]
  const __nv_bfloat16* w3;   // [128][256]
  const float* b1;
  const float* b2;
  const float* b3;
  __nv_bfloat16* a4;         // [n][14][128]
  long long* dbg;            // optional stage timestamps of CTA 0 (PSIM_DEBUG_TIMING), else nullptr
};

// conv3 epilogue, one channel half (64 channels = 128 B of an a4 row) of a tile: C3 columns
// 64 hf .. 64 hf + 63 -> relu(+b3) -> bf16 (TMEM released on read-out), staged in this warp's
// 4 KB (XOR-swizzled by 16-B chunk), then written out coalesced: one instruction stores four
// 128-B half rows.  EG-B takes half 0, EG-A half 1 (split so a lone tile's drain -- the G = 8
// critical path -- is two half-length epilogues in parallel).
__device__ __forceinline__ void e3_half(uint8_t* stg_base, uint32_t tmem_c3, const float* sb3, uint64_t* c3empty,
                                        __nv_bfloat16* a4, uint32_t id, int hf, int q, int lane, bool stores) {
  uint32_t pk[32];
  {
    uint32_t r0[32], r1[32];
    tmem_ld32_nowait(tmem_c3 + 64 * hf, r0);
    tmem_ld32_nowait(tmem_c3 + 64 * hf + 32, r1);
    tmem_wait_ld();
    fence_before();
    __syncwarp();
    if (lane == 0) mbar_arrive(c3empty);                // this half of C3 free for the next tile's conv3
    bias_relu_pack32(r0, sb3 + 64 * hf, pk);
    bias_relu_pack32(r1, sb3 + 64 * hf + 32, pk + 16);
  }
  auto stg = [&](int r, int c) -> uint4* {   // staged half row r (< 32) of this warp, 16-B chunk c (< 8)
    return reinterpret_cast<uint4*>(stg_base + q * 4096 + r * 128) + (c ^ (r & 7));
  };
#pragma unroll
  for (int c = 0; c < 8; ++c) *stg(lane, c) = make_uint4(pk[4 * c], pk[4 * c + 1], pk[4 * c + 2], pk[4 * c + 3]);
  __syncwarp();
  if (!stores) return;
#pragma unroll 4
  for (int u = 0; u < 8; ++u) {
    const int rr = 4 * u + (lane >> 3), cc = lane & 7;
    const uint32_t rid = __shfl_sync(0xffffffffu, id, rr);
    const uint4 v = *stg(rr, cc);
    if (rid != 0xFFFFFFFFu) reinterpret_cast<uint4*>(a4 + ((uint64_t)(rid >> 4) * 14 + (rid & 15)) * 128 + hf * 64)[cc] = v;
  }
  __syncwarp();                                         // staging reads done before it is rewritten
}
// the stores of a half staged by e3_half(..., stores = false)
__device__ __forceinline__ void e3_half_stores(uint8_t* stg_base, __nv_bfloat16* a4, uint32_t id, int hf, int q,
                                               int lane) {
  auto stg = [&](int r, int c) -> uint4* { return reinterpret_cast<uint4*>(stg_base + q * 4096 + r * 128) + (c ^ (r & 7)); };
#pragma unroll 4
  for (int u = 0; u < 8; ++u) {
    const int rr = 4 * u + (lane >> 3), cc = lane & 7;
    const uint32_t rid = __shfl_sync(0xffffffffu, id, rr);
    const uint4 v = *stg(rr, cc);
    if (rid != 0xFFFFFFFFu) reinterpret_cast<uint4*>(a4 + ((uint64_t)(rid >> 4) * 14 + (rid & 15)) * 128 + hf * 64)[cc] = v;
  }
  __syncwarp();
}

// debug timestamps (build with PSIM_TIMING=1): dbg[tile * 256 + slot] = clock64()
// for CTA 0, first 4 tiles of the step named by $PSIM_DEBUG_TIMING
#ifdef PSIM_TIMING
#define PSIM_TS(slot)                                                                                   \
  do {                                                                                                 \
    if (a.dbg && blockIdx.x == 0 && it < 4 && lane == 0) a.dbg[it * 256 + (slot)] = clock64();        \
  } while (0)
// per-CTA span of a kernel: dbg[1024 + (kernel * 160 + cta) * 4 + {0 entry, 1 after the PDL
// wait, 2 end, 3 tiles}] = %globaltimer (ns, comparable across SMs)
#define PSIM_CTA_TS(kern, slot, val)                                                                   \
  do {                                                                                                 \
    if (a.dbg && threadIdx.x == 0 && blockIdx.x < 160) a.dbg[1024 + ((kern) * 160 + blockIdx.x) * 4 + (slot)] = (val); \
  } while (0)
__device__ __forceinline__ long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return (long long)t;
}
#else
#define PSIM_TS(slot) \
  do {                \
  } while (0)
#define PSIM_CTA_TS(kern, slot, val) \
  do {                               \
  } while (0)
#endif

__device__ __forceinline__ uint32_t bf16_bits_u8(uint32_t v) {   // exact: v < 256
  return __float_as_uint((float)v) >> 16;
}
__device__ __forceinline__ uint32_t bf16_bits_int(int v) {       // RNE (time features up to 8190)
  return (uint32_t)__bfloat16_as_ushort(__float2bfloat16_rn((float)v));
}

// load a [rows][K] bf16 row-major weight into K-major SW128 atoms ([rows][64] each)
__device__ void load_weight_sw128(uint8_t* dst, const __nv_bfloat16* w, int rows, int K, int tid, int nthr) {
  const int chunks_per_row = K / 8;   // 16-byte chunks
  const int total = rows * chunks_per_row;
  const uint4* src = reinterpret_cast<const uint4*>(w);
  for (int idx = tid; idx < total; idx += nthr) {
    const int r = idx / chunks_per_row, ch = idx % chunks_per_row;
    const int atom = ch / 8, c = ch % 8;
    st_sw128(dst + atom * rows * 128, r, c, __ldg(src + idx));
  }
}

// conv2 epilogue of conv2 position h of a tile (one warp of a 4-warp epilogue group, TMEM
// quadrant lane_base): C2 slot h (128 fp32) -> relu(+b2) -> bf16x2 written back into the
// first 64 columns of the same slot (conv3's A operand), then a3full[h].
__device__ __forceinline__ void conv2_epilogue(uint32_t tmem, uint32_t lane_base, const float* sb2, uint64_t* c2full,
                                               uint64_t* a3full, uint32_t it, int h, int lane) {
  wait_full(c2full + h, it);
  fence_after();
#pragma unroll 1
  for (int cp = 0; cp < 2; ++cp) {   // channels 64 cp .. 64 cp + 63 -> A3 columns 32 cp .. 32 cp + 31
    uint32_t r0[32], r1[32];
    tmem_ld32_nowait(tmem + lane_base + cs::TMEM_C2 + h * 128 + cp * 64, r0);
    tmem_ld32_nowait(tmem + lane_base + cs::TMEM_C2 + h * 128 + cp * 64 + 32, r1);
    tmem_wait_ld();
    uint32_t pk[32];
    bias_relu_pack32(r0, sb2 + cp * 64, pk);
    bias_relu_pack32(r1, sb2 + cp * 64 + 32, pk + 16);
    // in place: columns 32 cp .. 32 cp + 31 were read already (cp = 1 reads 64 .. 127)
    tmem_st16(tmem + lane_base + cs::TMEM_C2 + h * 128 + cp * 32, pk);
    tmem_st16(tmem + lane_base + cs::TMEM_C2 + h * 128 + cp * 32 + 16, pk + 16);
  }
  tmem_wait_st();
  fence_before();
  __syncwarp();
  if (lane == 0) mbar_arrive(a3full + h);
}

__global__ void __launch_bounds__(cs::THREADS, 1)
    conv_stack_kernel(ConvArgs a, const __grid_constant__ CUtensorMap tmW1, const __grid_constant__ CUtensorMap tmW2,
                      const __grid_constant__ CUtensorMap tmW3, const __grid_constant__ CUtensorMap tmX) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);   // 1024-B aligned; stays in the shared window (LDS/STS, not generic LD/ST)
  uint64_t* bars = reinterpret_cast<uint64_t*>(sm + cs::BAR_OFF);
  PSIM_CTA_TS(0, 0, gtimer());
  uint64_t* xfull = bars + 24;     // [NX] 4 gather warps (arrive.expect_tx) + the gathered rows (complete_tx)
  uint64_t* xempty = bars + 28;    // [NX] commit
  uint64_t* c1full = bars + 4;     // [2] commit: conv1 of the slot's item done
  uint64_t* c1empty = bars + 6;    // [2] commit: the conv2 MMAs reading the slot's A2 done
  uint64_t* a2full = bars + 8;     // [2] 4 (EG-A): A2 (bf16) written into the C1 slot
  uint64_t* c2full = bars + 10;    // [2] commit (one TMEM slot per conv2 position)
  uint64_t* c2empty = bars + 12;   // [2] commit: the conv3 MMAs reading the slot's A3 done
  uint64_t* a3full = bars + 14;    // [2] 4 (EG-B): A3 (bf16) written into the C2 slot
  uint64_t* c3full = bars + 16;    //     commit
  uint64_t* c3empty = bars + 17;   //     8 (EG-B: C3 columns 0..63, EG-A: 64..127)
  uint64_t* wbar = bars + 18;      //     weights + biases landed
  uint64_t* w3full = bars + 21;    //     W3 K-half landed (TMA)
  uint64_t* w3empty = bars + 22;   //     commit: the conv3 MMAs of that half are done
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 44);

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (tid == 0) {
    for (int i = 0; i < cs::NX; ++i) { mbar_init(xfull + i, cs::NISSUE); mbar_init(xempty + i, 1); }
    for (int i = 0; i < 2; ++i) {
      mbar_init(c1full + i, 1); mbar_init(c1empty + i, 1); mbar_init(a2full + i, 4);
      mbar_init(c2full + i, 1); mbar_init(c2empty + i, 1); mbar_init(a3full + i, 4);
    }
    mbar_init(c3full, 1); mbar_init(c3empty, 8);
    mbar_init(wbar, 1);
    mbar_init(w3full, 1); mbar_init(w3empty, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    // resident weights W1/W2 (48 KB) by TMA, already in the SWIZZLE_128B operand layout
    mbar_expect_tx(wbar, 48 * 1024 + 1280);
    float* sbias = reinterpret_cast<float*>(sm + cs::BIAS_OFF);
    bulk_g2s(sbias, a.b1, 256, wbar);
    bulk_g2s(sbias + 64, a.b2, 512, wbar);
    bulk_g2s(sbias + 192, a.b3, 512, wbar);
    for (int kc = 0; kc < 2; ++kc) tma_load_2d(sm + cs::W1_OFF + kc * 8192, &tmW1, wbar, kc * 64, 0);
    for (int kc = 0; kc < 2; ++kc) tma_load_2d(sm + cs::W2_OFF + kc * 16384, &tmW2, wbar, kc * 64, 0);
    // W3 fill 0 (K-half 0 for the first tile's conv3) also before the PDL wait
    mbar_expect_tx(w3full, 32 * 1024);
    for (int a2 = 0; a2 < 2; ++a2) tma_load_2d(sm + cs::W3_OFF + a2 * 16384, &tmW3, w3full, a2 * 64, 0);
  }
  if (warp == cs::MMA_WARP) tmem_alloc(tmem_slot, cs::TMEM_COLS);
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  // Programmatic dependent launch: the setup above overlaps the previous kernel's
  // tail; everything below reads what it wrote (block list, counts, queue state).
  grid_dep_wait();
  grid_dep_launch_dependents();
  const uint32_t nblocks = *a.nblocks;
  const uint32_t ntiles = (nblocks + cs::TILE - 1) / cs::TILE;
  PSIM_CTA_TS(0, 1, gtimer());
  PSIM_CTA_TS(0, 3, (long long)((ntiles + gridDim.x - 1 - blockIdx.x) / gridDim.x));
  if (blockIdx.x == 0 && tid == 0) *a.next_count = 0;
  if (warp <= cs::MMA_WARP) mbar_wait(wbar, 0);   // weights (MMA issuer) and biases (epilogues) resident
  // register budget (setmaxnreg redistributes the launch allocation of 640 x 96; with
  // REG_MMA < 96 the MMA warpgroup would release registers to the issuers -- measured:
  // ptxas then spills in the MMA loop, so it stays at the launch value)
  if constexpr (cs::REG_MMA < 96) {
    if (warp >= cs::MMA_WARP && warp < cs::GATHER_WARP0) setmaxnreg_dec<cs::REG_MMA>();
  }
  const float* sb1 = reinterpret_cast<const float*>(sm + cs::BIAS_OFF);
  const float* sb2 = sb1 + 64;
  const float* sb3 = sb1 + 192;

  if (warp == cs::MMA_WARP) {
    {   // ============================ MMA issuer
      // Per tile: c1(0) c1(1) [c3 of the previous tile, K-half 1] c2(0,*) c1(2) c1(3) c3(0) c2(1,*);
      // deferring the previous tile's last conv3 MMA lets this tile's conv1 overlap its epilogues.
      // The whole warp runs this loop (descriptors stay warp-uniform, in uniform registers);
      // one elected lane issues each MMA group and its commits.
      const bool leader = elect_one();
      // W3 stream (K-halves 0, 1, 0, 1, ... into one 32 KB buffer): fill f after the conv3
      // MMAs of fill f-1 completed.  Issued two MMA groups ahead of its use, where that
      // completion has normally already happened.
      uint32_t nfill = 1;   // fill 0 was issued with the resident weights, before the PDL wait
      auto fill = [&]() {
        wait_empty(w3empty, nfill);
        if (leader) {
          mbar_expect_tx(w3full, 32 * 1024);
          for (int a2 = 0; a2 < 2; ++a2)
            tma_load_2d(sm + cs::W3_OFF + a2 * 16384, &tmW3, w3full, (int)(2 * (nfill & 1) + a2) * 64, 0);
        }
        __syncwarp();
        ++nfill;
      };
      const uint32_t sbase = smem_u32(sm);
      const uint32_t id64 = idesc_bf16(128, 64), id128 = idesc_bf16(128, 128);
      auto c1 = [&](uint32_t it, int j) {
        const int s = j & 1;                        // C1 TMEM slot
        const uint32_t n = it * 2 + (j >> 1);
        const uint32_t item = it * 4 + j, xs = item % cs::NX;   // X slot of this item
        PSIM_TS(0 + 2 * j);
        wait_full(xfull + xs, item / cs::NX);
        wait_empty(c1empty + s, n);
        PSIM_TS(1 + 2 * j);
        fence_after();
        const uint32_t xa = sbase + cs::X_OFF + xs * 32768;
        if (leader) {
#pragma unroll
          for (int k = 0; k < 8; ++k)
            mma_bf16(tmem + cs::TMEM_C1 + s * 64, sw128_desc(xa + (k >> 2) * 16384 + (k & 3) * 32),
                     sw128_desc(sbase + cs::W1_OFF + (k >> 2) * 8192 + (k & 3) * 32), id64, k > 0);
          mma_commit(xempty + xs);
          mma_commit(c1full + s);
        }
        __syncwarp();
      };
      auto c2 = [&](uint32_t it, int h, int kh) {   // conv2 position h, K-half kh = item 2h+kh (C1 slot kh)
        PSIM_TS(8 + 2 * (h * 2 + kh));
        wait_full(a2full + kh, it * 2 + h);
        if (kh == 0) wait_empty(c2empty + h, it);
        PSIM_TS(9 + 2 * (h * 2 + kh));
        fence_after();
        if (leader) {
#pragma unroll
          for (int k = 0; k < 4; ++k)
            mma_bf16_ts(tmem + cs::TMEM_C2 + h * 128, tmem + cs::TMEM_C1 + kh * 64 + 8 * k,
                        sw128_desc(sbase + cs::W2_OFF + kh * 16384 + k * 32), id128, (kh | k) != 0);
          mma_commit(c1empty + kh);   // C1 slot kh (its A2) free for conv1 two items later
          if (kh == 1) mma_commit(c2full + h);
        }
        __syncwarp();
      };
      auto c3 = [&](uint32_t it, int kh) {   // the (2 it + kh)-th conv3 MMA group: W3 K-half kh, A3 in C2 slot kh
        PSIM_TS(16 + 2 * kh);
        wait_full(a3full + kh, it);
        if (kh == 0) wait_empty(c3empty, it);
        wait_full(w3full, it * 2 + kh);
        PSIM_TS(17 + 2 * kh);
        fence_after();
        if (leader) {
#pragma unroll
          for (int k = 0; k < 8; ++k)
            mma_bf16_ts(tmem + cs::TMEM_C3, tmem + cs::TMEM_C2 + kh * 128 + 8 * k,
                        sw128_desc(sbase + cs::W3_OFF + (k >> 2) * 16384 + (k & 3) * 32), id128, (kh | k) != 0);
          mma_commit(w3empty);
          mma_commit(c2empty + kh);   // C2 slot kh free for the next tile's conv2 position kh
          if (kh == 1) mma_commit(c3full);
        }
        __syncwarp();
      };
      uint32_t it = 0;
      for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x, ++it) {
        c1(it, 0); c1(it, 1);
        if (it > 0) c3(it - 1, 1);
        c2(it, 0, 0); c2(it, 0, 1);
        if (it > 0) fill();                           // half 0 for c3(it, 0): after c3(it - 1, 1)
        c1(it, 2); c1(it, 3); c3(it, 0); c2(it, 1, 0);
        fill();                                       // half 1 for c3(it, 1): after c3(it, 0)
        c2(it, 1, 1);
      }
      if (it > 0) c3(it - 1, 1);
      if (it == 0) wait_full(w3full, 0);   // no tile: still let fill 0 land before the CTA exits
    }
    __syncwarp();
  } else if (warp < 4) {   // ============ EG-A: conv1 epilogues (C1 -> A2, in TMEM) + conv2 position 0 epilogue
    setmaxnreg_inc<cs::REG_EPI>();
    const int q = warp & 3;                         // TMEM lane quadrant (tile rows 32 q .. 32 q + 31)
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t it = 0;
    for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x, ++it) {
#pragma unroll 1
      for (int j = 0; j < 4; ++j) {
        const int s = j & 1;
        if (q == 0) PSIM_TS(32 + 4 * j);
        wait_full(c1full + s, it * 2 + (j >> 1));
        if (q == 0) PSIM_TS(33 + 4 * j);
        fence_after();
        uint32_t pk[32];
        {
          uint32_t r0[32], r1[32];
          tmem_ld32_nowait(tmem + lane_base + cs::TMEM_C1 + s * 64, r0);
          tmem_ld32_nowait(tmem + lane_base + cs::TMEM_C1 + s * 64 + 32, r1);
          tmem_wait_ld();
          bias_relu_pack32(r0, sb1, pk);
          bias_relu_pack32(r1, sb1 + 32, pk + 16);
        }
        if (q == 0) PSIM_TS(34 + 4 * j);
        // A2 = relu(C1 + b1) as bf16x2 into columns 0..31 of the same C1 slot (conv2's A operand)
        tmem_st16(tmem + lane_base + cs::TMEM_C1 + s * 64, pk);
        tmem_st16(tmem + lane_base + cs::TMEM_C1 + s * 64 + 16, pk + 16);
        tmem_wait_st();
        fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(a2full + s);
        if (q == 0) PSIM_TS(48 + j);
        if (j == 1 || (kEgaConv2Pos1 && j == 3)) {   // conv2 position j / 2 (items j - 1, j) after conv2 MMAs (j / 2, *)
          if (q == 0) PSIM_TS(j == 1 ? 56 : 60);
          conv2_epilogue(tmem, lane_base, sb2, c2full, a3full, it, j >> 1, lane);
          if (q == 0) PSIM_TS(j == 1 ? 59 : 63);
        }
        if (j == 1 && it > 0) {   // channels 64..127 of the previous tile's conv3 (complete by now: its last
                                  // MMAs were issued before this tile's conv2 position 0): read out + staged
          wait_full(c3full, it - 1);
          fence_after();
          e3_half(sm + cs::STG_OFF + 16384, tmem + lane_base + cs::TMEM_C3, sb3, c3empty, a.a4, 0u, 1, q, lane, false);
        }
      }
      if (it > 0) {             // ... and written out once this tile's conv1 epilogues are done
        const uint32_t bi = (tl - gridDim.x) * cs::TILE + q * 32 + lane;
        e3_half_stores(sm + cs::STG_OFF + 16384, a.a4, bi < nblocks ? a.blocks[bi].x : 0xFFFFFFFFu, 1, q, lane);
      }
    }
    if (it > 0) {               // the last tile's half: both halves drain in parallel (EG-B takes 0..63)
      const uint32_t tl_last = blockIdx.x + (it - 1) * gridDim.x;
      const uint32_t bi = tl_last * cs::TILE + q * 32 + lane;
      const uint32_t id = bi < nblocks ? a.blocks[bi].x : 0xFFFFFFFFu;
      wait_full(c3full, it - 1);
      fence_after();
      e3_half(sm + cs::STG_OFF + 16384, tmem + lane_base + cs::TMEM_C3, sb3, c3empty, a.a4, id, 1, q, lane, true);
    }
  } else if (warp < 8) {   // ============================ EG-B: conv2 position 1 + conv3 epilogues
    setmaxnreg_inc<cs::REG_EPI>();
    // Order per tile t: e3(t - 1), then the conv2 epilogue of position 1 of tile t (position
    // 0 is EG-A's, so conv3(t, 0) does not wait for e3(t - 1) to write its rows out).
    const int q = warp & 3;
    const int m = q * 32 + lane;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    // C3 (128 fp32) -> relu(+b3) -> bf16 -> a4[b][p], channels 0..63 here (e3_half); EG-A
    // drains channels 64..127 after its conv2 position-0 epilogue of the next tile.
    auto e3 = [&](uint32_t it, uint32_t tl) {   // channels 0..63 (EG-A takes 64..127)
      const uint32_t bi = tl * cs::TILE + m;
      const uint32_t id = bi < nblocks ? a.blocks[bi].x : 0xFFFFFFFFu;
      if (q == 0) PSIM_TS(64);
      wait_full(c3full, it);                          // conv3 accumulated
      if (q == 0) PSIM_TS(65);
      fence_after();
      e3_half(sm + cs::STG_OFF, tmem + lane_base + cs::TMEM_C3, sb3, c3empty, a.a4, id, 0, q, lane, true);
      if (q == 0) PSIM_TS(66);
    };
    uint32_t it = 0, prev_tl = 0;
    for (uint32_t tl = blockIdx.x; tl < ntiles; tl += gridDim.x, ++it) {
      if (it > 0) e3(it - 1, prev_tl);
      if constexpr (!kEgaConv2Pos1) {
        if (q == 0) PSIM_TS(60);
        conv2_epilogue(tmem, lane_base, sb2, c2full, a3full, it, 1, lane);
        if (q == 0) PSIM_TS(63);
      }
      prev_tl = tl;
    }
    if (it > 0) e3(it - 1, prev_tl);
  } else if (warp >= cs::GATHER_WARP0) {   // ============================ row builders + TMA issuers (warps 12..19)
    // Operand row layout (per input row, 64 bf16): cols 0..46 the trace attributes,
    // col 47 zero, cols 48..50 the time features, cols 51..63 zero.  Item n = conv1
    // position j = n % 4 of this CTA's tile n / 4: input rows R = 8p + 2j + h (h = 0, 1;
    // PAPER.md:93 row order) of the tile's 128 blocks (b, p).
    // Lane l of issuer warp wq BUILDS the row of block m = 16 wq + (l & 15), h = l >> 4:
    // padding (R > k) -> row kPadRow past the tensor (zero-filled by the TMA); R = 0 -> the
    // current instruction; context rows newest first -> the row of queue entry k - R (R6),
    // with the time features age / remaining-to-complete / remaining-to-retire (R2) in
    // chunk 6 (cols 48..55) of its SW128 operand row.  The metadata chain block entry
    // {b << 4 | p, k, ws, Clock} -> queue entry is software-pipelined in registers: the
    // block entries of tile T + 1 are loaded at the start of tile T and the queue entries
    // of item n + 2 after item n is issued (L2-only loads, .cg), so no load latency sits
    // on the issue path.  Lanes 0..7 then ISSUE the rows by TMA tile::gather4 (4 arbitrary
    // 96-B trace16 rows per instruction, SWIZZLE_128B applied on the way) into chunks 0..5
    // of the X slot: lane (g, h) = (l & 3, l >> 2 & 1) fetches blocks 16 wq + 4 g .. + 3,
    // atom h, with the row indices shuffled from the building lanes.  Each warp arrives on
    // the slot's xfull barrier with the byte count its gathers deliver (expect_tx), so
    // xfull completes when the last row lands.
    setmaxnreg_dec<cs::REG_ISSUE>();
    const int wq = warp - cs::GATHER_WARP0;          // issuer warp 0..7
    const int m = 16 * wq + (lane & 15), hh = lane >> 4;
#pragma unroll
    for (int s2 = 0; s2 < cs::NX; ++s2) st_sw128(sm + cs::X_OFF + s2 * 32768 + hh * 16384, m, 7, make_uint4(0, 0, 0, 0));
    const uint32_t my_tiles = blockIdx.x < ntiles ? (ntiles - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    const int g = lane & 3, h = (lane >> 2) & 1;     // TMA lane l < 8: rows of atom h, blocks 16 wq + 4 g .. + 3
    // trace rows are streamed through L2 with evict_first: the step's context rows
    // (~145 MB at config 3, G = 1) exceed L2 and would otherwise push out the queue
    // entries, states and a4 rows that are reused within the step
    const uint64_t pol = a.rows_keep ? l2_policy_evict_last() : l2_policy_evict_first();
    const uint4 kNoBlock = make_uint4(0xFFFFFFFFu, 0u, 0u, 0u);
    auto row_R = [&](const uint4& be, uint32_t n) -> int { return (int)(be.x & 15) * 8 + 2 * (int)(n & 3) + hh; };
    // Metadata pipeline, all through lane-private smem rings filled by cp.async (no register
    // ever waits on a load in flight): block entries of tile T in slot T % 3, staged two
    // tiles ahead (beC / beN = register copies of tiles T / T + 1 read at each tile start);
    // the queue entry of item n in slot n % ER, staged ED items ahead.  One cp.async group
    // per item (its entry) and one per tile (a block-entry slot): the wait before item n
    // allows the ED - 1 later entry groups (+ at most one block-entry group) to stay pending.
    uint4* sBE = reinterpret_cast<uint4*>(sm + cs::BE_OFF) + wq * 32 + lane;
    uint4* sER = reinterpret_cast<uint4*>(sm + cs::ER_OFF) + wq * 32 + lane;
    auto stage_block = [&](uint32_t T) {
      const uint32_t bi = (blockIdx.x + T * gridDim.x) * cs::TILE + m;
      uint4* dst = sBE + (T % 3) * 256;
      if (T < my_tiles && bi < nblocks) cp_async16(dst, a.blocks + bi);
      else *dst = kNoBlock;
      cp_async_commit();
    };
    const uint32_t n_items = my_tiles * 4;
    auto stage_entry = [&](const uint4& be, uint32_t n) {   // queue entry of this lane's row of item n
      const int R = row_R(be, n), k = (int)be.y;
      if (n < n_items && be.x != 0xFFFFFFFFu && R >= 1 && R <= k)
        cp_async16(sER + (n % cs::ER) * 256, a.q + (uint64_t)(k - R) * a.qn + (be.x >> 4));
      cp_async_commit();
    };
    stage_block(0);
    stage_block(1);
    cp_async_wait<0>();
    uint4 beC = sBE[0], beN = sBE[256];
#pragma unroll
    for (uint32_t n = 0; n < (uint32_t)cs::ED; ++n) stage_entry(beC, n);   // ED == 4: tile 0
    stage_block(2);
    // commit order ... E(n) E(n+1) E(n+2) E(n+3) with exactly one block-entry group among
    // the four groups after any E(n), and exactly four entry groups after BE(T + 2) at the
    // end of tile T: cp.async.wait_group 4 is exact in both places
    static_assert(cs::ED == 4 && cs::ER >= 2 * cs::ED, "entry ring: items n + ED stay in tile + 1");
    auto item = [&](uint32_t nI) {
      const uint32_t it = nI >> 2;                     // this CTA's tile of item nI
      [[maybe_unused]] const int j = (int)(nI & 3);    // conv1 position (timestamps)
      if (warp == cs::GATHER_WARP0) PSIM_TS(81 + 3 * j);
      cp_async_wait<cs::ED>();                         // item nI's entry has landed (own slot)
      // ---- build this lane's row of item nI
      uint32_t row;
      uint2 tc = make_uint2(0u, 0u);
      {
        const int R = row_R(beC, nI), k = (int)beC.y;
        if (beC.x == 0xFFFFFFFFu || R > k) {
          row = a.zero_row;                                        // zero padding at the tail
        } else if (R == 0) {
          row = (uint32_t)((int64_t)(beC.z + (uint32_t)a.step) - a.row_lo);   // current instruction first
        } else {
          const uint4 ev = sER[(nI % cs::ER) * 256];
          const int c = ev.z & 0xFFFF, sv = (ev.z >> 16) & 0xFFFF;
          const int age = (int)(beC.w - ev.y);
          const int t0 = min(age, kTimeMax), t1 = min(max(0, c - age), kTimeMax), t2 = min(c + sv - age, kTimeMax);
          tc = make_uint2(pack_bf16((float)t0, (float)t1), pack_bf16((float)t2, 0.f));
          row = (uint32_t)((int64_t)ev.x - a.row_lo);
        }
      }
      if (warp == cs::GATHER_WARP0) PSIM_TS(83 + 3 * j);
      stage_entry(beN, nI + cs::ED);                   // item nI + 4: tile it + 1
      if (warp == cs::GATHER_WARP0) PSIM_TS(97 + 2 * j);
      // row indices of the 4 blocks this lane gathers (TMA lanes 0..7): lanes 4 g + i + 16 h
      const uint32_t r0 = __shfl_sync(0xffffffffu, row, 4 * g + 0 + 16 * h);
      const uint32_t r1 = __shfl_sync(0xffffffffu, row, 4 * g + 1 + 16 * h);
      const uint32_t r2 = __shfl_sync(0xffffffffu, row, 4 * g + 2 + 16 * h);
      const uint32_t r3 = __shfl_sync(0xffffffffu, row, 4 * g + 3 + 16 * h);
      if (warp == cs::GATHER_WARP0) PSIM_TS(104 + j);
      const int xs = (int)(nI % cs::NX);
      wait_empty(xempty + xs, nI / cs::NX);
      if (warp == cs::GATHER_WARP0) PSIM_TS(82 + 3 * j);
      uint8_t* xa = sm + cs::X_OFF + xs * 32768;
      // chunk 6 (cols 48..55): time features of context rows, zero otherwise (R2); the TMA
      // writes only chunks 0..5, so this can go in before the rows land
      st_sw128(xa + hh * 16384, m, 6, make_uint4(tc.x, tc.y, 0u, 0u));
      if (warp == cs::GATHER_WARP0) PSIM_TS(112 + 3 * j);
      fence_async_smem();                               // chunk 6 visible to tcgen05
      __syncwarp();
      if (warp == cs::GATHER_WARP0) PSIM_TS(113 + 3 * j);
      if (lane == 0) mbar_expect_tx(xfull + xs, 32 * 96);   // arrive + this warp's 32 rows of 96 B
      __syncwarp();
      if (warp == cs::GATHER_WARP0) PSIM_TS(114 + 3 * j);
      if (lane < 8)
        tma_gather4_hint(xa + h * 16384 + (16 * wq + 4 * g) * 128, &tmX, xfull + xs, 0, r0, r1, r2, r3, pol);
      __syncwarp();
      if (warp == cs::GATHER_WARP0) PSIM_TS(96 + 2 * j);
      if (((nI + 1) & 3) == 0) {                        // the next item starts tile it + 1
        cp_async_wait<4>();                             // tile it + 2's block entries (staged a tile ago;
                                                        // only this tile's 4 entry groups are younger)
        beC = beN;
        beN = sBE[((it + 2) % 3) * 256];
        stage_block(it + 3);                            // into slot it % 3 (tile it is done)
      }
    };
#pragma unroll 1
    for (uint32_t nI = 0; nI < n_items; ++nI) item(nI);
  }
  fence_before();
  __syncthreads();
  PSIM_CTA_TS(0, 2, gtimer());
  if (warp == cs::MMA_WARP) {
    fence_after();
    tmem_dealloc(tmem, cs::TMEM_COLS);
  }
}

// ============================================================ fc1 / head / update
namespace fh {
constexpr int BM = 128, BN = 256, BK = 64;
constexpr int A_BYTES = BM * BK * 2, B_BYTES = BN * BK * 2, STAGE = A_BYTES + B_BYTES;
constexpr int STAGES = 4;
constexpr int T_STRIDE = 260;                 // padded rows of the constant table (bank spread, 16-B rows)
constexpr int T_OFF = STAGES * STAGE;         // float [15][257]
constexpr int W2_OFF = T_OFF + 15 * T_STRIDE * 4;   // float [3][256] + bias[3]
#ifndef PSIM_FC1_UPD_GROUPS
#define PSIM_FC1_UPD_GROUPS 2
#endif
constexpr int UPD_GROUPS = PSIM_FC1_UPD_GROUPS;   // update groups of 4 warps, tiles round-robin
constexpr int Y_OFF = W2_OFF + (3 * 256 + 4) * 4;   // float [UPD_GROUPS][128][3]: y of tile t in buffer t % UPD_GROUPS
constexpr int P_OFF = Y_OFF + UPD_GROUPS * 128 * 3 * 4;      // int [UPD_GROUPS][16] tile scan scratch per update group
constexpr int H_OFF = P_OFF + UPD_GROUPS * 16 * 4;  // uint [112] k histogram of this CTA
constexpr int BAR_OFF = (H_OFF + 112 * 4 + 7) & ~7;
static_assert(8 * (4 + 4 + 2 + 2 + 1 + 2 * UPD_GROUPS) + 4 <= 256, "barrier area");
constexpr int SMEM = BAR_OFF + 256 + 1024;
// pair mode (fc1 on 2-SM MMAs): a cluster of two CTAs computes two tiles with one
// tcgen05.mma.cta_group::2 (M = 256): each CTA stages its own tile's a4 rows and HALF of the
// W_fc1 slice (N rows 128 r .. 128 r + 127), so the W_fc1 stream per SM halves; smaller
// stages (32 KB) -> 6 of them in the same 192 KB
constexpr int PSTAGE = A_BYTES + B_BYTES / 2, PSTAGES = (STAGES * STAGE) / PSTAGE;
constexpr int THREADS = 192 + 128 * UPD_GROUPS;   // warp 0 TMA, 1 MMA, 2-5 epilogue (F -> y), 6.. update groups (4 warps each)
}  // namespace fh

__device__ __forceinline__ void named_bar_sync(int id, int nthreads) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

struct HeadArgs {
  UpdateArgs u;              // state, step, cap, forced, records (y unused)
  const int64_t* e;
  const uint8_t* tileP;      // [ntiles] P_tile of this step
  uint8_t* tileP_next;       // [ntiles] P_tile of the next step
  uint4* blocks_next;        // block list of the next step
  uint32_t* next_count;
  __nv_bfloat16* a4;         // [n][14][128] (zero-fill of [P_b, P_tile) for the next step)
  const float* T;            // [15][256] constant table
  const float* w2;           // [3][256]
  const float* b2;           // [3]
  int force_predict;         // run the head even when teacher-forced
  long long* dbg;            // optional timestamps (PSIM_DEBUG_TIMING), slots 128..
  unsigned long long* ptile_sum;   // sum of P_tile over the tiles of the run (fc1 K statistics)
};

template <bool kPair>
__global__ void __launch_bounds__(fh::THREADS, 1)
    fc1_head_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, HeadArgs a) {
  constexpr int kStages = kPair ? fh::PSTAGES : fh::STAGES;
  constexpr int kStage = kPair ? fh::PSTAGE : fh::STAGE;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* sm = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);   // 1024-B aligned; stays in the shared window (LDS/STS, not generic LD/ST)
  float* sT = reinterpret_cast<float*>(sm + fh::T_OFF);
  PSIM_CTA_TS(1, 0, gtimer());
  float* sW2 = reinterpret_cast<float*>(sm + fh::W2_OFF);
  int* sP = reinterpret_cast<int*>(sm + fh::P_OFF);
  unsigned int* sHist = reinterpret_cast<unsigned int*>(sm + fh::H_OFF);
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + fh::BAR_OFF);
  uint64_t* empty = full + kStages;
  uint64_t* tfull = empty + kStages;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = nullptr;

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const uint64_t n = a.u.st.n;
  const uint32_t ntiles = (uint32_t)((n + fh::BM - 1) / fh::BM);
  // tile schedule: single mode, CTA c takes tiles c, c + G, ...; pair mode, the CTA of rank r in
  // cluster q takes tiles 2 (q + k Q) + r (k = 0, 1, ...; a tile >= ntiles is empty: its a4 rows
  // read as zero past the tensor, its rows are skipped by the epilogue and the update)
  const uint32_t rank = kPair ? cluster_ctarank() : 0u;
  const uint32_t t0 = kPair ? 2 * cluster_id_x() + rank : blockIdx.x;
  const uint32_t tstep = kPair ? 2 * ncluster_x() : gridDim.x;
  const uint32_t tend = kPair ? ((ntiles + 1) & ~1u) : ntiles;   // pairs cover the odd last tile
  auto tileP_of = [&](uint32_t t) -> int { return t < ntiles ? (int)a.tileP[t] : 0; };
  auto nk_of = [&](uint32_t t) -> int {                           // k-blocks of tile t (pair: of its pair)
    return kPair ? 2 * max(tileP_of(t & ~1u), tileP_of(t | 1u)) : 2 * tileP_of(t);
  };

  uint64_t* cbar = tempty + 2;   // constant table + fc2 landed (bulk copies)
  // y of tile it in sY[it % UPD_GROUPS], consumed by update group it % UPD_GROUPS (so one
  // buffer's phases are always consumed in order by one group)
  uint64_t* yfull = cbar + 1;                   // [UPD_GROUPS] epilogue -> update
  uint64_t* yempty = yfull + fh::UPD_GROUPS;    // [UPD_GROUPS] update -> epilogue: consumed
  float* sY = reinterpret_cast<float*>(sm + fh::Y_OFF);
  tmem_slot = reinterpret_cast<uint32_t*>(yempty + fh::UPD_GROUPS);
  if (tid < 3) sW2[768 + tid] = a.b2[tid];
  for (int idx = tid; idx < 112; idx += fh::THREADS) sHist[idx] = 0;
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    // pair mode: tempty of the even CTA collects the epilogue warps of both CTAs
    for (int i = 0; i < 2; ++i) { mbar_init(tfull + i, 1); mbar_init(tempty + i, kPair ? 8 : 4); }
    mbar_init(cbar, 1);
    for (int i = 0; i < fh::UPD_GROUPS; ++i) { mbar_init(yfull + i, 4); mbar_init(yempty + i, 4); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    mbar_expect_tx(cbar, 15 * 1024 + 3 * 1024);
    for (int r = 0; r < 15; ++r) bulk_g2s(sT + r * fh::T_STRIDE, a.T + r * 256, 1024, cbar);
    bulk_g2s(sW2, a.w2, 3 * 1024, cbar);
  }
  if (warp == 1) {
    if constexpr (kPair) tmem_alloc_2sm(tmem_slot, 512);   // both CTAs, same warp
    else tmem_alloc(tmem_slot, 512);
  }
  fence_before();
  __syncthreads();
  if constexpr (kPair) cluster_sync();   // barrier inits visible to the peer before any remote use
  fence_after();
  const uint32_t tmem = *tmem_slot;
  // PDL: every role waits (griddepcontrol.wait) for a4, block counts and queue state of
  // conv_stack / the previous step before touching them; the TMA producer first puts the
  // weight (B) halves of its first tile's first stages in flight: W_fc1 does not depend on
  // the previous kernels, and tileP of this step was written by the previous fc1_head,
  // complete before conv_stack of this step passed its own wait (and so before this
  // kernel could launch).
  grid_dep_launch_dependents();
  const bool run_head = (a.u.forced == nullptr) || a.force_predict;
  int npre = 0;   // producer: k-blocks of the first tile whose B half was issued before the wait
  if (warp == 0 && lane == 0 && run_head && t0 < tend) {
    npre = min(nk_of(t0), kStages);
    for (int kb = 0; kb < npre; ++kb) {
      uint8_t* sa = sm + kb * kStage;
      if constexpr (kPair) {
        if (rank == 0) mbar_expect_tx(full + kb, 2 * kStage);   // both CTAs' A + B-half bytes
        tma_load_2d_2sm(sa + fh::A_BYTES, &tmB, full + kb, kb * fh::BK, 128 * (int)rank, l2_policy_evict_last());
      } else {
        mbar_expect_tx(full + kb, fh::STAGE);
        tma_load_2d_hint(sa + fh::A_BYTES, &tmB, full + kb, kb * fh::BK, 0, l2_policy_evict_last());
      }
    }
  }
  grid_dep_wait();
  PSIM_CTA_TS(1, 1, gtimer());
  if (warp >= 2 && warp < 6) mbar_wait(cbar, 0);   // epilogue warps read T and fc2 from smem

  if (warp == 0) {
    if (lane == 0 && run_head) {   // ---- TMA producer
      // L2 policies: a4 rows are read once per step (evict_first), W_fc1 by every tile (evict_last)
      const uint64_t polA = l2_policy_evict_first(), polB = l2_policy_evict_last();
      uint32_t stage = 0, phase = 0;
      uint32_t it = 0;
      for (uint32_t tt = t0; tt < tend; tt += tstep, ++it) {
        const int nk = nk_of(tt);
        PSIM_TS(128);
        for (int kb = 0; kb < nk; ++kb) {
          uint8_t* sa = sm + stage * kStage;
          if constexpr (kPair) {
            if (!(it == 0 && kb < npre)) {              // else B already in flight (issued before the PDL wait)
              mbar_wait(empty + stage, phase ^ 1);      // released by the pair's MMA commit (multicast)
              if (rank == 0) mbar_expect_tx(full + stage, 2 * kStage);
              tma_load_2d_2sm(sa + fh::A_BYTES, &tmB, full + stage, kb * fh::BK, 128 * (int)rank, polB);
            }
            tma_load_2d_2sm(sa, &tmA, full + stage, kb * fh::BK, (int)(tt * fh::BM), polA);
          } else if (it == 0 && kb < npre) {            // B already in flight (issued before the PDL wait)
            tma_load_2d_hint(sa, &tmA, full + stage, kb * fh::BK, (int)(tt * fh::BM), polA);
          } else {
            mbar_wait(empty + stage, phase ^ 1);
            mbar_expect_tx(full + stage, fh::STAGE);
            tma_load_2d_hint(sa, &tmA, full + stage, kb * fh::BK, (int)(tt * fh::BM), polA);
            tma_load_2d_hint(sa + fh::A_BYTES, &tmB, full + stage, kb * fh::BK, 0, polB);
          }
          if (++stage == kStages) { stage = 0; phase ^= 1; }
        }
        PSIM_TS(129);
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && run_head && rank == 0) {   // ---- MMA issuer (pair mode: the even CTA issues for both)
      constexpr uint32_t idesc = idesc_bf16(kPair ? 2 * fh::BM : fh::BM, fh::BN);
      uint32_t stage = 0, phase = 0, it = 0;
      for (uint32_t tt = t0; tt < tend; tt += tstep, ++it) {
        const int nk = nk_of(tt);
        const int acc = it & 1;
        PSIM_TS(132);
        wait_empty(tempty + acc, it >> 1);
        PSIM_TS(133);
        fence_after();
        for (int kb = 0; kb < nk; ++kb) {
          mbar_wait(full + stage, phase);
          fence_after();
          const uint32_t sa = smem_u32(sm + stage * kStage), sb = sa + fh::A_BYTES;
#pragma unroll
          for (int k = 0; k < fh::BK / 16; ++k) {
            if constexpr (kPair)   // A: 128 rows per CTA (M = 256), B: 128 N-rows per CTA (N = 256)
              mma_bf16_2sm(tmem + acc * fh::BN, sw128_desc(sa + 32 * k), sw128_desc(sb + 32 * k), idesc, (kb | k) != 0);
            else
              mma_bf16(tmem + acc * fh::BN, sw128_desc(sa + 32 * k), sw128_desc(sb + 32 * k), idesc, (kb | k) != 0);
          }
          if constexpr (kPair) mma_commit_2sm_mc(empty + stage, 0x3);   // frees the stage in both CTAs
          else mma_commit(empty + stage);
          if (++stage == kStages) { stage = 0; phase ^= 1; }
        }
        // accumulator ready (nk == 0: arrives once the earlier MMAs are done)
        if constexpr (kPair) mma_commit_2sm_mc(tfull + acc, 0x3);
        else mma_commit(tfull + acc);
        PSIM_TS(134);
      }
    }
  } else if (warp < 6) {   // ---- epilogue (warps 2..5): F -> relu(F + T[P_b]) . fc2 -> y in smem
    const int q = warp & 3;
    const int m = q * 32 + lane;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t it = 0;
    for (uint32_t tt = t0; tt < tend; tt += tstep, ++it) {
      const int acc = it & 1, yb = it % fh::UPD_GROUPS;
      const uint64_t b = (uint64_t)tt * fh::BM + m;
      const int ptile = tileP_of(tt);
      const int kb = b < n ? a.u.st.count[b] : 0;   // read before this tile's update (y handoff orders it)
      const int pb = min((kb + 8) >> 3, 14);        // computed positions of this sub-trace
      float y0 = 0.f, y1 = 0.f, y2 = 0.f;
      if (q == 2) PSIM_TS(140);
      if (run_head) {
        wait_full(tfull + acc, it >> 1);
        if (q == 2) PSIM_TS(141);
        fence_after();
        y0 = sW2[768]; y1 = sW2[769]; y2 = sW2[770];
        const float* Trow = sT + pb * fh::T_STRIDE;
        // fc1 = F (positions < P_tile; rows [P_b, P_tile) are zero) + T[P_b]; ReLU; fc2 (R16, R18).
        // Two TMEM loads in flight (the next 32 columns load while these are consumed) and
        // two partial sums per output (halves the dependent FMA chains).
        float z0 = 0.f, z1 = 0.f, z2 = 0.f;
        const uint32_t tbase = tmem + lane_base + acc * fh::BN;
        uint32_t ra[32], rb[32];
        tmem_ld32_nowait(tbase, ra);
        auto consume = [&](const uint32_t (&r0)[32], int cc) {
#pragma unroll
          for (int j4 = 0; j4 < 8; ++j4) {
            const int col = cc * 32 + j4 * 4;
            const float4 tv = *reinterpret_cast<const float4*>(Trow + col);
            const float4 w0 = *reinterpret_cast<const float4*>(sW2 + col);
            const float4 w1 = *reinterpret_cast<const float4*>(sW2 + 256 + col);
            const float4 w2v = *reinterpret_cast<const float4*>(sW2 + 512 + col);
            const float f0 = ptile > 0 ? __uint_as_float(r0[j4 * 4]) : 0.f, f1 = ptile > 0 ? __uint_as_float(r0[j4 * 4 + 1]) : 0.f;
            const float f2 = ptile > 0 ? __uint_as_float(r0[j4 * 4 + 2]) : 0.f, f3 = ptile > 0 ? __uint_as_float(r0[j4 * 4 + 3]) : 0.f;
            const float h0 = fmaxf(f0 + tv.x, 0.f), h1 = fmaxf(f1 + tv.y, 0.f);
            const float h2 = fmaxf(f2 + tv.z, 0.f), h3 = fmaxf(f3 + tv.w, 0.f);
            y0 = fmaf(h0, w0.x, y0); z0 = fmaf(h1, w0.y, z0); y0 = fmaf(h2, w0.z, y0); z0 = fmaf(h3, w0.w, z0);
            y1 = fmaf(h0, w1.x, y1); z1 = fmaf(h1, w1.y, z1); y1 = fmaf(h2, w1.z, y1); z1 = fmaf(h3, w1.w, z1);
            y2 = fmaf(h0, w2v.x, y2); z2 = fmaf(h1, w2v.y, z2); y2 = fmaf(h2, w2v.z, y2); z2 = fmaf(h3, w2v.w, z2);
          }
        };
#pragma unroll 1
        for (int cc = 0; cc < fh::BN / 32; cc += 2) {
          tmem_wait_ld();                                   // columns cc (ra) landed
          tmem_ld32_nowait(tbase + (cc + 1) * 32, rb);
          consume(ra, cc);
          tmem_wait_ld();                                   // columns cc + 1 (rb) landed
          if (cc + 2 < fh::BN / 32) tmem_ld32_nowait(tbase + (cc + 2) * 32, ra);
          consume(rb, cc + 1);
        }
        y0 += z0; y1 += z1; y2 += z2;
        fence_before();
        __syncwarp();
        if (lane == 0) {
          if constexpr (kPair) mbar_arrive_cluster(mapa_shared(tempty + acc, 0));   // the issuing CTA's barrier
          else mbar_arrive(tempty + acc);
        }
      }
      wait_empty(yempty + yb, it / fh::UPD_GROUPS);
      float* yrow = sY + (yb * 128 + m) * 3;
      yrow[0] = y0; yrow[1] = y1; yrow[2] = y2;
      __syncwarp();
      if (lane == 0) mbar_arrive(yfull + yb);
      if (q == 2) PSIM_TS(142);
    }
  } else {   // ---- update (group 0: warps 6..9 even tiles, group 1: 10..13 odd tiles), thread per sub-trace
    const int grp = (warp - 6) >> 2;
    const int q = (warp - 6) & 3;
    const int m = q * 32 + lane;
    int* sPg = sP + grp * 16;
    uint32_t it = grp;
    for (uint32_t tt = t0 + grp * tstep; tt < tend; tt += fh::UPD_GROUPS * tstep, it += fh::UPD_GROUPS) {
      const int yb = it % fh::UPD_GROUPS;   // == grp
      const uint64_t b = (uint64_t)tt * fh::BM + m;
      const bool inb = b < n;
      if (q == 0) PSIM_TS(145);
      const int tileP_cur = tileP_of(tt);
      int64_t ws = 0, s_b = 0, nsteps = 0, clock = 0;
      int kb = 0;
      uint32_t rmin = 0;
      if (inb) {   // prefetch the state and the first queue entries while the head runs
        ws = a.u.st.ws[b]; s_b = a.u.st.s[b]; nsteps = a.e[b] - ws;
        kb = a.u.st.count[b]; clock = a.u.st.clock[b]; rmin = a.u.st.rmin[b];
      }
      const bool active = inb && a.u.step < nsteps;
      QBatch first;
      if (active) load_qbatch(a.u.st, b, kb, first);   // (an L2 prefetch of the rest of the queue here: no gain)
      const int pb = min((kb + 8) >> 3, 14);
      wait_full(yfull + yb, it / fh::UPD_GROUPS);
      if (q == 0) PSIM_TS(146);
      const float* yrow = sY + (yb * 128 + m) * 3;
      const float y0 = yrow[0], y1 = yrow[1], y2 = yrow[2];
      __syncwarp();
      if (lane == 0) mbar_arrive(yempty + yb);
      int pnext = 0, knext = 0;
      if (active) {
        bool stopped = false;
        long long* uts = nullptr;
#ifdef PSIM_TIMING
        if (a.dbg && blockIdx.x == 0 && it < 4 && q == 0 && lane == 0) uts = a.dbg + it * 256 + 160;   // slots 160..172
        {
          const unsigned am = __activemask();
          const int kmx = __reduce_max_sync(am, kb);
          if (uts) uts[15] = kmx;   // slot 175
        }
#endif
        const int knew = update_subtrace_thread(a.u, b, ws, s_b, nsteps, kb, clock, rmin, first, run_head, y0, y1, y2, sHist,
                                                &stopped, uts);
        if (a.u.step + 1 < nsteps && !stopped) {
          pnext = (knew + 8) >> 3;                 // ceil((k+1)/8)
          knext = knew;
          // keep a4 rows >= P_b zero: clear the rows this sub-trace no longer computes
          for (int p = pnext; p < pb; ++p) {
            uint4* dst = reinterpret_cast<uint4*>(a.a4 + (b * 14 + p) * 128);
#pragma unroll
            for (int c = 0; c < 16; ++c) dst[c] = make_uint4(0, 0, 0, 0);
          }
        }
      }
      if (q == 0) PSIM_TS(143);
      // tile-wide scan of pnext: one atomic per tile reserves the block-list range
      int incl = pnext;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
      }
      int wmax = pnext;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) wmax = max(wmax, __shfl_xor_sync(0xffffffffu, wmax, o));
      if (lane == 31) { sPg[q] = incl; sPg[4 + q] = wmax; }
      named_bar_sync(2 + grp, 128);
      int before = 0;
      for (int w2 = 0; w2 < q; ++w2) before += sPg[w2];
      if (m == 0) {
        const int total = sPg[0] + sPg[1] + sPg[2] + sPg[3];
        sPg[8] = total ? (int)atomicAdd(a.next_count, (uint32_t)total) : 0;
        const int ptn = max(max(sPg[4], sPg[5]), max(sPg[6], sPg[7]));
        if (tt < ntiles) a.tileP_next[tt] = (uint8_t)ptn;
        if (a.ptile_sum && tileP_cur > 0) atomicAdd(a.ptile_sum, (unsigned long long)tileP_cur);
      }
      named_bar_sync(2 + grp, 128);
      const uint32_t base = (uint32_t)sPg[8] + (uint32_t)(before + incl - pnext);
      if (q == 0) PSIM_TS(144);
      for (int p = 0; p < pnext; ++p)
        a.blocks_next[base + p] = make_uint4((uint32_t)(b << 4) | (uint32_t)p, (uint32_t)knext, (uint32_t)ws, (uint32_t)clock);
      named_bar_sync(2 + grp, 128);   // sP reused by the next tile
    }
  }
  __syncthreads();
  for (int k = tid; k < 112; k += fh::THREADS)
    if (sHist[k]) atomicAdd(a.u.st.k_hist + k, (unsigned long long)sHist[k]);
  fence_before();
  __syncthreads();
  PSIM_CTA_TS(1, 2, gtimer());
#ifdef PSIM_TIMING
  {
    int nt = 0, pmax = 0;
    for (uint32_t tt = t0; tt < tend; tt += tstep) { ++nt; pmax = max(pmax, tileP_of(tt)); }
    PSIM_CTA_TS(1, 3, (long long)(nt * 256 + pmax));
  }
#endif
  if constexpr (kPair) cluster_sync();   // the peer no longer signals this CTA's barriers
  if (warp == 1) {
    fence_after();
    if constexpr (kPair) tmem_dealloc_2sm(tmem, 512);
    else tmem_dealloc(tmem, 512);
  }
}

// trace rows -> bf16 operand rows: cols 0..46 = attributes (exact: integers < 256),
// cols 47..63 = 0 (time features are inserted by the gather at cols 48..50)
__global__ void trace16_kernel(const uint8_t* __restrict__ trace, int64_t stride, int64_t rows,
                               __nv_bfloat16* __restrict__ out) {
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;   // one 16-B output chunk (6 per row)
  if (t >= rows * 6) return;
  const int64_t r = t / 6;
  const int c = (int)(t - r * 6);
  const uint8_t* src = trace + r * stride;
  uint32_t w[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const int a0 = c * 8 + 2 * q, a1 = a0 + 1;
    const float f0 = a0 < 47 ? (float)src[a0] : 0.f;
    const float f1 = a1 < 47 ? (float)src[a1] : 0.f;
    w[q] = pack_bf16(f0, f1);
  }
  reinterpret_cast<uint4*>(out)[t] = make_uint4(w[0], w[1], w[2], w[3]);
}
void launch_trace16(const uint8_t* trace, int64_t stride, int64_t rows, __nv_bfloat16* out, cudaStream_t st) {
  const int64_t n = rows * 6;
  if (n > 0) trace16_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(trace, stride, rows, out);
}

// one warp per sub-trace: rows [ws + t0, min(e, ws + t1)) of a pinned, device-mapped
// host trace (48-byte rows, contiguous per sub-trace) -> bf16 operand rows.  Lane l
// reads 16-byte segment q = l % 3 of row l / 3 (10 rows, 480 contiguous bytes per
// warp step, 4 steps in flight) and writes output chunks 2q, 2q+1 (+ the zero chunks
// 6, 7 for q = 2).  No shared memory, 128 threads: co-resides with the persistent
// compute kernels, so the copy overlaps the simulation.
__global__ void __launch_bounds__(128) load_chunk16_kernel(const uint8_t* __restrict__ host, int64_t host_first_row,
                                                           int64_t stride, const int64_t* __restrict__ ws,
                                                           const int64_t* __restrict__ e, uint64_t n, int64_t t0,
                                                           int64_t t1, int64_t row_lo, __nv_bfloat16* __restrict__ out,
                                                           uint8_t* __restrict__ mrow) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (gridDim.x * (uint64_t)blockDim.x) >> 5;
  const int rl = lane / 3, q = lane % 3;
  for (uint64_t b = warp; b < n; b += nwarps) {
    const int64_t r0 = ws[b] + t0;
    const int64_t r1 = min(e[b], ws[b] + t1);
#pragma unroll 4
    for (int64_t rb = r0; rb < r1; rb += 10) {   // warp-uniform trip count
      const int64_t r = rb + rl;
      const bool own = lane < 30 && r < r1;
      uint4 v = make_uint4(0, 0, 0, 0);
      if (own) v = *reinterpret_cast<const uint4*>(host + (r - host_first_row) * stride + q * 16);
      // metric code of row r (interval metrics, R20): attributes 7, 8, 14 are in
      // segment 0 (this lane, q == 0), attribute 34 in segment 2 (lane + 2)
      const uint32_t seg2x = __shfl_down_sync(0xffffffffu, v.x, 2);
      if (mrow && own && q == 0) {
        const uint32_t ld = (v.y >> 24) & 0xFFu, stv = v.z & 0xFFu, dl = (v.w >> 16) & 0xFFu;
        const uint32_t l2 = (seg2x >> 16) & 0xFFu;
        const uint32_t mem = ((ld | stv) != 0u && dl == 2u) ? min(l2, 62u) + 1u : 0u;
        mrow[r - row_lo] = (uint8_t)((stv ? 0x80u : 0u) | mem);
      }
      if (own) {
        const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
        uint32_t o[8];
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          const int a0 = q * 16 + 2 * t, a1 = a0 + 1;   // attribute indices (cols 0..46 of the output row)
          const float f0 = a0 < 47 ? (float)((wv[(2 * t) >> 2] >> (((2 * t) & 3) * 8)) & 0xFFu) : 0.f;
          const float f1 = a1 < 47 ? (float)((wv[(2 * t + 1) >> 2] >> (((2 * t + 1) & 3) * 8)) & 0xFFu) : 0.f;
          o[t] = pack_bf16(f0, f1);
        }
        uint4* dst = reinterpret_cast<uint4*>(out + (r - row_lo) * 48);
        dst[2 * q] = make_uint4(o[0], o[1], o[2], o[3]);
        dst[2 * q + 1] = make_uint4(o[4], o[5], o[6], o[7]);
      }
    }
  }
}
void launch_load_chunk16(const uint8_t* host_rows, int64_t host_first_row, int64_t stride, const int64_t* ws,
                         const int64_t* e, uint64_t n, int64_t t0, int64_t t1, int64_t row_lo,
                         __nv_bfloat16* trace16, uint8_t* mrow, cudaStream_t st) {
  uint64_t blocks = (n * 32 + 127) / 128;
  // Loader grid cap (PSIM_LOADER_CTAS, default 64): each loader CTA takes an SM slot the
  // fused kernels need at every kernel boundary, so fewer, longer-lived loader CTAs slow
  // the simulation far less while still streaming faster than it consumes rows --
  // measured on config 3 (2 cohorts): e2e 446 / 476 / 533 / 528 / 500 MIPS with
  // 296 / 32 / 64 / 48 / 128 CTAs (tools/gpu/loaderctas.sh)
  static const uint64_t cap = [] {
    const char* e = getenv("PSIM_LOADER_CTAS");
    return (uint64_t)(e && atoi(e) > 0 ? atoi(e) : 64);
  }();
  if (blocks > cap) blocks = cap;
  if (blocks < 1) blocks = 1;
  load_chunk16_kernel<<<(unsigned)blocks, 128, 0, st>>>(host_rows, host_first_row, stride, ws, e, n, t0, t1, row_lo,
                                                         trace16, mrow);
}

// step-0 block list: every sub-trace has k = 0 -> P = 1
__global__ void fused_init_kernel(uint64_t n, const int64_t* __restrict__ ws, uint4* blocks, uint32_t* count,
                                  uint8_t* tileP, uint32_t* next_count) {
  const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (t < n) blocks[t] = make_uint4((uint32_t)(t << 4), 0u, (uint32_t)ws[t], 0u);   // empty queue, Clock 0
  if (t < (n + 127) / 128) tileP[t] = 1;
  if (t == 0) { *count = (uint32_t)n; *next_count = 0; }
}

// step-0 block list of a pass that starts from existing queues (correction pass):
// one CTA of 128 threads per 128-sub-trace tile, P_b = ceil((k+1)/8) for active b
__global__ void __launch_bounds__(128) fused_init_state_kernel(uint64_t n, const int32_t* __restrict__ count,
                                                                const int64_t* __restrict__ clock,
                                                                const int64_t* __restrict__ ws,
                                                                const int64_t* __restrict__ e, uint4* blocks,
                                                                uint32_t* nblocks, uint8_t* tileP) {
  __shared__ int sSum[4], sMax[4], sBase;
  const int m = threadIdx.x, lane = m & 31, w = m >> 5;
  const uint64_t b = (uint64_t)blockIdx.x * 128 + m;
  int P = 0;
  if (b < n && e[b] > ws[b]) P = min((count[b] + 8) >> 3, 14);
  int incl = P;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  int wmax = P;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) wmax = max(wmax, __shfl_xor_sync(0xffffffffu, wmax, o));
  if (lane == 31) { sSum[w] = incl; sMax[w] = wmax; }
  __syncthreads();
  if (m == 0) {
    const int tot = sSum[0] + sSum[1] + sSum[2] + sSum[3];
    sBase = tot ? (int)atomicAdd(nblocks, (uint32_t)tot) : 0;
    tileP[blockIdx.x] = (uint8_t)max(max(sMax[0], sMax[1]), max(sMax[2], sMax[3]));
  }
  __syncthreads();
  int before = 0;
  for (int q = 0; q < w; ++q) before += sSum[q];
  const uint32_t base = (uint32_t)sBase + (uint32_t)(before + incl - P);
  for (int p = 0; p < P; ++p)
    blocks[base + p] = make_uint4((uint32_t)(b << 4) | (uint32_t)p, (uint32_t)count[b], (uint32_t)ws[b], (uint32_t)clock[b]);
}

void launch_fused_init_from_state(FusedC3& f, const int32_t* count, const int64_t* clock, const int64_t* ws, const int64_t* e,
                                  uint64_t n, cudaStream_t st) {
  cudaMemsetAsync(f.count, 0, 8, st);
  const uint64_t nt = (n + 127) / 128;
  if (nt) fused_init_state_kernel<<<(unsigned)nt, 128, 0, st>>>(n, count, clock, ws, e, f.blocks, f.count, f.tileP[0]);
}

// ---------------------------------------------------------------- host side
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_fn2() {
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
static bool map2d(CUtensorMap* m, const void* ptr, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  EncodeTiledFn fn = encode_fn2();
  if (!fn) return false;
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {64, box_rows};
  cuuint32_t es[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

// launch with programmatic stream serialization (PDL): the kernel may start while the
// previous kernel on the stream drains; it calls griddepcontrol.wait before touching
// anything that kernel produced
template <typename... KArgs, typename... Args>
static void launch_pdl(void (*kern)(KArgs...), int grid, int threads, int smem, cudaStream_t st, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3((unsigned)threads);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  // PSIM_NO_PDL=1 (experiments): plain stream-ordered launches; griddepcontrol.wait is then a no-op
  static const bool no_pdl = [] { const char* e = getenv("PSIM_NO_PDL"); return e && atoi(e) != 0; }();
  cfg.attrs = attr;
  cfg.numAttrs = no_pdl ? 0 : 1;
  cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

void launch_fused_init(FusedC3& f, const int64_t* ws, uint64_t n, cudaStream_t st) {
  const uint64_t th = n > 1 ? n : 1;
  fused_init_kernel<<<(unsigned)((th + 255) / 256), 256, 0, st>>>(n, ws, f.blocks, f.count + 0, f.tileP[0], f.count + 1);
}

// PSIM_DEBUG_TIMING=<step>: CTA 0 of conv_stack records clock64() at every
// pipeline event of its first 4 tiles of that step (dumped to
// $PSIM_DEBUG_TIMING_OUT by fused_dump_debug).  Off by default.
static long long* g_dbg = nullptr;
constexpr int kDbgWords = 1024 + 2 * 160 * 4;   // CTA-0 slots, then per-CTA spans
static int64_t g_dbg_step = -2;
static long long* debug_buffer(int64_t step) {
  if (g_dbg_step == -2) {
    const char* e = getenv("PSIM_DEBUG_TIMING");
    g_dbg_step = e ? atoll(e) : -1;
    if (g_dbg_step >= 0) { cudaMalloc(&g_dbg, 2 * kDbgWords * 8); cudaMemset(g_dbg, 0, 2 * kDbgWords * 8); }
  }
  if (g_dbg_step < 0) return nullptr;
  if (step == g_dbg_step) return g_dbg;
  return step == g_dbg_step + 1 ? g_dbg + kDbgWords : nullptr;   // the next step: per-CTA spans
}
void fused_dump_debug() {
  const char* out = getenv("PSIM_DEBUG_TIMING_OUT");
  if (!g_dbg || !out) return;
  static long long h[2 * kDbgWords];
  cudaMemcpy(h, g_dbg, sizeof h, cudaMemcpyDeviceToHost);
  FILE* f = fopen(out, "w");
  if (!f) return;
  for (int t = 0; t < 4; ++t)
    for (int sidx = 0; sidx < 256; ++sidx)
      if (h[t * 256 + sidx]) fprintf(f, "%d %d %lld\n", t, sidx, h[t * 256 + sidx]);
  for (int st = 0; st < 2; ++st)   // per-CTA spans: "cta <kernel> <cta> <entry> <after wait> <end> <tiles>"
    for (int k = 0; k < 2; ++k)     // kernel 0/1 = conv_stack / fc1_head of the step, 2/3 of the next step
      for (int c = 0; c < 160; ++c) {
        const long long* r = h + st * kDbgWords + 1024 + (k * 160 + c) * 4;
        if (r[0]) fprintf(f, "cta %d %d %lld %lld %lld %lld\n", k + 2 * st, c, r[0], r[1], r[2], r[3]);
      }
  fclose(f);
}

void launch_conv_stack(FusedC3& f, const GatherArgs& g, int64_t step, uint64_t n, cudaStream_t st) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(conv_stack_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, cs::SMEM);
    attr = true;
  }
  ConvArgs a;
  a.blocks = f.blocks;
  a.nblocks = f.count + (step & 1);
  a.next_count = f.count + ((step + 1) & 1);
  a.trace16 = f.trace16; a.row_lo = g.row_lo;
  a.zero_row = f.zero_row;
  a.ws = g.ws; a.clock = g.clock; a.count = g.count;
  a.q = g.q;
  a.step = step;
  a.qn = g.qn ? g.qn : g.n;
  // L2 policy of the gathered trace rows: a sub-trace's context rows are re-read every step while
  // they stay in its queue (~25 steps).  Up to 16384 sub-traces per launch the live window
  // (~25 rows x 96 B each, <= 40 MB) fits L2 beside the queue and a4: evict_last (+1 % at the
  // G = 4 / 8 slices); at config 3 on one GPU (157 MB per step) the rows would push out the
  // queue entries and a4 rows reused within the step: evict_first (evict_last: -4 %, any
  // evict_last fraction 0.25..0.75: -3..-4 %, evict_normal: -24 %; tools/gpu/abe.sh, frac.sh).
  // PSIM_ROW_POLICY=first|last overrides (experiments).
  static const int row_policy = [] {
    const char* e = getenv("PSIM_ROW_POLICY");
    return !e ? -1 : (e[0] == 'l' ? 1 : 0);
  }();
  a.rows_keep = row_policy >= 0 ? row_policy : (n <= 16384 ? 1 : 0);
  a.w1 = f.w1; a.w2 = f.w2; a.w3 = f.w3;
  a.b1 = f.b1; a.b2 = f.b2; a.b3 = f.b3;
  a.a4 = f.a4;
  a.dbg = debug_buffer(step);
  // the block count is only known on the device: launch one persistent CTA per SM
  // (n*14 blocks at most); CTAs with no tile exit after setup.
  const uint64_t max_tiles = (n * 14 + cs::TILE - 1) / cs::TILE;
  const int grid = (int)std::min<uint64_t>(max_tiles, (uint64_t)(f.grid_cap > 0 ? f.grid_cap : sm_count()));
  launch_pdl(conv_stack_kernel, grid, cs::THREADS, cs::SMEM, st, a, f.mapW1, f.mapW2, f.mapW3, f.mapX);
}

void launch_fc1_head(FusedC3& f, const UpdateArgs& u, const int64_t* e, int64_t step, bool force_predict,
                     cudaStream_t st) {
  static bool attr = false;
  static int max_pairs = 0;
  if (!attr) {
    cudaFuncSetAttribute(fc1_head_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, fh::SMEM);
    cudaFuncSetAttribute(fc1_head_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, fh::SMEM);
    // co-resident 2-CTA clusters of the pair kernel (SM pairs within a GPC)
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * (unsigned)sm_count());
    cfg.blockDim = dim3(fh::THREADS);
    cfg.dynamicSmemBytes = fh::SMEM;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (cudaOccupancyMaxActiveClusters(&max_pairs, fc1_head_kernel<true>, &cfg) != cudaSuccess) {
      max_pairs = 0;
      cudaGetLastError();
    }
    attr = true;
  }
  HeadArgs a;
  a.u = u;
  a.e = e;
  a.tileP = f.tileP[step & 1];
  a.tileP_next = f.tileP[(step + 1) & 1];
  a.blocks_next = f.blocks;   // conv_stack of this step has finished with the list
  a.next_count = f.count + ((step + 1) & 1);
  a.a4 = f.a4;
  a.T = f.T; a.w2 = f.head_w; a.b2 = f.head_b;
  a.force_predict = force_predict ? 1 : 0;
  a.dbg = debug_buffer(step);
  a.ptile_sum = u.st.ptile_sum;
  const uint64_t ntiles = (u.st.n + fh::BM - 1) / fh::BM;
  const int cap = f.grid_cap > 0 ? f.grid_cap : sm_count();
  // pair mode (psim_opts flag PSIM_FC1_PAIR): fc1 on 2-SM MMAs, two tiles per CTA pair
  if (f.pair && max_pairs > 0 && ntiles >= 2) {
    const uint64_t pairs = std::min<uint64_t>(std::min<uint64_t>((ntiles + 1) / 2, (uint64_t)max_pairs),
                                              (uint64_t)std::max(1, cap / 2));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(2 * pairs));
    cfg.blockDim = dim3(fh::THREADS);
    cfg.dynamicSmemBytes = fh::SMEM;
    cfg.stream = st;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    at[1].id = cudaLaunchAttributeClusterDimension;
    at[1].val.clusterDim.x = 2; at[1].val.clusterDim.y = 1; at[1].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 2;
    cudaLaunchKernelEx(&cfg, fc1_head_kernel<true>, f.mapA, f.mapB128, a);
    return;
  }
  const int grid = (int)std::min<uint64_t>(ntiles, (uint64_t)cap);
  launch_pdl(fc1_head_kernel<false>, grid, fh::THREADS, fh::SMEM, st, f.mapA, f.mapB, a);
}

bool fused_make_weight_maps(FusedC3& f) {
  return map2d(&f.mapW1, f.w1p, 64, 128, 64) && map2d(&f.mapW2, f.w2, 128, 128, 128) &&
         map2d(&f.mapW3, f.w3, 128, 256, 128);
}

bool fused_make_trace_map(FusedC3& f, uint64_t rows) {
  // padding rows of the gathered input (rows R > k) use a row index past the
  // tensor: the TMA zero-fills out-of-bounds rows without reading memory.  (Pointing them at
  // one all-zero trace16 row made that 96-B line an L2 hot spot -- ~230k reads per step at
  // config 3, all served by one L2 slice: conv_stack 131 -> 114 ms per run without it.)
  f.zero_row = kPadRow;
  // 96-B rows (48 bf16: 47 attributes + 0); a 48-column box lands in chunks 0..5 of the
  // 128-B SWIZZLE_128B operand rows, chunks 6 (time features) and 7 (zero) are the gather's
  EncodeTiledFn fn = encode_fn2();
  if (!fn) return false;
  cuuint64_t dims[2] = {48, rows + 1};
  cuuint64_t strides[1] = {96};
  cuuint32_t box[2] = {48, 1};
  cuuint32_t es[2] = {1, 1};
  return fn(&f.mapX, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, f.trace16, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool fused_make_maps(FusedC3& f, uint64_t n) {
  return map2d(&f.mapA, f.a4, n, 14 * 128, fh::BM) && map2d(&f.mapB, f.wfc1, 256, 14 * 128, fh::BN) &&
         map2d(&f.mapB128, f.wfc1, 256, 14 * 128, fh::BN / 2);   // pair mode: each CTA's 128 N-rows
}

}  // namespace psim
