// internal.h -- product-side declarations shared by the libpsim translation
// units.  Nothing here is visible through the C ABI (include/psim.h) and
// nothing here is shared with oracle/.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "psim.h"

namespace psim {

constexpr int kRows = 112;      // 111 instruction rows + 1 zero row (R11)
constexpr int kFeat = 50;       // 3 time features + 47 attributes (R1)
constexpr int kFeatPad = 64;    // device row width: features padded with zeros to 64
constexpr int kQStride = 112;   // queue entries reserved per sub-trace (cap <= 110, +1 push)
constexpr int kLatMax = 4095;   // R7
constexpr int kTimeMax = 65535; // R7
constexpr uint32_t kPadRow = 0x7FFF0000u;   // gather4 row past any trace16 tensor: TMA zero fill

// One GEMM layer of the lowered CNN: out[M][N] = act(A[M][K] . W[N][K]^T + b[N]).
// Convolutions with k = s = 2 read A as the row-pair reshape of the previous
// activation [B*pos][C] -> [B*pos/2][2C] (K index = tap*C + channel), so no
// im2col is ever materialised.
struct GemmLayer {
  int K = 0, N = 0;        // reduction length, output channels
  int rows_per_item = 0;   // output positions per sub-trace (M = B * rows_per_item)
  bool relu = true;
  int taps = 1;            // 3: stride-1 k3 conv over the pad-row layout (RB7)
  bool block_begin = false;   // this layer's input is a residual block input x
  bool add_block_input = false;   // y = relu(x + conv(...)) with x the block input (RB7, R11)
  int pad_period = 0;      // output rows r with r % P in {0, P-1} are zero pad rows
  void* w = nullptr;       // device [N][K], fp32 or bf16 (K-major)
  float* bias = nullptr;   // device [N] fp32
  void* w_tc = nullptr;    // device weights pre-tiled for the tcgen05 kernel (bf16)
  // 2:4 structured sparsity (PSIM_SPARSE24, R22): compressed weights [sp_mh*128][K/2]
  // bf16 and the tcgen05.mma.sp metadata words [sp_mh * K/32][128] (gemm_sp.cu)
  void* w_sp = nullptr;
  uint32_t* meta = nullptr;
  int sp_mh = 0;
};

struct Model {
  uint32_t arch = 0;
  uint32_t precision = PSIM_FP32;
  std::vector<GemmLayer> layers;  // tensor-core-able layers (all but the head)
  float* head_w = nullptr;        // fc2 [3][256] fp32
  float* head_b = nullptr;        // fc2 bias [3]
  int head_in = 0;                // 256
  int item_rows = kRows;          // device input rows per sub-trace (RB7: 116 = 2 + 112 + 2 pad rows)
  int row_off = 0;                // first input row inside an item (RB7: 2)
  bool loaded = false;
};

// Per-rank lockstep state: structure-of-arrays in HBM, sub-trace-major.
struct SimState {
  uint64_t n = 0;               // local sub-traces
  uint64_t qn = 0;              // queue entry stride (0: n); a cohort's view of a larger state keeps
                                // the full state's stride (its pointers are offset by its first sub-trace)
  int64_t* ws = nullptr;        // [n] first row (warm-up start)
  int64_t* s = nullptr;         // [n] first real row
  int64_t* e = nullptr;         // [n] end row
  int64_t* clock = nullptr;     // [n] Clock
  int64_t* bnd = nullptr;       // [n] Clock at the end of warm-up
  int64_t* cycles = nullptr;    // [n] Clock_end - bnd
  int32_t* count = nullptr;     // [n] live context entries
  uint32_t* rmin = nullptr;     // [n] low 32 bits of the smallest retire Clock of the live entries
                                // (valid when count > 0; maintained by the thread-per-sub-trace update)
  // queue entries are ENTRY-MAJOR: entry e of sub-trace b at [e * n + b], so the
  // threads of a warp (consecutive sub-traces) touch consecutive 16-byte words, and
  // one entry is one 16-byte load (one DRAM sector) for the gather
  uint4* q = nullptr;           // [kQStride][n] {global row index (fetch order), low 32 bits of
                                //  the fetch Clock, c | s << 16, bit 0: store (metrics, R20)}
  unsigned long long* k_hist = nullptr;   // [112]
  unsigned long long* stalls = nullptr;   // [1]
  unsigned long long* ptile_sum = nullptr;   // [1] fused fc1: sum of P_tile over tiles and steps
  long long* total = nullptr;             // [1] local sum of cycles (NCCL send/recv buffer)
};

struct Buffers {
  size_t bytes = 0;
  void* x = nullptr;            // gathered inputs [n][112][64] (fp32 or bf16)
  void* act[8] = {};            // per-layer activations
  float* h = nullptr;           // fc1 output [n][256] fp32
  float* y = nullptr;           // head output [n][3] fp32
};

// ----------------------------- kernels ---------------------------------
struct GatherArgs {
  const uint8_t* trace;      // device rows, row r at trace + (r - row_lo) * stride
  int64_t row_lo;
  int64_t stride;
  const int64_t* ws;
  const int64_t* e;
  const int64_t* clock;
  const int32_t* count;
  const uint4* q;
  uint64_t n;
  int64_t step;
  int item_rows = kRows;     // rows per sub-trace in x (RB7: 116)
  uint64_t qn = 0;           // queue entry stride (0: n)
  int row_off = 0;           // row of the current instruction inside an item (RB7: 2)
};
void launch_gather_f32(const GatherArgs& a, float* x, cudaStream_t st);
void launch_gather_bf16(const GatherArgs& a, __nv_bfloat16* x, cudaStream_t st);

struct UpdateArgs {
  SimState st;
  int64_t row_lo;
  int64_t step;
  int cap;
  const float* y;            // [n][3] raw CNN outputs (CNN mode, or forced+predict) or nullptr
  const uint16_t* forced;    // [rows][3] teacher-forced latencies (row - row_lo) or nullptr
  uint16_t* rec_lat;         // [rows][3] or nullptr (PSIM_RECORD_ROWS)
  int32_t* rec_k;            // [rows] or nullptr
  int64_t* rec_clock;        // [rows] or nullptr
  float* rec_y = nullptr;    // [rows][3] raw fp32 CNN outputs y of the step that predicted row r
                             // (PSIM_RECORD_ROWS with a CNN, parity stage S2 of the hot path)
  // post-error correction (R19), entry-major [t][n]:
  uint8_t* k1_rec = nullptr;   // first pass: context count at real row s_b + t, t < limit
  uint32_t* c1_rec = nullptr;  // first pass: Clock - bnd after real row s_b + t
  int limit = 0;
  const uint8_t* kref = nullptr;   // correction pass: stop corrector b when its count equals
                                   // kref[(step+1) * n + b + 1] (cycles -> st.cycles, st.e[b] = row + 1)
  // interval metrics (R20).  mrow tags pushed entries
  // (queue word .w bit 0 = store) whenever it is set; macc/mout nullptr = no metrics.
  const uint8_t* mrow = nullptr;   // [rows] (row - row_lo): bit 7 store, bits 0..6 0 or 1 + log2(bytes)
                                   // of a memory-served load/store
  uint4* macc = nullptr;           // [n] {retired, retired stores, Clock lo at segment start, 0}
  unsigned long long* mout = nullptr;   // [n_int][4] cycles, retired, retired stores, mem bytes
  int64_t interval = 0;
};
void launch_update(const UpdateArgs& a, cudaStream_t st);
// per-row metric codes (UpdateArgs::mrow) from device-accessible uint8 trace rows
void launch_mrow(const uint8_t* trace, int64_t stride, int64_t rows, uint8_t* out, cudaStream_t st);

// Post-error correction state (per rank, local sub-traces; R19).  The
// correction pass reuses the lockstep kernels on a SimState whose ws/s/e/bnd/cycles
// point here: corrector b re-simulates rows [ws[b], e[b]) of sub-trace b+1 from
// its own final state.
struct Pec {
  int limit = 0;
  uint64_t cap = 0;             // sub-traces allocated
  uint8_t* k1 = nullptr;        // [limit][n]
  uint32_t* c1 = nullptr;       // [limit][n]
  int64_t *ws = nullptr, *s = nullptr, *e = nullptr, *bnd = nullptr, *cyc = nullptr;   // [n]
  int64_t* cycles1 = nullptr;   // [n] first-pass cycles
  int32_t* len = nullptr;       // [n] rows of sub-trace b re-simulated by b-1
  unsigned long long* corrected = nullptr;   // [1]
  uint16_t* rec_lat = nullptr;  // [rows][3] re-simulated (f,c,s) (PSIM_RECORD_ROWS)
  int32_t* rec_k = nullptr;     // [rows] re-simulated k, -1 elsewhere
  size_t rec_cap = 0;
};
// set up the correction pass from the first pass's final state
void launch_pec_init(const SimState& s, const Pec& p, cudaStream_t st);
// cycles[b+1] = cycles1[b+1] - c1[len-1][b+1] + cyc[b] for corrected sub-traces
void launch_pec_apply(const SimState& s, const Pec& p, cudaStream_t st);
void launch_state_init(const SimState& s, cudaStream_t st);
void launch_reduce_cycles(const SimState& s, cudaStream_t st);

// head: y[b][o] = sum_i h[b][i] * w[o][i] + bias[o] (fp32, o < 3)
void launch_head(const float* h, const float* w, const float* b, int in, float* y, uint64_t n,
                 cudaStream_t st);

// SIMT GEMM (CUDA cores): C = act(A . W^T + b); A [M][K], W [N][K]
void launch_gemm_simt_f32(const float* A, const float* W, const float* b, float* C, int64_t M,
                          int N, int K, bool relu, cudaStream_t st);
void launch_gemm_simt_bf16(const __nv_bfloat16* A, const __nv_bfloat16* W, const float* b,
                           void* C, bool c_is_f32, int64_t M, int N, int K, bool relu,
                           cudaStream_t st);

// tcgen05 GEMM (tensor cores, sm_100a): bf16 A/W, fp32 accumulate in TMEM.
// Returns false if the shape is not supported by the tensor-core kernel.
bool gemm_tc_supported(int N, int K);
// taps = 3: stride-1 k3 convolution over a pad-row layout (A is [M][K/3], tap t reads
// row m + t - 1, zero outside [0, M)); resid: bf16 [M][N] added before the ReLU;
// pad_period > 0: output rows with row % P in {0, P-1} are written as zero.
void launch_gemm_tc(const __nv_bfloat16* A, const void* Wtc, const float* b, void* C,
                    bool c_is_f32, int64_t M, int N, int K, bool relu, cudaStream_t st, int taps = 1,
                    const __nv_bfloat16* resid = nullptr, int pad_period = 0);
// 2:4 sparse layer (gemm_sp.cu): W bf16 [N][K] (host, RNE bits) -> compressed [mh*128][K/2]
// and metadata words; 0 on success, -1 unsupported shape, -2 not 2:4 sparse along K
int sparse24_compress(const uint16_t* W, int N, int K, std::vector<uint16_t>* wc, std::vector<uint32_t>* meta,
                      int* mh);
// C[M][N] = act(X[M][K] . W^T + b) with W 2:4-sparse (compressed + metadata from sparse24_compress)
void launch_gemm_sp(const __nv_bfloat16* X, const __nv_bfloat16* Wc, const uint32_t* meta, int mh, const float* b,
                    void* C, bool c_is_f32, int64_t M, int N, int K, bool relu, cudaStream_t st);
// RB7 gather + stem convolution fused on tcgen05 (rb7_stem.cu): the step's inputs built straight
// into the stem's A operand; y = the stem output in the pad-row layout [n * 58][64] bf16
void launch_rb7_stem(const GatherArgs& g, const __nv_bfloat16* w, const float* bias, __nv_bfloat16* y,
                     cudaStream_t st);
// RB7 residual block fused on tcgen05 (resblock.cu): y = relu(x + conv_b(relu(conv_a(x)))) over the
// pad-row layout [M = n * 58][64] bf16; wa / wb: [64][192] bf16 (K = tap * 64 + channel)
void launch_resblock(const __nv_bfloat16* x, const __nv_bfloat16* wa, const float* ba, const __nv_bfloat16* wb,
                     const float* bb, __nv_bfloat16* y, int64_t M, cudaStream_t st);
// Pre-tile a [N][K] bf16 weight for the tensor-core kernel (device -> device).
void* pretile_weight_tc(const __nv_bfloat16* W, int N, int K, cudaStream_t st);

// ---- fused padding-aware C3 step (fused_c3.cu), bf16 tensor cores ----
struct FusedC3 {
  bool ready = false;                 // model side prepared (weights, T table)
  const __nv_bfloat16* w1 = nullptr;  // aliases of the model's layer weights [N][K]
  const __nv_bfloat16* w2 = nullptr;
  const __nv_bfloat16* w3 = nullptr;
  const __nv_bfloat16* wfc1 = nullptr;
  const float *b1 = nullptr, *b2 = nullptr, *b3 = nullptr;
  float* T = nullptr;                 // [15][256] constant fc1 table (owned)
  __nv_bfloat16* w1p = nullptr;       // conv1 weight [64][128] in the fused row layout (owned):
                                      // per tap h: cols 0..46 attributes, 48..50 time features
  __nv_bfloat16* trace16 = nullptr;   // per-run bf16 copy of the rank's trace rows [rows + 1][48] (owned)
  size_t trace16_cap = 0;
  const float* head_w = nullptr;      // fc2 [3][256]
  const float* head_b = nullptr;
  // per-run buffers (owned), sized for cap_n sub-traces
  uint64_t cap_n = 0;
  uint4* blocks = nullptr;            // [n*14] block entries {b<<4|p, k_b, ws_b lo, Clock_b lo}: the sub-trace
                                      // state the gather needs travels with the block id (one 16-B read)
  uint32_t* count = nullptr;          // [2] block counts by step parity
  uint8_t* tileP[2] = {nullptr, nullptr};   // [ceil(n/128)] P_tile by step parity
  __nv_bfloat16* a4 = nullptr;        // [n][14][128] conv3 outputs
  CUtensorMap mapA, mapB;             // TMA maps of a4 [n][1792] and wfc1 [256][1792]
  CUtensorMap mapB128;                // wfc1 with a 128-row box (fc1_head pair mode)
  bool pair = false;                  // fc1_head on 2-SM MMAs (PSIM_FC1_PAIR)
  int grid_cap = 0;                   // max CTAs of the persistent fused kernels (0: one per SM);
                                      // cohorts with disjoint SM shares run side by side
  CUtensorMap mapW1, mapW2, mapW3;    // TMA maps of the resident conv weights (SWIZZLE_128B)
  CUtensorMap mapX;                   // TMA gather4 map of trace16 [rows + 1][48] (box 48 x 1, SWIZZLE_128B)
  uint32_t zero_row = 0;              // gather row index of the input's padding rows (kPadRow: out of
                                      // bounds of mapX, zero-filled by the TMA)
};
void launch_fused_init(FusedC3& f, const int64_t* ws, uint64_t n, cudaStream_t st);
// block list / P_tile of step 0 of a pass whose sub-traces start from a non-empty
// queue (the correction pass): P_b = ceil((count+1)/8) for active b (ws < e)
void launch_fused_init_from_state(FusedC3& f, const int32_t* count, const int64_t* clock, const int64_t* ws, const int64_t* e,
                                  uint64_t n, cudaStream_t st);
// trace rows (uint8 attributes) -> bf16 operand rows of the fused conv1 layout
void launch_trace16(const uint8_t* trace, int64_t stride, int64_t rows, __nv_bfloat16* out, cudaStream_t st);
// streamed variant for pinned host traces: the rows sub-trace b touches in lockstep
// steps [t0, t1) are read over PCIe (zero-copy) and written as bf16 operand rows
void launch_load_chunk16(const uint8_t* host_rows, int64_t host_first_row, int64_t stride, const int64_t* ws,
                         const int64_t* e, uint64_t n, int64_t t0, int64_t t1, int64_t row_lo,
                         __nv_bfloat16* trace16, uint8_t* mrow, cudaStream_t st);
void launch_conv_stack(FusedC3& f, const GatherArgs& g, int64_t step, uint64_t n, cudaStream_t st);
void launch_fc1_head(FusedC3& f, const UpdateArgs& u, const int64_t* e, int64_t step, bool force_predict,
                     cudaStream_t st);
bool fused_make_maps(FusedC3& f, uint64_t n);
int sm_count();   // SMs of the current device
bool fused_make_weight_maps(FusedC3& f);
// gather4 map of f.trace16 with rows + 1 rows (the last one zero); sets f.zero_row = kPadRow
bool fused_make_trace_map(FusedC3& f, uint64_t rows);
void fused_dump_debug();

// pad/convert the caller's [B][112][50] fp32 inputs (psim_cnn_forward)
void launch_pad_inputs(const float* X, uint64_t B, void* x, bool bf16, cudaStream_t st, int item_rows = kRows,
                       int row_off = 0);

}  // namespace psim
