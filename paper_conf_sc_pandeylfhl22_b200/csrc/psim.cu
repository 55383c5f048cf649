// psim.cu -- host runtime behind the C ABI (include/psim.h): context and
// state machine, partitioner, trace loader, model repacking, the lockstep
// step loop and the end-of-run NCCL reduction.
//
// Step t (PAPER.md:91-107 per instruction, lockstep over sub-traces :179):
//   gather -> conv/fc GEMMs -> head (fc2) -> update (round, Clock, retire, push)
// After the last step: reduce cycles, ncclAllReduce(int64, sum).
#include <dlfcn.h>
#include <nccl.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <mutex>
#include <string>
#include <vector>

#include "internal.h"

using namespace psim;

namespace {
// ---- NCCL, resolved at run time (the library never links a specific NCCL) ----
struct NcclApi {
  bool tried = false, ok = false;
  ncclResult_t (*commInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*allReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*commDestroy)(ncclComm_t) = nullptr;
  const char* (*errStr)(ncclResult_t) = nullptr;
  ncclResult_t (*getUniqueId)(ncclUniqueId*) = nullptr;
};
NcclApi g_nccl;
std::mutex g_nccl_mu;

bool load_nccl() {
  std::lock_guard<std::mutex> lk(g_nccl_mu);
  if (g_nccl.tried) return g_nccl.ok;
  g_nccl.tried = true;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
  if (!h) return false;
  g_nccl.commInitRank = (decltype(g_nccl.commInitRank))dlsym(h, "ncclCommInitRank");
  g_nccl.allReduce = (decltype(g_nccl.allReduce))dlsym(h, "ncclAllReduce");
  g_nccl.commDestroy = (decltype(g_nccl.commDestroy))dlsym(h, "ncclCommDestroy");
  g_nccl.errStr = (decltype(g_nccl.errStr))dlsym(h, "ncclGetErrorString");
  g_nccl.getUniqueId = (decltype(g_nccl.getUniqueId))dlsym(h, "ncclGetUniqueId");
  g_nccl.ok = g_nccl.commInitRank && g_nccl.allReduce && g_nccl.commDestroy && g_nccl.errStr && g_nccl.getUniqueId;
  return g_nccl.ok;
}

inline uint16_t f32_to_bf16_rne(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  if ((u & 0x7f800000u) == 0x7f800000u && (u & 0x7fffffu)) return (uint16_t)((u >> 16) | 0x40);  // NaN
  u += 0x7fffu + ((u >> 16) & 1u);
  return (uint16_t)(u >> 16);
}
}  // namespace

// Per-kernel-class device timing with CUDA events on the launch stream
// (PSIM_PROFILE); launch counting is always on (psim_stats.gpu_launches).
struct Prof {
  bool on = false;
  bool sample = true;          // time this launch (lockstep kernels: every kEvery-th step only,
                               // so the events do not serialise the PDL overlap of the others)
  static constexpr int kEvery = 16;
  uint64_t timed[PSIM_KC_COUNT] = {};
  cudaStream_t st = nullptr;
  std::vector<cudaEvent_t> pool;
  size_t used = 0;
  std::vector<std::pair<int, size_t>> marks;   // (class, index of the start event)
  size_t open_idx = 0;
  uint64_t launches[PSIM_KC_COUNT] = {};
  void reset(bool enable, cudaStream_t s) {
    on = enable; st = s; used = 0; marks.clear(); sample = true;
    for (auto& l : launches) l = 0;
    for (auto& l : timed) l = 0;
  }
  cudaEvent_t next() {
    if (used == pool.size()) { cudaEvent_t e; cudaEventCreate(&e); pool.push_back(e); }
    return pool[used++];
  }
  void count(int cls) { launches[cls]++; }
  void begin(int cls) {
    launches[cls]++;
    if (!on || !sample) return;
    timed[cls]++;
    open_idx = used;
    cudaEventRecord(next(), st);
  }
  void end(int cls) {
    if (!on || !sample) return;
    cudaEventRecord(next(), st);
    marks.push_back({cls, open_idx});
  }
  // per-class device time, scaled from the timed launches to all launches of the class
  void collect(double* ms) {
    for (int c = 0; c < PSIM_KC_COUNT; ++c) ms[c] = 0;
    for (auto& m : marks) {
      float t = 0;
      cudaEventElapsedTime(&t, pool[m.second], pool[m.second + 1]);
      ms[m.first] += t;
    }
    for (int c = 0; c < PSIM_KC_COUNT; ++c)
      if (timed[c]) ms[c] *= (double)launches[c] / (double)timed[c];
  }
  ~Prof() { for (auto e : pool) cudaEventDestroy(e); }
};

// A cohort: a contiguous block of this rank's sub-traces simulated on its own stream
// with its own fused-path block lists, so the kernels of different cohorts overlap on
// the device (one cohort's conv_stack fills the SMs another cohort's fc1_head tail and
// the kernel boundaries leave idle).  Sub-traces are independent, so the
// results are bit-identical to one cohort.
struct Cohort {
  FusedC3 fz;                 // shared model/trace fields + this cohort's per-run buffers
  cudaStream_t st = nullptr;
  cudaEvent_t ev = nullptr;
  uint64_t b0 = 0, n = 0, cap = 0;
  uint4* blocks = nullptr;
  uint32_t* count = nullptr;
  uint8_t* tileP[2] = {nullptr, nullptr};
};

struct psim_ctx {
  psim_opts opts{};
  Prof prof;
  FusedC3 fused;
  std::vector<Cohort> cohorts;
  int cap = 110;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  std::string err;
  // trace
  bool have_trace = false;
  const uint8_t* trace = nullptr;
  uint64_t L = 0, first_row = 0, n_rows = 0, stride = 48;
  int trace_mode = 0;
  uint8_t* d_trace = nullptr;
  size_t d_trace_cap = 0;
  const uint8_t* trace_devptr = nullptr;   // device-accessible address of a pinned host trace
  cudaStream_t ld_stream = nullptr;        // trace streaming (pinned host traces, fused path)
  std::vector<cudaEvent_t> ld_events;
  // partition
  bool partitioned = false;
  uint64_t N = 0, W = 0, j0 = 0, j1 = 0;
  int64_t row_lo = 0, row_hi = 0, steps = 0;
  std::vector<int64_t> h_ws, h_s, h_e;
  // model / forcing
  Model model;
  std::vector<uint16_t> forced;
  uint16_t* d_forced = nullptr;
  size_t d_forced_cap = 0;
  // state
  SimState st{};
  uint64_t st_cap = 0;
  Buffers buf{};
  uint64_t buf_n = 0;
  uint16_t* rec_lat = nullptr;
  int32_t* rec_k = nullptr;
  int64_t* rec_clock = nullptr;
  float* rec_y = nullptr;       // [rows][3] raw CNN outputs (PSIM_RECORD_ROWS with a CNN)
  size_t rec_y_cap = 0;
  bool rec_y_valid = false;
  size_t rec_cap = 0;
  Pec pec;                 // post-error correction (opts.correction_limit > 0)
  bool pec_done = false;
  // interval metrics (opts.interval > 0, R20)
  uint8_t* mrow = nullptr;             // [rows] per-row metric codes
  size_t mrow_cap = 0;
  uint4* macc = nullptr;               // [n] per-sub-trace segment accumulators
  uint64_t macc_cap = 0;
  unsigned long long* mout = nullptr;  // [n_int][4] global intervals
  uint64_t mout_cap = 0, n_int = 0;
  bool metrics_done = false;
  // results
  bool done = false;
  int64_t total = 0;
  psim_stats stats{};
  ncclComm_t comm = nullptr;
  cudaEvent_t ev[4] = {};
};

#define FAIL(code, ...)                                   \
  do {                                                    \
    char _b[512];                                         \
    snprintf(_b, sizeof _b, __VA_ARGS__);                 \
    ctx->err = _b;                                        \
    return code;                                          \
  } while (0)
#define CK(x)                                                                              \
  do {                                                                                     \
    cudaError_t _e = (x);                                                                  \
    if (_e != cudaSuccess) FAIL(_e == cudaErrorMemoryAllocation ? PSIM_ERR_OOM : PSIM_ERR_CUDA, \
                                "%s failed: %s (%s:%d)", #x, cudaGetErrorString(_e), __FILE__, __LINE__); \
  } while (0)

static void dfree(void* p) {
  if (p) cudaFree(p);
}

extern "C" {

const char* psim_version(void) {
  return "psim 0.1 (sm_100a; gather/update warp-per-sub-trace, GEMM: tcgen05+TMA bf16, SIMT fp32)";
}

int psim_create(const psim_opts* opts, psim_ctx** out) {
  if (!out) return PSIM_ERR_ARG;
  *out = nullptr;
  if (!opts) return PSIM_ERR_ARG;
  if (opts->world_size < 1 || opts->rank < 0 || opts->rank >= opts->world_size) return PSIM_ERR_ARG;
  if (opts->queue_cap > PSIM_MAX_CAP) return PSIM_ERR_ARG;
  if (opts->correction_limit > PSIM_MAX_CORRECTION) return PSIM_ERR_ARG;
  if (opts->interval > PSIM_MAX_INTERVAL) return PSIM_ERR_ARG;
  if (opts->precision != PSIM_FP32 && opts->precision != PSIM_BF16) return PSIM_ERR_ARG;
  psim_ctx* ctx = new psim_ctx();
  ctx->opts = *opts;
  ctx->cap = opts->queue_cap ? (int)opts->queue_cap : (int)PSIM_MAX_CAP;
  if (cudaSetDevice(opts->device) != cudaSuccess) { delete ctx; return PSIM_ERR_CUDA; }
  if (opts->stream) {
    ctx->stream = (cudaStream_t)opts->stream;
  } else {
    if (cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking) != cudaSuccess) { delete ctx; return PSIM_ERR_CUDA; }
    ctx->own_stream = true;
  }
  for (auto& e : ctx->ev) cudaEventCreate(&e);
  // a communicator whenever an id is given (also world_size 1: the NCCL leg then runs
  // as it does on G ranks and must leave the totals unchanged -- tested)
  if (opts->nccl_id) {
    if (!load_nccl()) { psim_destroy(ctx); return PSIM_ERR_NCCL; }
    ncclUniqueId id;
    memcpy(&id, opts->nccl_id, sizeof id);
    if (g_nccl.commInitRank(&ctx->comm, opts->world_size, id, opts->rank) != ncclSuccess) {
      ctx->comm = nullptr;
      psim_destroy(ctx);
      return PSIM_ERR_NCCL;
    }
  }
  *out = ctx;
  return PSIM_OK;
}

void psim_destroy(psim_ctx* ctx) {
  if (!ctx) return;
  cudaSetDevice(ctx->opts.device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream);
  if (ctx->comm && g_nccl.ok) g_nccl.commDestroy(ctx->comm);
  dfree(ctx->d_trace);
  dfree(ctx->d_forced);
  for (auto e : ctx->ld_events) cudaEventDestroy(e);
  if (ctx->ld_stream) cudaStreamDestroy(ctx->ld_stream);
  for (auto& l : ctx->model.layers) { dfree(l.w); dfree(l.bias); dfree(l.w_sp); dfree(l.meta); }
  dfree(ctx->model.head_w);
  dfree(ctx->model.head_b);
  SimState& s = ctx->st;
  for (void* p : {(void*)s.ws, (void*)s.s, (void*)s.e, (void*)s.clock, (void*)s.bnd, (void*)s.cycles,
                  (void*)s.count, (void*)s.q, (void*)s.rmin, (void*)s.k_hist,
                  (void*)s.stalls, (void*)s.total, (void*)s.ptile_sum})
    dfree(p);
  dfree(ctx->buf.x);
  for (void* p : ctx->buf.act) dfree(p);
  dfree(ctx->buf.h);
  dfree(ctx->buf.y);
  dfree(ctx->rec_lat);
  dfree(ctx->rec_k);
  dfree(ctx->rec_clock);
  dfree(ctx->rec_y);
  dfree(ctx->fused.T);
  dfree(ctx->fused.w1p);
  dfree(ctx->fused.trace16);
  dfree(ctx->fused.blocks);
  dfree(ctx->fused.count);
  dfree(ctx->fused.tileP[0]);
  dfree(ctx->fused.tileP[1]);
  dfree(ctx->fused.a4);
  for (Cohort& c : ctx->cohorts) {
    dfree(c.blocks); dfree(c.count); dfree(c.tileP[0]); dfree(c.tileP[1]);
    if (c.st) cudaStreamDestroy(c.st);
    if (c.ev) cudaEventDestroy(c.ev);
  }
  for (void* p : {(void*)ctx->pec.k1, (void*)ctx->pec.c1, (void*)ctx->pec.ws, (void*)ctx->pec.s, (void*)ctx->pec.e,
                  (void*)ctx->pec.bnd, (void*)ctx->pec.cyc, (void*)ctx->pec.cycles1, (void*)ctx->pec.len,
                  (void*)ctx->pec.corrected, (void*)ctx->pec.rec_lat, (void*)ctx->pec.rec_k})
    dfree(p);
  dfree(ctx->mrow);
  dfree(ctx->macc);
  dfree(ctx->mout);
  for (auto& e : ctx->ev) if (e) cudaEventDestroy(e);
  if (ctx->own_stream) cudaStreamDestroy(ctx->stream);
  delete ctx;
}

const char* psim_last_error(const psim_ctx* ctx) { return ctx ? ctx->err.c_str() : "null context"; }

int psim_load_trace(psim_ctx* ctx, const uint8_t* attrs, uint64_t n_instr, uint64_t first_row,
                    uint64_t n_rows, uint32_t n_attr, uint64_t row_stride) {
  if (!ctx) return PSIM_ERR_ARG;
  if (!attrs || n_instr == 0) FAIL(PSIM_ERR_ARG, "empty trace");
  if (n_instr >= (1ull << 32)) FAIL(PSIM_ERR_ARG, "L must be < 2^32 (row indices are uint32)");
  if (n_attr != PSIM_NATTR) FAIL(PSIM_ERR_ARG, "n_attr must be 47, got %u", n_attr);
  if (row_stride < 48) FAIL(PSIM_ERR_ARG, "row_stride must be >= 48");
  if (n_rows == 0 || first_row + n_rows > n_instr) FAIL(PSIM_ERR_ARG, "rows [%llu,%llu) outside [0,%llu)",
                                                         (unsigned long long)first_row,
                                                         (unsigned long long)(first_row + n_rows),
                                                         (unsigned long long)n_instr);
  cudaPointerAttributes pa{};
  int mode = 2;
  if (cudaPointerGetAttributes(&pa, attrs) == cudaSuccess) {
    if (pa.type == cudaMemoryTypeDevice || pa.type == cudaMemoryTypeManaged) mode = 0;
    else if (pa.type == cudaMemoryTypeHost) mode = 1;
  }
  cudaGetLastError();
  if (mode == 0 && (row_stride % 16)) FAIL(PSIM_ERR_ARG, "device trace row_stride must be a multiple of 16");
  ctx->trace_devptr = nullptr;
  if (mode == 1) {
    void* dp = nullptr;
    if (cudaHostGetDevicePointer(&dp, const_cast<uint8_t*>(attrs), 0) == cudaSuccess && dp &&
        (row_stride % 16) == 0 && (reinterpret_cast<uintptr_t>(dp) % 16) == 0)
      ctx->trace_devptr = static_cast<const uint8_t*>(dp);
    cudaGetLastError();
  }
  if (ctx->L != n_instr) ctx->partitioned = false;
  ctx->trace = attrs;
  ctx->L = n_instr;
  ctx->first_row = first_row;
  ctx->n_rows = n_rows;
  ctx->stride = row_stride;
  ctx->trace_mode = mode;
  ctx->have_trace = true;
  ctx->done = false;
  return PSIM_OK;
}

// Rank g of G owns sub-traces [floor(gN/G), floor((g+1)N/G)); sub-trace j is
// [s_j, e_j) with s_j = floor(jL/N) (R8) and warm-up start max(0, s_j - W) (R9).
static void rank_block(uint64_t L, uint64_t N, uint64_t W, int g, int G, std::vector<int64_t>* ws_,
                       std::vector<int64_t>* s_, std::vector<int64_t>* e_, uint64_t* j0p, uint64_t* j1p,
                       int64_t* lop, int64_t* hip, int64_t* stepsp) {
  const uint64_t j0 = (uint64_t)(((unsigned __int128)g * N) / G);
  const uint64_t j1 = (uint64_t)(((unsigned __int128)(g + 1) * N) / G);
  auto sj = [&](uint64_t j) { return (int64_t)(((unsigned __int128)j * L) / N); };
  int64_t lo = INT64_MAX, hi = 0, steps = 0;
  for (uint64_t j = j0; j < j1; ++j) {
    const int64_t s = sj(j), e = sj(j + 1);
    const int64_t ws = s > (int64_t)W ? s - (int64_t)W : 0;
    if (ws_) { ws_->push_back(ws); s_->push_back(s); e_->push_back(e); }
    lo = std::min(lo, ws); hi = std::max(hi, e);
    steps = std::max(steps, e - ws);
  }
  if (j1 == j0) { lo = 0; hi = 0; }
  *j0p = j0; *j1p = j1; *lop = lo; *hip = hi; *stepsp = steps;
}

int psim_partition_range(uint64_t L, uint64_t N, uint64_t W, int rank, int world, uint64_t* j0,
                         uint64_t* j1, uint64_t* row_lo, uint64_t* row_hi, uint64_t* steps) {
  if (N == 0 || N > L || world < 1 || rank < 0 || rank >= world) return PSIM_ERR_ARG;
  uint64_t a, b;
  int64_t lo, hi, st;
  rank_block(L, N, W, rank, world, nullptr, nullptr, nullptr, &a, &b, &lo, &hi, &st);
  if (j0) *j0 = a;
  if (j1) *j1 = b;
  if (row_lo) *row_lo = (uint64_t)lo;
  if (row_hi) *row_hi = (uint64_t)hi;
  if (steps) *steps = (uint64_t)st;
  return PSIM_OK;
}

int psim_partition(psim_ctx* ctx, uint64_t N, uint64_t W) {
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->have_trace) FAIL(PSIM_ERR_STATE, "partition before load_trace");
  const uint64_t L = ctx->L;
  if (N == 0 || N > L) FAIL(PSIM_ERR_ARG, "need 1 <= N <= L (N=%llu, L=%llu)", (unsigned long long)N,
                            (unsigned long long)L);
  const int G = ctx->opts.world_size, g = ctx->opts.rank;
  ctx->h_ws.clear(); ctx->h_s.clear(); ctx->h_e.clear();
  uint64_t j0, j1;
  int64_t lo, hi, steps;
  rank_block(L, N, W, g, G, &ctx->h_ws, &ctx->h_s, &ctx->h_e, &j0, &j1, &lo, &hi, &steps);
  if (j1 > j0 && ((uint64_t)lo < ctx->first_row || (uint64_t)hi > ctx->first_row + ctx->n_rows))
    FAIL(PSIM_ERR_ARG, "loaded rows [%llu,%llu) do not cover this rank's range [%lld,%lld)",
         (unsigned long long)ctx->first_row, (unsigned long long)(ctx->first_row + ctx->n_rows),
         (long long)lo, (long long)hi);
  ctx->N = N; ctx->W = W; ctx->j0 = j0; ctx->j1 = j1;
  ctx->row_lo = lo; ctx->row_hi = hi; ctx->steps = steps;
  ctx->partitioned = true;
  ctx->done = false;
  return PSIM_OK;
}

int psim_load_model(psim_ctx* ctx, const psim_model_desc* desc, const float* w, uint64_t n_floats) {
  if (!ctx || !desc || !w) return PSIM_ERR_ARG;
  if (desc->rows != 112 || desc->features != 50) FAIL(PSIM_ERR_ARG, "model input must be 112 x 50");
  struct L_ { int kind, cin, cout, k; };   // kind 0 conv k=s=2, 1 linear, 2 conv k=3 s=1 pad 1
  std::vector<L_> ls;
  const bool rb7 = desc->arch == PSIM_ARCH_RB7;
  if (desc->arch == PSIM_ARCH_M2) ls = {{0, 50, 64, 2}, {0, 64, 64, 2}, {1, 1792, 256, 0}, {1, 256, 3, 0}};
  else if (desc->arch == PSIM_ARCH_C3) ls = {{0, 50, 64, 2}, {0, 64, 128, 2}, {0, 128, 128, 2}, {1, 1792, 256, 0}, {1, 256, 3, 0}};
  else if (rb7) {
    // stem + 3 residual blocks y = relu(x + conv_b(relu(conv_a(x)))) + fc1 3584 -> 256 + fc2 (R11)
    ls = {{0, 50, 64, 2}};
    for (int b = 0; b < 6; ++b) ls.push_back({2, 64, 64, 3});
    ls.push_back({1, 3584, 256, 0});
    ls.push_back({1, 256, 3, 0});
    if (ctx->opts.precision != PSIM_BF16) FAIL(PSIM_ERR_UNSUPPORTED, "RB7 runs on the bf16 tensor-core path only");
  } else FAIL(PSIM_ERR_ARG, "unknown arch %u", desc->arch);
  const bool sparse = (ctx->opts.flags & PSIM_SPARSE24) != 0;
  if (sparse && (rb7 || ctx->opts.precision != PSIM_BF16))
    FAIL(PSIM_ERR_UNSUPPORTED, "PSIM_SPARSE24 needs the bf16 C3 or M2 model");
  uint64_t need = 0;
  for (auto& l : ls) need += (uint64_t)l.cout * l.cin * (l.kind != 1 ? l.k : 1) + l.cout;
  if (need != n_floats) FAIL(PSIM_ERR_ARG, "weight count %llu != %llu for arch %u", (unsigned long long)n_floats,
                             (unsigned long long)need, desc->arch);
  CK(cudaSetDevice(ctx->opts.device));
  Model& m = ctx->model;
  for (auto& l : m.layers) { dfree(l.w); dfree(l.bias); dfree(l.w_sp); dfree(l.meta); }
  m.layers.clear();
  dfree(m.head_w); dfree(m.head_b);
  m.head_w = m.head_b = nullptr;
  const bool bf16 = ctx->opts.precision == PSIM_BF16;
  const float* p = w;
  int pos = 112;   // current positions
  int ch = 50;     // current channels (device layout pads 50 -> 64)
  for (size_t li = 0; li < ls.size(); ++li) {
    const L_& l = ls[li];
    const float* W = p;
    const float* B = p + (uint64_t)l.cout * l.cin * (l.kind != 1 ? l.k : 1);
    p = B + l.cout;
    if (li == ls.size() - 1) {   // head: fc2 stays fp32 (R16)
      CK(cudaMalloc(&m.head_w, sizeof(float) * 3 * l.cin));
      CK(cudaMalloc(&m.head_b, sizeof(float) * 3));
      CK(cudaMemcpy(m.head_w, W, sizeof(float) * 3 * l.cin, cudaMemcpyHostToDevice));
      CK(cudaMemcpy(m.head_b, B, sizeof(float) * 3, cudaMemcpyHostToDevice));
      m.head_in = l.cin;
      break;
    }
    GemmLayer g;
    std::vector<float> Wk;
    if (l.kind == 0) {
      // conv k=s=2: K index = tap * Cin_dev + channel (Cin_dev = 64 for the first layer)
      const int cin_dev = (li == 0) ? kFeatPad : l.cin;
      g.K = 2 * cin_dev;
      g.N = l.cout;
      Wk.assign((size_t)g.N * g.K, 0.f);
      for (int o = 0; o < l.cout; ++o)
        for (int c = 0; c < l.cin; ++c)
          for (int t = 0; t < 2; ++t) Wk[(size_t)o * g.K + t * cin_dev + c] = W[((size_t)o * l.cin + c) * 2 + t];
      pos /= 2;
      g.rows_per_item = pos;
      if (rb7) { g.rows_per_item = pos + 2; g.pad_period = pos + 2; }   // pad-row layout of the k3 convs
      ch = l.cout;
    } else if (l.kind == 2) {
      // conv k=3, stride 1, zero pad 1 over the pad-row layout [pos + 2][C]: K index = tap * Cin + channel,
      // tap t reads position p + t - 1 (PyTorch Conv1d definition)
      g.K = 3 * l.cin;
      g.N = l.cout;
      g.taps = 3;
      Wk.assign((size_t)g.N * g.K, 0.f);
      for (int o = 0; o < l.cout; ++o)
        for (int c = 0; c < l.cin; ++c)
          for (int t = 0; t < 3; ++t) Wk[(size_t)o * g.K + t * l.cin + c] = W[((size_t)o * l.cin + c) * 3 + t];
      g.rows_per_item = pos + 2;
      g.pad_period = pos + 2;
      const int conv_idx = (int)li - 1;         // 0..5: conv_a of block conv_idx/2 when even
      g.block_begin = (conv_idx & 1) == 0;
      g.add_block_input = (conv_idx & 1) == 1;
      ch = l.cout;
    } else {
      if (l.cin != pos * ch) FAIL(PSIM_ERR_ARG, "internal: fc1 fan-in %d != %d", l.cin, pos * ch);
      g.N = l.cout;
      if (rb7) {
        // A = the pad-row layout [pos + 2][ch] flattened; pad positions get zero weights
        g.K = (pos + 2) * ch;
        Wk.assign((size_t)g.N * g.K, 0.f);
        for (int o = 0; o < g.N; ++o)
          for (int q = 0; q < pos * ch; ++q) Wk[(size_t)o * g.K + ch + q] = W[(size_t)o * l.cin + q];
      } else {
        g.K = l.cin;
        Wk.assign(W, W + (size_t)g.N * g.K);   // position-major already (R11)
      }
      g.rows_per_item = 1;
      pos = 1;
      ch = l.cout;
    }
    g.relu = true;
    CK(cudaMalloc(&g.bias, sizeof(float) * g.N));
    CK(cudaMemcpy(g.bias, B, sizeof(float) * g.N, cudaMemcpyHostToDevice));
    if (bf16) {
      std::vector<uint16_t> wb(Wk.size());
      for (size_t t = 0; t < Wk.size(); ++t) wb[t] = f32_to_bf16_rne(Wk[t]);
      CK(cudaMalloc(&g.w, wb.size() * 2));
      CK(cudaMemcpy(g.w, wb.data(), wb.size() * 2, cudaMemcpyHostToDevice));
      if (gemm_tc_supported(g.N, g.K)) {
        g.w_tc = pretile_weight_tc((const __nv_bfloat16*)g.w, g.N, g.K, ctx->stream);
        CK(cudaStreamSynchronize(ctx->stream));
        CK(cudaGetLastError());
      }
      if (sparse) {   // 2:4 compression + tcgen05.mma.sp metadata (gemm_sp.cu)
        std::vector<uint16_t> wc;
        std::vector<uint32_t> meta;
        const int rc = sparse24_compress(wb.data(), g.N, g.K, &wc, &meta, &g.sp_mh);
        if (rc == -2) FAIL(PSIM_ERR_ARG, "layer %zu: weights are not 2:4 sparse along K (PSIM_SPARSE24)", li);
        if (rc != 0) FAIL(PSIM_ERR_UNSUPPORTED, "layer %zu: K = %d, N = %d unsupported by the sparse GEMM", li, g.K, g.N);
        CK(cudaMalloc(&g.w_sp, wc.size() * 2));
        CK(cudaMemcpy(g.w_sp, wc.data(), wc.size() * 2, cudaMemcpyHostToDevice));
        CK(cudaMalloc(&g.meta, meta.size() * 4));
        CK(cudaMemcpy(g.meta, meta.data(), meta.size() * 4, cudaMemcpyHostToDevice));
      }
    } else {
      CK(cudaMalloc(&g.w, Wk.size() * 4));
      CK(cudaMemcpy(g.w, Wk.data(), Wk.size() * 4, cudaMemcpyHostToDevice));
    }
    m.layers.push_back(g);
  }
  m.arch = desc->arch;
  m.precision = ctx->opts.precision;
  m.item_rows = rb7 ? kRows + 4 : kRows;   // RB7: 2 zero rows on each side = one zero pad position
  m.row_off = rb7 ? 2 : 0;
  m.loaded = true;
  ctx->buf_n = 0;                            // layer buffers depend on the architecture
  // fused padding-aware path (bf16 C3): constant table of the all-padding positions
  FusedC3& fz = ctx->fused;
  dfree(fz.T);
  fz.T = nullptr;
  fz.ready = false;
  if (bf16 && desc->arch == PSIM_ARCH_C3 && !sparse) {   // (a 2:4 model runs layer-wise on the sparse GEMM)
    // c3 = conv3(conv2(conv1(0))) with the GPU's rounding points (bf16 operands,
    // bias + ReLU, bf16 activations); T[P] = b_fc1 + sum_{p>=P} Wfc1[:, p*128:(p+1)*128] . c3
    auto bf = [](double v) { uint16_t h = f32_to_bf16_rne((float)v); uint32_t u = (uint32_t)h << 16; float f; memcpy(&f, &u, 4); return (double)f; };
    const float* W1 = w;              const float* B1 = W1 + 64 * 50 * 2;
    const float* W2 = B1 + 64;        const float* B2 = W2 + 128 * 64 * 2;
    const float* W3 = B2 + 128;       const float* B3 = W3 + 128 * 128 * 2;
    const float* WF = B3 + 128;       const float* BF = WF + 256 * 1792;
    double r1[64], r2[128], c3[128];
    for (int o = 0; o < 64; ++o) r1[o] = bf(std::max(0.0, (double)B1[o]));
    for (int o = 0; o < 128; ++o) {
      double acc = 0;
      for (int c = 0; c < 64; ++c) for (int t = 0; t < 2; ++t) acc += bf(W2[(o * 64 + c) * 2 + t]) * r1[c];
      r2[o] = bf(std::max(0.0, acc + B2[o]));
    }
    for (int o = 0; o < 128; ++o) {
      double acc = 0;
      for (int c = 0; c < 128; ++c) for (int t = 0; t < 2; ++t) acc += bf(W3[(o * 128 + c) * 2 + t]) * r2[c];
      c3[o] = bf(std::max(0.0, acc + B3[o]));
    }
    std::vector<float> T(15 * 256);
    for (int o = 0; o < 256; ++o) {
      double acc = (double)BF[o];
      T[14 * 256 + o] = (float)acc;
      for (int P = 13; P >= 0; --P) {
        for (int c = 0; c < 128; ++c) acc += bf(WF[(size_t)o * 1792 + P * 128 + c]) * c3[c];
        T[P * 256 + o] = (float)acc;
      }
    }
    CK(cudaMalloc(&fz.T, T.size() * 4));
    CK(cudaMemcpy(fz.T, T.data(), T.size() * 4, cudaMemcpyHostToDevice));
    fz.w1 = (const __nv_bfloat16*)m.layers[0].w; fz.b1 = m.layers[0].bias;
    {   // conv1 weight in the fused row layout: K = h*64 + col, col < 47 attribute col-3.., 48..50 time
      std::vector<uint16_t> w1p((size_t)64 * 128, 0);
      for (int o = 0; o < 64; ++o)
        for (int h = 0; h < 2; ++h) {
          for (int a = 0; a < 47; ++a) w1p[(size_t)o * 128 + h * 64 + a] = f32_to_bf16_rne(W1[((size_t)o * 50 + 3 + a) * 2 + h]);
          for (int t = 0; t < 3; ++t) w1p[(size_t)o * 128 + h * 64 + 48 + t] = f32_to_bf16_rne(W1[((size_t)o * 50 + t) * 2 + h]);
        }
      dfree(fz.w1p);
      CK(cudaMalloc(&fz.w1p, w1p.size() * 2));
      CK(cudaMemcpy(fz.w1p, w1p.data(), w1p.size() * 2, cudaMemcpyHostToDevice));
    }
    fz.w2 = (const __nv_bfloat16*)m.layers[1].w; fz.b2 = m.layers[1].bias;
    fz.w3 = (const __nv_bfloat16*)m.layers[2].w; fz.b3 = m.layers[2].bias;
    fz.wfc1 = (const __nv_bfloat16*)m.layers[3].w;
    fz.head_w = m.head_w; fz.head_b = m.head_b;
    if (!fused_make_weight_maps(fz)) FAIL(PSIM_ERR_CUDA, "cuTensorMapEncodeTiled failed for the conv weights");
    fz.ready = true;
    fz.cap_n = 0;   // per-run buffers and TMA maps are (re)made by simulate
  }
  ctx->done = false;
  return PSIM_OK;
}

int psim_force_latencies(psim_ctx* ctx, const uint16_t* lat3, uint64_t n_instr) {
  if (!ctx) return PSIM_ERR_ARG;
  if (!lat3) { ctx->forced.clear(); return PSIM_OK; }
  if (!ctx->have_trace || n_instr != ctx->L) FAIL(PSIM_ERR_ARG, "forced latencies must cover all L rows");
  ctx->forced.assign(lat3, lat3 + 3 * n_instr);
  ctx->done = false;
  return PSIM_OK;
}

}  // extern "C"

// ---------------------------------------------------------------------------
static int ensure_buffers(psim_ctx* ctx, uint64_t n) {
  const bool bf16 = ctx->opts.precision == PSIM_BF16;
  const size_t es = bf16 ? 2 : 4;
  if (ctx->buf_n >= n && ctx->buf.x) return PSIM_OK;
  dfree(ctx->buf.x);
  for (void*& p : ctx->buf.act) { dfree(p); p = nullptr; }
  dfree(ctx->buf.h);
  dfree(ctx->buf.y);
  ctx->buf = Buffers{};
  const size_t xr = (size_t)ctx->model.item_rows;
  CK(cudaMalloc(&ctx->buf.x, n * xr * kFeatPad * es));
  CK(cudaMemset(ctx->buf.x, 0, n * xr * kFeatPad * es));   // pad rows stay zero
  for (size_t li = 0; li + 1 < ctx->model.layers.size(); ++li) {
    const GemmLayer& g = ctx->model.layers[li];
    CK(cudaMalloc(&ctx->buf.act[li], n * g.rows_per_item * g.N * es));
  }
  CK(cudaMalloc(&ctx->buf.h, n * 256 * sizeof(float)));
  CK(cudaMalloc(&ctx->buf.y, n * 3 * sizeof(float)));
  ctx->buf_n = n;
  return PSIM_OK;
}

// Run the lowered CNN on buf.x (n items) -> buf.y.  Counts launches.
// layers [first, end) of the lowered CNN on `in0` (default: the gathered inputs buf.x)
static int run_cnn(psim_ctx* ctx, uint64_t n, size_t first = 0, const void* in0 = nullptr) {
  const Model& m = ctx->model;
  Prof& pf = ctx->prof;
  const bool bf16 = m.precision == PSIM_BF16;
  const void* in = in0 ? in0 : ctx->buf.x;
  const void* block_in = nullptr;
  // RB7 residual blocks fused into one kernel each (resblock.cu; PSIM_RB7_FUSED=0: layer-wise A/B)
  static const bool rb7_fused = [] { const char* e = getenv("PSIM_RB7_FUSED"); return !(e && atoi(e) == 0); }();
  for (size_t li = first; li < m.layers.size(); ++li) {
    const GemmLayer& g = m.layers[li];
    const bool last = li + 1 == m.layers.size();
    void* out = last ? (void*)ctx->buf.h : ctx->buf.act[li];
    const int64_t M = (int64_t)n * g.rows_per_item;
    if (g.block_begin) block_in = in;
    if (bf16 && rb7_fused && g.block_begin && g.taps == 3 && li + 1 < m.layers.size() && g.N == 64 && g.K == 192 &&
        m.layers[li + 1].add_block_input && m.layers[li + 1].taps == 3 && !g.w_sp) {
      const GemmLayer& gb = m.layers[li + 1];
      void* outb = ctx->buf.act[li + 1];
      pf.begin(PSIM_KC_LAYER0 + (int)std::min<size_t>(li, 3));
      launch_resblock((const __nv_bfloat16*)in, (const __nv_bfloat16*)g.w, g.bias, (const __nv_bfloat16*)gb.w, gb.bias,
                      (__nv_bfloat16*)outb, M, ctx->stream);
      CK(cudaGetLastError());
      pf.end(PSIM_KC_LAYER0 + (int)std::min<size_t>(li, 3));
      in = outb;
      ++li;   // conv_b done inside the block kernel
      continue;
    }
    pf.begin(PSIM_KC_LAYER0 + (int)std::min<size_t>(li, 3));
    if (bf16 && g.w_sp) {   // 2:4 structured-sparse tcgen05.mma.sp (PSIM_SPARSE24)
      launch_gemm_sp((const __nv_bfloat16*)in, (const __nv_bfloat16*)g.w_sp, g.meta, g.sp_mh, g.bias, out, last, M,
                     g.N, g.K, g.relu, ctx->stream);
    } else if (bf16) {
      if (g.taps > 1 || g.add_block_input || g.pad_period) {
        if (!g.w_tc) FAIL(PSIM_ERR_UNSUPPORTED, "layer %zu needs the tensor-core kernel", li);
        launch_gemm_tc((const __nv_bfloat16*)in, g.w_tc, g.bias, out, last, M, g.N, g.K, g.relu, ctx->stream, g.taps,
                       g.add_block_input ? (const __nv_bfloat16*)block_in : nullptr, g.pad_period);
      } else if (g.w_tc) launch_gemm_tc((const __nv_bfloat16*)in, g.w_tc, g.bias, out, last, M, g.N, g.K, g.relu, ctx->stream);
      else launch_gemm_simt_bf16((const __nv_bfloat16*)in, (const __nv_bfloat16*)g.w, g.bias, out, last, M, g.N, g.K, g.relu, ctx->stream);
    } else {
      launch_gemm_simt_f32((const float*)in, (const float*)g.w, g.bias, (float*)out, M, g.N, g.K, g.relu, ctx->stream);
    }
    CK(cudaGetLastError());
    pf.end(PSIM_KC_LAYER0 + (int)std::min<size_t>(li, 3));
    in = out;
  }
  pf.begin(PSIM_KC_HEAD);
  launch_head(ctx->buf.h, m.head_w, m.head_b, m.head_in, ctx->buf.y, n, ctx->stream);
  pf.end(PSIM_KC_HEAD);
  return PSIM_OK;
}

extern "C" int psim_cnn_forward(psim_ctx* ctx, const float* X, uint64_t B, float* Y) {
  if (!ctx || !X || !Y || B == 0) return PSIM_ERR_ARG;
  if (!ctx->model.loaded) FAIL(PSIM_ERR_STATE, "load_model first");
  CK(cudaSetDevice(ctx->opts.device));
  int rc = ensure_buffers(ctx, B);
  if (rc) return rc;
  float* dX = nullptr;
  CK(cudaMalloc(&dX, B * kRows * kFeat * sizeof(float)));
  cudaError_t e = cudaMemcpyAsync(dX, X, B * kRows * kFeat * sizeof(float), cudaMemcpyHostToDevice, ctx->stream);
  if (e == cudaSuccess) {
    launch_pad_inputs(dX, B, ctx->buf.x, ctx->model.precision == PSIM_BF16, ctx->stream, ctx->model.item_rows,
                      ctx->model.row_off);
    ctx->prof.reset(false, ctx->stream);
    const int rc2 = run_cnn(ctx, B);
    if (rc2) {
      cudaFree(dX);
      return rc2;
    }
    e = cudaMemcpyAsync(Y, ctx->buf.y, B * 3 * sizeof(float), cudaMemcpyDeviceToHost, ctx->stream);
  }
  if (e == cudaSuccess) e = cudaStreamSynchronize(ctx->stream);
  if (e == cudaSuccess) e = cudaGetLastError();
  cudaFree(dX);
  CK(e);
  return PSIM_OK;
}

static int ensure_state(psim_ctx* ctx) {
  const uint64_t n = ctx->j1 - ctx->j0;
  SimState& s = ctx->st;
  if (ctx->st_cap < n || !s.clock) {
    for (void* p : {(void*)s.ws, (void*)s.s, (void*)s.e, (void*)s.clock, (void*)s.bnd, (void*)s.cycles,
                    (void*)s.count, (void*)s.q, (void*)s.rmin})
      dfree(p);
    const uint64_t a = std::max<uint64_t>(n, 1);
    CK(cudaMalloc(&s.rmin, a * 4));
    CK(cudaMalloc(&s.ws, a * 8)); CK(cudaMalloc(&s.s, a * 8)); CK(cudaMalloc(&s.e, a * 8));
    CK(cudaMalloc(&s.clock, a * 8)); CK(cudaMalloc(&s.bnd, a * 8)); CK(cudaMalloc(&s.cycles, a * 8));
    CK(cudaMalloc(&s.count, a * 4));
    CK(cudaMalloc(&s.q, a * kQStride * 16));
    ctx->st_cap = a;
  }
  if (!s.k_hist) {
    CK(cudaMalloc(&s.k_hist, 112 * 8));
    CK(cudaMalloc(&s.stalls, 8));
    CK(cudaMalloc(&s.total, 8));
    CK(cudaMalloc(&s.ptile_sum, 8));
  }
  s.n = n;
  if (n) {
    CK(cudaMemcpyAsync(s.ws, ctx->h_ws.data(), n * 8, cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaMemcpyAsync(s.s, ctx->h_s.data(), n * 8, cudaMemcpyHostToDevice, ctx->stream));
    CK(cudaMemcpyAsync(s.e, ctx->h_e.data(), n * 8, cudaMemcpyHostToDevice, ctx->stream));
  }
  return PSIM_OK;
}

static int ensure_pec(psim_ctx* ctx, uint64_t n, int64_t rows, bool rec) {
  Pec& p = ctx->pec;
  const int limit = (int)ctx->opts.correction_limit;
  const uint64_t a = std::max<uint64_t>(n, 1);
  if (p.cap < a || p.limit < limit) {
    for (void* q : {(void*)p.k1, (void*)p.c1, (void*)p.ws, (void*)p.s, (void*)p.e, (void*)p.bnd, (void*)p.cyc,
                    (void*)p.cycles1, (void*)p.len})
      dfree(q);
    CK(cudaMalloc(&p.k1, (size_t)limit * a + 16));
    CK(cudaMalloc(&p.c1, (size_t)limit * a * 4 + 16));
    CK(cudaMalloc(&p.ws, a * 8)); CK(cudaMalloc(&p.s, a * 8)); CK(cudaMalloc(&p.e, a * 8));
    CK(cudaMalloc(&p.bnd, a * 8)); CK(cudaMalloc(&p.cyc, a * 8)); CK(cudaMalloc(&p.cycles1, a * 8));
    CK(cudaMalloc(&p.len, a * 4));
    p.cap = a;
  }
  p.limit = limit;
  if (!p.corrected) CK(cudaMalloc(&p.corrected, 8));
  if (rec && p.rec_cap < (size_t)rows) {
    dfree(p.rec_lat); dfree(p.rec_k);
    CK(cudaMalloc(&p.rec_lat, rows * 6 + 8));
    CK(cudaMalloc(&p.rec_k, rows * 4 + 8));
    p.rec_cap = rows;
  }
  return PSIM_OK;
}

extern "C" int psim_simulate(psim_ctx* ctx) {
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->have_trace || !ctx->partitioned) FAIL(PSIM_ERR_STATE, "simulate needs load_trace and partition");
  const bool forced = !ctx->forced.empty();
  if (!forced && !ctx->model.loaded) FAIL(PSIM_ERR_STATE, "simulate needs load_model or force_latencies");
  const bool predict = !forced || (ctx->opts.flags & PSIM_FORCE_PREDICT);   // run the CNN each step
  if (predict && !ctx->model.loaded) FAIL(PSIM_ERR_STATE, "PSIM_FORCE_PREDICT needs load_model");
  CK(cudaSetDevice(ctx->opts.device));
  cudaStream_t st = ctx->stream;
  const uint64_t n = ctx->j1 - ctx->j0;
  const int64_t rows = ctx->row_hi - ctx->row_lo;
  psim_stats stats{};
  Prof& pf = ctx->prof;
  pf.reset((ctx->opts.flags & PSIM_PROFILE) != 0, st);
  stats.subtraces = n;
  stats.trace_mode = ctx->trace_mode;
  stats.comm_ranks = ctx->comm ? (int32_t)ctx->opts.world_size : 0;

  int rc = ensure_state(ctx);
  if (rc) return rc;
  const bool fused = predict && ctx->fused.ready && !(ctx->opts.flags & PSIM_LAYERWISE);
  if (predict && !fused) { rc = ensure_buffers(ctx, std::max<uint64_t>(n, 1)); if (rc) return rc; }
  if (fused) {
    FusedC3& fz = ctx->fused;
    fz.pair = (ctx->opts.flags & PSIM_FC1_PAIR) != 0;
    const uint64_t nn = std::max<uint64_t>(n, 1);
    if (fz.cap_n != nn) {
      dfree(fz.blocks); dfree(fz.count); dfree(fz.tileP[0]); dfree(fz.tileP[1]); dfree(fz.a4);
      fz.blocks = nullptr; fz.count = nullptr; fz.tileP[0] = fz.tileP[1] = nullptr; fz.a4 = nullptr;
      const uint64_t nt = (nn + 127) / 128;
      CK(cudaMalloc(&fz.blocks, nn * 14 * 16));
      CK(cudaMalloc(&fz.count, 16));
      CK(cudaMalloc(&fz.tileP[0], nt + 16));
      CK(cudaMalloc(&fz.tileP[1], nt + 16));
      CK(cudaMalloc(&fz.a4, nn * 14 * 128 * 2));
      CK(cudaMemset(fz.a4, 0, nn * 14 * 128 * 2));
      if (!fused_make_maps(fz, nn)) FAIL(PSIM_ERR_CUDA, "cuTensorMapEncodeTiled failed for the fused path");
      fz.cap_n = nn;
    }
  }
  const bool rec = (ctx->opts.flags & PSIM_RECORD_ROWS) != 0;
  if (rec && ctx->rec_cap < (size_t)rows) {
    dfree(ctx->rec_lat); dfree(ctx->rec_k); dfree(ctx->rec_clock);
    CK(cudaMalloc(&ctx->rec_lat, rows * 6 + 8));
    CK(cudaMalloc(&ctx->rec_k, rows * 4 + 8));
    CK(cudaMalloc(&ctx->rec_clock, rows * 8 + 8));
    ctx->rec_cap = rows;
  }
  if (rec && predict && ctx->rec_y_cap < (size_t)rows) {
    dfree(ctx->rec_y);
    ctx->rec_y = nullptr;
    CK(cudaMalloc(&ctx->rec_y, rows * 12 + 16));
    ctx->rec_y_cap = rows;
  }
  ctx->rec_y_valid = rec && predict;
  if (forced) {
    if (ctx->d_forced_cap < (size_t)rows) {
      dfree(ctx->d_forced);
      CK(cudaMalloc(&ctx->d_forced, rows * 6 + 8));
      ctx->d_forced_cap = rows;
    }
    CK(cudaMemcpyAsync(ctx->d_forced, ctx->forced.data() + 3 * ctx->row_lo, rows * 6, cudaMemcpyHostToDevice, st));
  }

  const bool metrics = ctx->opts.interval > 0;
  ctx->metrics_done = false;
  if (metrics) {
    const uint64_t I = ctx->opts.interval;
    ctx->n_int = (ctx->L + I - 1) / I;
    if (ctx->mrow_cap < (size_t)rows) {
      dfree(ctx->mrow); ctx->mrow = nullptr;
      CK(cudaMalloc(&ctx->mrow, rows + 16));
      ctx->mrow_cap = rows;
    }
    if (ctx->macc_cap < std::max<uint64_t>(n, 1)) {
      dfree(ctx->macc); ctx->macc = nullptr;
      CK(cudaMalloc(&ctx->macc, std::max<uint64_t>(n, 1) * 16));
      ctx->macc_cap = std::max<uint64_t>(n, 1);
    }
    if (ctx->mout_cap < ctx->n_int) {
      dfree(ctx->mout); ctx->mout = nullptr;
      CK(cudaMalloc(&ctx->mout, ctx->n_int * 32));
      ctx->mout_cap = ctx->n_int;
    }
    CK(cudaMemsetAsync(ctx->mout, 0, ctx->n_int * 32, st));
  }

  // ---- trace: the rank's rows cross the host link once ----
  CK(cudaEventRecord(ctx->ev[0], st));
  // pinned host trace + fused path: stream it in chunks of lockstep steps, overlapped with
  // the simulation (the paper's pipelined copy, :163), converting to bf16 operand rows on the way
  const bool stream_load = fused && n && ctx->trace_mode == 1 && ctx->trace_devptr;
  const int64_t chunk = ctx->opts.chunk_steps ? (int64_t)ctx->opts.chunk_steps : 64;
  const uint8_t* dtr = nullptr;
  if (stream_load) {
    stats.h2d_bytes = (size_t)rows * 48;
  } else if (ctx->trace_mode == 0) {
    dtr = ctx->trace + (ctx->row_lo - (int64_t)ctx->first_row) * ctx->stride;
  } else {
    const size_t bytes = (size_t)rows * ctx->stride;
    if (ctx->d_trace_cap < bytes) {
      dfree(ctx->d_trace);
      ctx->d_trace = nullptr;
      CK(cudaMalloc(&ctx->d_trace, bytes + 64));
      ctx->d_trace_cap = bytes;
    }
    if (bytes)
      CK(cudaMemcpyAsync(ctx->d_trace, ctx->trace + (ctx->row_lo - (int64_t)ctx->first_row) * ctx->stride, bytes,
                         cudaMemcpyHostToDevice, st));
    stats.h2d_bytes = bytes;
    dtr = ctx->d_trace;
  }
  CK(cudaEventRecord(ctx->ev[1], st));
  const bool pec = ctx->opts.correction_limit > 0 && n > 1;
  if (pec) { rc = ensure_pec(ctx, n, rows, rec); if (rc) return rc; }

  pf.begin(PSIM_KC_OTHER);
  launch_state_init(ctx->st, st);
  pf.end(PSIM_KC_OTHER);
  const bool bf16 = ctx->model.precision == PSIM_BF16;
  GatherArgs ga{dtr, ctx->row_lo, (int64_t)ctx->stride, ctx->st.ws, ctx->st.e, ctx->st.clock, ctx->st.count,
                ctx->st.q, n, 0};
  ga.item_rows = ctx->model.item_rows;
  ga.row_off = ctx->model.row_off;
  UpdateArgs ua{ctx->st, ctx->row_lo, 0, ctx->cap, predict ? ctx->buf.y : nullptr,
                forced ? ctx->d_forced : nullptr, rec ? ctx->rec_lat : nullptr, rec ? ctx->rec_k : nullptr,
                rec ? ctx->rec_clock : nullptr};
  ua.rec_y = (rec && predict) ? ctx->rec_y : nullptr;
  if (pec) { ua.k1_rec = ctx->pec.k1; ua.c1_rec = ctx->pec.c1; ua.limit = ctx->pec.limit; }
  if (metrics) {
    // per-row metric codes: from the device-visible uint8 rows, or written by the
    // streaming loader chunk by chunk (stream_load)
    if (!stream_load && rows > 0) {
      pf.begin(PSIM_KC_OTHER);
      launch_mrow(dtr, (int64_t)ctx->stride, rows, ctx->mrow, st);
      pf.end(PSIM_KC_OTHER);
    }
    ua.mrow = ctx->mrow; ua.macc = ctx->macc; ua.mout = ctx->mout; ua.interval = (int64_t)ctx->opts.interval;
  }
  if (fused && n) {
    // bf16 operand rows of the rank's trace (once per run; the trace crosses HBM once more)
    const size_t t16 = (size_t)rows * 96;
    if (ctx->fused.trace16_cap < t16) {
      dfree(ctx->fused.trace16);
      ctx->fused.trace16 = nullptr;
      CK(cudaMalloc(&ctx->fused.trace16, t16 + 256));
      ctx->fused.trace16_cap = t16;
    }
    // row `rows` of trace16 is all zero: the padding rows of the gathered input point at it
    CK(cudaMemsetAsync(ctx->fused.trace16 + (size_t)rows * 48, 0, 96, st));
    if (!fused_make_trace_map(ctx->fused, (uint64_t)rows))
      FAIL(PSIM_ERR_CUDA, "cuTensorMapEncodeTiled failed for the trace gather map");
    if (stream_load) {
      if (!ctx->ld_stream) CK(cudaStreamCreateWithFlags(&ctx->ld_stream, cudaStreamNonBlocking));
      const size_t nch = (size_t)((ctx->steps + chunk - 1) / chunk);
      while (ctx->ld_events.size() < nch) {
        cudaEvent_t e;
        CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        ctx->ld_events.push_back(e);
      }
      CK(cudaStreamWaitEvent(ctx->ld_stream, ctx->ev[0], 0));
      for (size_t c = 0; c < nch; ++c) {
        launch_load_chunk16(ctx->trace_devptr, (int64_t)ctx->first_row, (int64_t)ctx->stride, ctx->st.ws, ctx->st.e,
                            n, (int64_t)c * chunk, (int64_t)(c + 1) * chunk, ctx->row_lo, ctx->fused.trace16,
                            metrics ? ctx->mrow : nullptr, ctx->ld_stream);
        CK(cudaEventRecord(ctx->ld_events[c], ctx->ld_stream));
      }
      pf.launches[PSIM_KC_OTHER] += nch;
    } else {
      pf.begin(PSIM_KC_OTHER);
      launch_trace16(dtr, (int64_t)ctx->stride, rows, ctx->fused.trace16, st);
      pf.end(PSIM_KC_OTHER);
    }
    // invariant of the fused path: a4 rows p >= P_b are zero (fc1 reads them as 0)
    CK(cudaMemsetAsync(ctx->fused.a4, 0, n * 14 * 128 * 2, st));
    pf.begin(PSIM_KC_OTHER);
    launch_fused_init(ctx->fused, ctx->st.ws, n, st);
    pf.end(PSIM_KC_OTHER);
  }
  // cohorts (fused first pass without correction / interval metrics): PSIM_COHORTS, default
  // 2 when the trace streams from pinned host memory (measured on config 3: e2e 406 -> 428
  // MIPS, the chunk copies overlap better), 1 otherwise (device-resident: 537.6 vs 537.0,
  // 3-4 cohorts slower; profiles/r01_cohorts.txt)
  int ncoh = 1;
  if (fused && n && !pec && !metrics) {
    const char* ev = getenv("PSIM_COHORTS");
    ncoh = ev ? std::max(1, atoi(ev)) : (stream_load ? 2 : 1);
    while (ncoh > 1 && n < (uint64_t)ncoh * 256) --ncoh;
  }
  if (ncoh > 1) {
    if ((int)ctx->cohorts.size() < ncoh) ctx->cohorts.resize(ncoh);
    CK(cudaEventRecord(ctx->ev[3], st));   // common preparation done
    for (int c = 0; c < ncoh; ++c) {
      Cohort& ch = ctx->cohorts[c];
      const uint64_t b0 = (n * (uint64_t)c / ncoh) & ~uint64_t(127), b1 = c + 1 == ncoh ? n : (n * (uint64_t)(c + 1) / ncoh) & ~uint64_t(127);
      ch.b0 = b0; ch.n = b1 - b0;
      if (!ch.st) CK(cudaStreamCreateWithFlags(&ch.st, cudaStreamNonBlocking));
      if (!ch.ev) CK(cudaEventCreateWithFlags(&ch.ev, cudaEventDisableTiming));
      if (ch.cap < ch.n) {
        dfree(ch.blocks); dfree(ch.count); dfree(ch.tileP[0]); dfree(ch.tileP[1]);
        const uint64_t nt = (ch.n + 127) / 128;
        CK(cudaMalloc(&ch.blocks, ch.n * 14 * 16));
        CK(cudaMalloc(&ch.count, 16));
        CK(cudaMalloc(&ch.tileP[0], nt + 16));
        CK(cudaMalloc(&ch.tileP[1], nt + 16));
        ch.cap = ch.n;
      }
      ch.fz = ctx->fused;
      ch.fz.blocks = ch.blocks; ch.fz.count = ch.count; ch.fz.tileP[0] = ch.tileP[0]; ch.fz.tileP[1] = ch.tileP[1];
      ch.fz.a4 = ctx->fused.a4 + b0 * 14 * 128;
      // PSIM_COHORT_SMS=1: each cohort's persistent kernels get a disjoint share of the SMs,
      // so one cohort's conv_stack runs beside another's fc1_head instead of queueing behind it
      static const bool share = [] { const char* e = getenv("PSIM_COHORT_SMS"); return e && atoi(e) != 0; }();
      ch.fz.grid_cap = share ? std::max(1, sm_count() / ncoh) : 0;
      if (!fused_make_maps(ch.fz, ch.n)) FAIL(PSIM_ERR_CUDA, "cuTensorMapEncodeTiled failed for a cohort");
      CK(cudaStreamWaitEvent(ch.st, ctx->ev[3], 0));
      launch_fused_init(ch.fz, ctx->st.ws + ch.b0, ch.n, ch.st);
      pf.count(PSIM_KC_OTHER);
    }
  }
  // a cohort's view of the state: pointers offset by its first sub-trace, queue stride kept
  auto view = [&](const SimState& s0, uint64_t b0, uint64_t nc) {
    SimState v = s0;
    v.n = nc; v.qn = s0.n;
    v.ws = s0.ws + b0; v.s = s0.s + b0; v.e = s0.e + b0; v.clock = s0.clock + b0; v.bnd = s0.bnd + b0;
    v.cycles = s0.cycles + b0; v.count = s0.count + b0; v.rmin = s0.rmin + b0; v.q = s0.q + b0;
    return v;
  };
  // one lockstep step t of a pass: gather -> CNN -> rounding -> queue update
  auto step = [&](GatherArgs& g, UpdateArgs& u, const int64_t* e_arr, int64_t t) -> int {
    if (fused) {
      g.step = t;
      u.step = t;
      pf.begin(PSIM_KC_LAYER0);
      launch_conv_stack(ctx->fused, g, t, n, st);
      pf.end(PSIM_KC_LAYER0);
      pf.begin(PSIM_KC_LAYER0 + 3);
      launch_fc1_head(ctx->fused, u, e_arr, t, forced, st);
      pf.end(PSIM_KC_LAYER0 + 3);
      return PSIM_OK;
    }
    if (predict) {
      g.step = t;
      // RB7: gather + stem convolution in one kernel (rb7_stem.cu; PSIM_RB7_STEM=0: layer-wise A/B)
      static const bool rb7_stem = [] { const char* e = getenv("PSIM_RB7_STEM"); return !(e && atoi(e) == 0); }();
      if (bf16 && rb7_stem && ctx->model.arch == PSIM_ARCH_RB7 && !ctx->model.layers.empty() &&
          ctx->model.layers[0].K == 128 && ctx->model.layers[0].N == 64) {
        const GemmLayer& l0 = ctx->model.layers[0];
        pf.begin(PSIM_KC_LAYER0);
        launch_rb7_stem(g, (const __nv_bfloat16*)l0.w, l0.bias, (__nv_bfloat16*)ctx->buf.act[0], st);
        CK(cudaGetLastError());
        pf.end(PSIM_KC_LAYER0);
        const int r = run_cnn(ctx, n, 1, ctx->buf.act[0]);
        if (r) return r;
        u.step = t;
        pf.begin(PSIM_KC_UPDATE);
        launch_update(u, st);
        pf.end(PSIM_KC_UPDATE);
        return PSIM_OK;
      }
      pf.begin(PSIM_KC_GATHER);
      if (bf16) launch_gather_bf16(g, (__nv_bfloat16*)ctx->buf.x, st);
      else launch_gather_f32(g, (float*)ctx->buf.x, st);
      pf.end(PSIM_KC_GATHER);
      const int r = run_cnn(ctx, n);
      if (r) return r;
    }
    u.step = t;
    pf.begin(PSIM_KC_UPDATE);
    launch_update(u, st);
    pf.end(PSIM_KC_UPDATE);
    return PSIM_OK;
  };
  if (ncoh > 1) {
    // cohorts on their own streams, launches interleaved step by step; cohort 0's
    // launches carry the (sampled) kernel timing, the others are counted only
    std::vector<GatherArgs> gc(ncoh, ga);
    std::vector<UpdateArgs> uc(ncoh, ua);
    for (int c = 0; c < ncoh; ++c) {
      const Cohort& ch = ctx->cohorts[c];
      const SimState v = view(ctx->st, ch.b0, ch.n);
      gc[c].ws = v.ws; gc[c].e = v.e; gc[c].clock = v.clock; gc[c].count = v.count; gc[c].q = v.q;
      gc[c].n = ch.n; gc[c].qn = n;
      uc[c].st = v;
    }
    cudaStream_t st0 = pf.st;
    for (int64_t t = 0; t < ctx->steps; ++t) {
      for (int c = 0; c < ncoh; ++c) {
        Cohort& ch = ctx->cohorts[c];
        if (stream_load && t % chunk == 0) CK(cudaStreamWaitEvent(ch.st, ctx->ld_events[t / chunk], 0));
        gc[c].step = t; uc[c].step = t;
        const bool timed = c == 0 && t % Prof::kEvery == 0;
        pf.st = ch.st;
        pf.sample = timed;
        pf.begin(PSIM_KC_LAYER0);
        launch_conv_stack(ch.fz, gc[c], t, ch.n, ch.st);
        pf.end(PSIM_KC_LAYER0);
        pf.begin(PSIM_KC_LAYER0 + 3);
        launch_fc1_head(ch.fz, uc[c], ctx->st.e + ch.b0, t, forced, ch.st);
        pf.end(PSIM_KC_LAYER0 + 3);
      }
    }
    pf.st = st0;
    for (int c = 0; c < ncoh; ++c) {
      CK(cudaEventRecord(ctx->cohorts[c].ev, ctx->cohorts[c].st));
      CK(cudaStreamWaitEvent(st, ctx->cohorts[c].ev, 0));
    }
  } else {
    for (int64_t t = 0; t < ctx->steps && n; ++t) {
      if (stream_load && t % chunk == 0) CK(cudaStreamWaitEvent(st, ctx->ld_events[t / chunk], 0));
      pf.sample = t % Prof::kEvery == 0;
      rc = step(ga, ua, ctx->st.e, t);
      if (rc) return rc;
    }
  }
  pf.sample = true;
  // ---- post-error correction pass (PAPER.md:203-219 [V-B], Fig. 9; R19) ----
  // corrector b continues from its final state over rows of sub-trace b+1 (same
  // kernels, lockstep over correctors, at most `limit` steps), then the
  // re-simulated cycles replace b+1's.  Local sub-traces only: the first
  // sub-trace of this rank is never corrected (:219).
  if (pec) {
    Pec& p = ctx->pec;
    pf.begin(PSIM_KC_OTHER);
    launch_pec_init(ctx->st, p, st);
    pf.end(PSIM_KC_OTHER);
    SimState s2 = ctx->st;
    s2.ws = p.ws; s2.s = p.s; s2.e = p.e; s2.bnd = p.bnd; s2.cycles = p.cyc;
    GatherArgs g2 = ga;
    g2.ws = p.ws; g2.e = p.e;
    UpdateArgs u2 = ua;
    u2.st = s2;
    u2.k1_rec = nullptr; u2.c1_rec = nullptr;
    u2.kref = p.k1;
    u2.macc = nullptr; u2.mout = nullptr;   // metrics come from the first pass (R20)
    u2.rec_lat = rec ? p.rec_lat : nullptr;
    u2.rec_k = rec ? p.rec_k : nullptr;
    u2.rec_clock = nullptr;
    u2.rec_y = nullptr;   // recorded outputs stay the first pass's
    if (rec) {
      CK(cudaMemsetAsync(p.rec_lat, 0, rows * 6, st));
      CK(cudaMemsetAsync(p.rec_k, 0xFF, rows * 4, st));
    }
    if (fused) {
      // a4 rows >= P_b must be zero again: the final steps of the first pass leave rows behind
      CK(cudaMemsetAsync(ctx->fused.a4, 0, n * 14 * 128 * 2, st));
      pf.begin(PSIM_KC_OTHER);
      launch_fused_init_from_state(ctx->fused, ctx->st.count, ctx->st.clock, p.ws, p.e, n, st);
      pf.end(PSIM_KC_OTHER);
    }
    for (int64_t t = 0; t < p.limit; ++t) {
      pf.sample = t % Prof::kEvery == 0;
      rc = step(g2, u2, p.e, t);
      if (rc) return rc;
    }
    pf.sample = true;
    pf.begin(PSIM_KC_OTHER);
    launch_pec_apply(ctx->st, p, st);
    pf.end(PSIM_KC_OTHER);
    stats.corr_steps = (uint64_t)p.limit;
  }
  pf.begin(PSIM_KC_OTHER);
  launch_reduce_cycles(ctx->st, st);
  pf.end(PSIM_KC_OTHER);
  CK(cudaGetLastError());
  if (ctx->comm) {
    ncclResult_t r = g_nccl.allReduce(ctx->st.total, ctx->st.total, 1, ncclInt64, ncclSum, ctx->comm, st);
    if (r != ncclSuccess) FAIL(PSIM_ERR_NCCL, "ncclAllReduce: %s", g_nccl.errStr(r));
    if (metrics && ctx->n_int) {   // interval sums over all ranks (intervals straddle rank boundaries)
      r = g_nccl.allReduce(ctx->mout, ctx->mout, ctx->n_int * 4, ncclUint64, ncclSum, ctx->comm, st);
      if (r != ncclSuccess) FAIL(PSIM_ERR_NCCL, "ncclAllReduce (metrics): %s", g_nccl.errStr(r));
    }
  }
  CK(cudaEventRecord(ctx->ev[2], st));
  long long total = 0;
  CK(cudaMemcpyAsync(&total, ctx->st.total, 8, cudaMemcpyDeviceToHost, st));
  unsigned long long hist[112], stalls = 0, ptile_sum = 0;
  CK(cudaMemcpyAsync(hist, ctx->st.k_hist, sizeof hist, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(&stalls, ctx->st.stalls, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(&ptile_sum, ctx->st.ptile_sum, 8, cudaMemcpyDeviceToHost, st));
  unsigned long long corrected = 0;
  if (pec) CK(cudaMemcpyAsync(&corrected, ctx->pec.corrected, 8, cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  CK(cudaGetLastError());
  float ms_all = 0, ms_load = 0;
  cudaEventElapsedTime(&ms_all, ctx->ev[0], ctx->ev[2]);
  cudaEventElapsedTime(&ms_load, ctx->ev[0], ctx->ev[1]);
  ctx->total = total;
  for (int k = 0; k < 112; ++k) stats.k_hist[k] = hist[k];
  stats.stalls = stalls;
  stats.steps = (uint64_t)ctx->steps;
  uint64_t sim = 0, cnt = 0;
  for (uint64_t b = 0; b < n; ++b) { sim += ctx->h_e[b] - ctx->h_ws[b]; cnt += ctx->h_e[b] - ctx->h_s[b]; }
  stats.corrected = corrected;
  stats.simulated = sim + corrected;
  ctx->pec_done = pec;
  stats.counted = cnt;
  uint64_t launches = 0;
  for (int c = 0; c < PSIM_KC_COUNT; ++c) { stats.kernel_launches[c] = pf.launches[c]; launches += pf.launches[c]; }
  stats.gpu_launches = launches;
  pf.collect(stats.kernel_ms);
  for (size_t li = 0; li < ctx->model.layers.size() && li < 4 && predict && !fused; ++li) {
    const GemmLayer& g = ctx->model.layers[li];
    stats.layer_m[li] = n * g.rows_per_item;
    stats.layer_n[li] = g.N;
    stats.layer_k[li] = g.K;
  }
  stats.sim_ms = ms_all;
  stats.load_ms = ms_load;
  if (ctx->comm == nullptr) stats.local_cycles = total;
  else {
    long long lc = 0;
    // local sum = re-reduce the cycles (cheap; diagnostics only)
    std::vector<long long> cyc(n);
    if (n) CK(cudaMemcpy(cyc.data(), ctx->st.cycles, n * 8, cudaMemcpyDeviceToHost));
    for (auto v : cyc) lc += v;
    stats.local_cycles = lc;
  }
  if (fused) fused_dump_debug();
  if (fused) {   // GEMM shapes of the fused kernels: blocks (conv stack) and fc1 rows
    uint64_t blocks = 0;
    for (int k = 0; k < 112; ++k) blocks += stats.k_hist[k] * (uint64_t)((k + 8) / 8);
    stats.layer_m[0] = blocks / std::max<uint64_t>(stats.steps, 1);   // mean blocks per step
    stats.layer_n[0] = 128; stats.layer_k[0] = 0;
    // fc1: M = sub-traces, N = 256, K = 128 x (mean P_tile over tiles), reported x1000 in layer_k
    const uint64_t tiles = ((n + 127) / 128) * std::max<uint64_t>(stats.steps, 1);
    stats.layer_m[3] = n; stats.layer_n[3] = 256;
    stats.layer_k[3] = (uint32_t)(1000.0 * 128.0 * (double)ptile_sum / (double)tiles);
  }
  ctx->stats = stats;
  ctx->done = true;
  ctx->metrics_done = metrics;
  return PSIM_OK;
}

extern "C" int psim_get_interval_metrics(const psim_ctx* cctx, uint64_t first, uint64_t n, int64_t* cycles,
                                         int64_t* retired, int64_t* retired_st, int64_t* mem_bytes) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (!ctx->metrics_done) FAIL(PSIM_ERR_STATE, "context created with interval = 0");
  if (first > ctx->n_int || n > ctx->n_int - first) FAIL(PSIM_ERR_ARG, "intervals outside [0, %llu)",
                                                          (unsigned long long)ctx->n_int);
  if (n == 0) return PSIM_OK;
  CK(cudaSetDevice(ctx->opts.device));
  std::vector<unsigned long long> h(n * 4);
  CK(cudaMemcpy(h.data(), ctx->mout + first * 4, n * 32, cudaMemcpyDeviceToHost));
  for (uint64_t g = 0; g < n; ++g) {
    if (cycles) cycles[g] = (int64_t)h[4 * g];
    if (retired) retired[g] = (int64_t)h[4 * g + 1];
    if (retired_st) retired_st[g] = (int64_t)h[4 * g + 2];
    if (mem_bytes) mem_bytes[g] = (int64_t)h[4 * g + 3];
  }
  return PSIM_OK;
}

extern "C" const char* psim_kernel_class_name(int i) {
  static const char* names[PSIM_KC_COUNT] = {"gather", "gemm_layer0", "gemm_layer1", "gemm_layer2",
                                             "gemm_layer3", "head", "update", "other"};
  return (i >= 0 && i < PSIM_KC_COUNT) ? names[i] : nullptr;
}

extern "C" int psim_nccl_unique_id(void* out128) {
  if (!out128) return PSIM_ERR_ARG;
  if (!load_nccl()) return PSIM_ERR_NCCL;
  ncclUniqueId id;
  if (g_nccl.getUniqueId(&id) != ncclSuccess) return PSIM_ERR_NCCL;
  memcpy(out128, &id, sizeof id);
  return PSIM_OK;
}

extern "C" int psim_total_cycles(const psim_ctx* ctx, int64_t* out) {
  if (!ctx || !out) return PSIM_ERR_ARG;
  if (!ctx->done) return PSIM_ERR_STATE;
  *out = ctx->total;
  return PSIM_OK;
}

extern "C" int psim_get_rows(const psim_ctx* cctx, uint64_t first, uint64_t n, uint16_t* out3, int32_t* k,
                             int64_t* clock) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (!(ctx->opts.flags & PSIM_RECORD_ROWS)) FAIL(PSIM_ERR_STATE, "context created without PSIM_RECORD_ROWS");
  const int64_t s_first = ctx->h_s.empty() ? 0 : ctx->h_s.front();
  if ((int64_t)first < s_first || (int64_t)(first + n) > ctx->row_hi) FAIL(PSIM_ERR_ARG, "rows outside this rank");
  const int64_t off = (int64_t)first - ctx->row_lo;
  CK(cudaSetDevice(ctx->opts.device));
  if (out3) CK(cudaMemcpy(out3, ctx->rec_lat + 3 * off, n * 6, cudaMemcpyDeviceToHost));
  if (k) CK(cudaMemcpy(k, ctx->rec_k + off, n * 4, cudaMemcpyDeviceToHost));
  if (clock) CK(cudaMemcpy(clock, ctx->rec_clock + off, n * 8, cudaMemcpyDeviceToHost));
  return PSIM_OK;
}

extern "C" int psim_get_outputs(const psim_ctx* cctx, uint64_t first, uint64_t n, float* out3) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx || !out3) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (!ctx->rec_y_valid) FAIL(PSIM_ERR_STATE, "no recorded CNN outputs (needs PSIM_RECORD_ROWS and a CNN run)");
  const int64_t s_first = ctx->h_s.empty() ? 0 : ctx->h_s.front();
  if ((int64_t)first < s_first || (int64_t)(first + n) > ctx->row_hi) FAIL(PSIM_ERR_ARG, "rows outside this rank");
  const int64_t off = (int64_t)first - ctx->row_lo;
  CK(cudaSetDevice(ctx->opts.device));
  CK(cudaMemcpy(out3, ctx->rec_y + 3 * off, n * 12, cudaMemcpyDeviceToHost));
  return PSIM_OK;
}

extern "C" int psim_get_subtrace_cycles(const psim_ctx* cctx, uint64_t first, uint64_t n, int64_t* out) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx || !out) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (first + n > ctx->j1 - ctx->j0) FAIL(PSIM_ERR_ARG, "sub-traces outside this rank");
  CK(cudaSetDevice(ctx->opts.device));
  CK(cudaMemcpy(out, ctx->st.cycles + first, n * 8, cudaMemcpyDeviceToHost));
  return PSIM_OK;
}

extern "C" int psim_get_corrections(const psim_ctx* cctx, uint64_t first, uint64_t n, int32_t* corr_len,
                                    int64_t* cycles1) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (first + n > ctx->j1 - ctx->j0) FAIL(PSIM_ERR_ARG, "sub-traces outside this rank");
  CK(cudaSetDevice(ctx->opts.device));
  if (ctx->opts.correction_limit == 0) FAIL(PSIM_ERR_STATE, "context created with correction_limit = 0");
  if (!ctx->pec_done) {   // a single local sub-trace: nothing re-simulated
    if (corr_len) memset(corr_len, 0, n * 4);
    if (cycles1 && n) CK(cudaMemcpy(cycles1, ctx->st.cycles + first, n * 8, cudaMemcpyDeviceToHost));
    return PSIM_OK;
  }
  if (corr_len && n) CK(cudaMemcpy(corr_len, ctx->pec.len + first, n * 4, cudaMemcpyDeviceToHost));
  if (cycles1 && n) CK(cudaMemcpy(cycles1, ctx->pec.cycles1 + first, n * 8, cudaMemcpyDeviceToHost));
  return PSIM_OK;
}

extern "C" int psim_get_corrected_rows(const psim_ctx* cctx, uint64_t first, uint64_t n, uint16_t* out3,
                                       int32_t* k) {
  psim_ctx* ctx = const_cast<psim_ctx*>(cctx);
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->done) FAIL(PSIM_ERR_STATE, "no simulate yet");
  if (!(ctx->opts.flags & PSIM_RECORD_ROWS)) FAIL(PSIM_ERR_STATE, "context created without PSIM_RECORD_ROWS");
  if (ctx->opts.correction_limit == 0) FAIL(PSIM_ERR_STATE, "context created with correction_limit = 0");
  const int64_t s_first = ctx->h_s.empty() ? 0 : ctx->h_s.front();
  if ((int64_t)first < s_first || (int64_t)(first + n) > ctx->row_hi) FAIL(PSIM_ERR_ARG, "rows outside this rank");
  if (!ctx->pec_done) {
    if (out3) memset(out3, 0, n * 6);
    if (k) for (uint64_t r = 0; r < n; ++r) k[r] = -1;
    return PSIM_OK;
  }
  const int64_t off = (int64_t)first - ctx->row_lo;
  CK(cudaSetDevice(ctx->opts.device));
  if (out3) CK(cudaMemcpy(out3, ctx->pec.rec_lat + 3 * off, n * 6, cudaMemcpyDeviceToHost));
  if (k) CK(cudaMemcpy(k, ctx->pec.rec_k + off, n * 4, cudaMemcpyDeviceToHost));
  return PSIM_OK;
}

extern "C" int psim_rank_range(const psim_ctx* ctx, uint64_t* j0, uint64_t* j1, uint64_t* lo, uint64_t* hi) {
  if (!ctx) return PSIM_ERR_ARG;
  if (!ctx->partitioned) return PSIM_ERR_STATE;
  if (j0) *j0 = ctx->j0;
  if (j1) *j1 = ctx->j1;
  if (lo) *lo = (uint64_t)ctx->row_lo;
  if (hi) *hi = (uint64_t)ctx->row_hi;
  return PSIM_OK;
}

extern "C" int psim_get_stats(const psim_ctx* ctx, psim_stats* out) {
  if (!ctx || !out) return PSIM_ERR_ARG;
  if (!ctx->done) return PSIM_ERR_STATE;
  *out = ctx->stats;
  return PSIM_OK;
}
