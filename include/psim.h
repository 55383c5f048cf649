/*
 * psim.h -- C ABI of the B200-native parallel sub-trace ML microarchitecture
 * simulator (the data-parallel hot path of Pandey et al., "Scalable Deep
 * Learning-Based Microarchitecture Simulation on GPUs", SC'22).
 *
 * Citations: PAPER.md:<line> and DESIGN.md R<n>
 * (the readings taken where the paper is silent or garbled).
 *
 * The calls follow the paper's problem statement: a trace of L encoded
 * instructions, a trained latency model (:63), a partition into
 * N sub-traces with W warm-up instructions each (:171-181, :197), simulation
 * and one gather of the Clocks (:181) giving the total cycles (:107).
 *
 * Conventions
 *  - Every function returns int status: PSIM_OK (0) or a negative PSIM_ERR_*.
 *    No exception or abort crosses the ABI; psim_last_error() describes the
 *    last failure on a context.
 *  - One context per thread; one process (one context) per GPU.
 *  - Pointers are plain host or device pointers (the library inspects them
 *    with cudaPointerGetAttributes); sizes are element counts unless noted.
 *  - State machine: CREATED -> (load_trace) -> (partition) -> simulate -> DONE.
 *    load_model (or psim_force_latencies) may come at any point before
 *    simulate.  Out-of-order calls return PSIM_ERR_STATE.
 */
#ifndef PSIM_H
#define PSIM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PSIM_OK 0
#define PSIM_ERR_ARG (-1)          /* bad argument (sizes, N = 0, N > L, ...)          */
#define PSIM_ERR_STATE (-2)        /* call out of order                               */
#define PSIM_ERR_CUDA (-3)         /* CUDA runtime / launch failure                    */
#define PSIM_ERR_NCCL (-4)         /* NCCL missing or failed                           */
#define PSIM_ERR_OOM (-5)          /* device or pinned allocation failed               */
#define PSIM_ERR_UNSUPPORTED (-6)  /* model/precision combination not built            */

#define PSIM_FP32 0u  /* CNN operands and accumulation in fp32 (CUDA cores)            */
#define PSIM_BF16 1u  /* bf16 operands, fp32 accumulation (tcgen05 tensor cores, R16)  */

#define PSIM_ARCH_M2 1u   /* 2 conv + 2 FC ("2-conv-layer" model, config 1, R11)      */
#define PSIM_ARCH_C3 2u   /* 3 conv + 2 FC ("3C+2F", PAPER.md:63, 64 conv1 ch :161)   */
#define PSIM_ARCH_RB7 3u  /* residual 7-conv variant (config 5, R11)                   */

#define PSIM_MAX_CAP 110u /* Context_length: input length 111 = Context_length + 1 */
#define PSIM_MAX_CORRECTION 4096u /* largest psim_opts.correction_limit (the paper uses 100, :291) */
#define PSIM_MAX_INTERVAL 262144u /* largest psim_opts.interval (keeps a sub-trace's per-interval
                                     Clock advance below 2^32: <= 12285 per row)                */
#define PSIM_NATTR 47u    /* trace attributes per instruction; + 3 time features = 50 (R1) */

/* flags for psim_opts.flags */
#define PSIM_RECORD_ROWS 1u  /* keep per-instruction (f,c,s), context count k and Clock
                                (device buffers sized to the rank's rows) for parity reads */
#define PSIM_FORCE_PREDICT 4u /* with psim_force_latencies: still run gather + CNN + rounding every
                                step and record the CNN's (f,c,s) in the per-row outputs, while the
                                queue update follows the forced latencies (decision parity on a
                                given trajectory, R17)                              */
#define PSIM_LAYERWISE 8u    /* bf16 C3: use the layer-by-layer GEMM path instead of the fused
                                padding-aware kernels (A/B comparison, parity of both)       */
#define PSIM_SPARSE24 16u    /* 2:4 structured sparsity (PAPER.md:157 [IV-B], :261 [VI-B]): the
                                model's tensor-core layers (C3 / M2 conv1..3 and fc1, bf16) must be
                                2:4 sparse along their reduction dimension K in the device order
                                (conv: K = tap * Cin_dev + channel, groups of 4 consecutive input
                                channels of one tap; fc1: 4 consecutive flattened inputs) -- e.g.
                                magnitude-pruned weights, which the oracle loads unchanged; they are
                                compressed at psim_load_model and every layer runs on the sparse
                                tcgen05.mma.sp GEMM of the layer-wise path.  load_model returns ARG
                                if a group holds more than 2 nonzeros, UNSUPPORTED for other
                                architectures or fp32                                          */
#define PSIM_FC1_PAIR 32u    /* fused C3 path: fc1_head on 2-SM MMAs (tcgen05.mma.cta_group::2,
                                M = 256 over a cluster of two CTAs, each staging its own tile's
                                activations and half of the fc1 weights; multicast commits,
                                2-SM TMA).  Same results; measured slower on B200 (fc1_head is
                                not bound by its weight stream), so off by default       */
#define PSIM_PROFILE 2u      /* time kernel classes with CUDA events on the launch stream: every
                                launch outside the step loop and the launches of every 16th
                                lockstep step (events between all launches would serialise the
                                programmatic-dependent-launch overlap of the fused kernels);
                                psim_stats.kernel_ms is scaled to all launches of a class  */

/* kernel classes reported in psim_stats.kernel_ms (names: psim_kernel_class_name) */
#define PSIM_KC_GATHER 0
#define PSIM_KC_LAYER0 1   /* first GEMM layer (conv1); layer i is PSIM_KC_LAYER0 + i;
                              fused path: 1 = conv_stack (gather+conv1-3), 4 = fc1_head (+update) */
#define PSIM_KC_HEAD 5
#define PSIM_KC_UPDATE 6
#define PSIM_KC_OTHER 7
#define PSIM_KC_COUNT 8

typedef struct psim_ctx psim_ctx;  /* opaque; owns every device allocation it makes */

typedef struct {
    int device;             /* CUDA ordinal for this process (one process per GPU)            */
    int rank, world_size;   /* 0, 1 for a single GPU                                           */
    const void* nccl_id;    /* 128-byte ncclUniqueId from rank 0; NULL: no in-library collective,
                               psim_total_cycles then returns this rank's sum and the caller
                               reduces (e.g. torch.distributed over gloo in CPU tests)          */
    uint32_t queue_cap;     /* max live context entries after a step, 1..110 (0 -> 110)        */
    uint32_t precision;     /* PSIM_FP32 | PSIM_BF16                                           */
    uint64_t chunk_steps;   /* trace loader chunk length in lockstep steps (0 = automatic)     */
    void* stream;           /* cudaStream_t to launch on (NULL: the library creates one)       */
    uint32_t flags;         /* PSIM_RECORD_ROWS | 0                                            */
    uint32_t correction_limit; /* post-error correction (PAPER.md:203-219 [V-B], Fig. 9; DESIGN.md
                               R19): after the lockstep pass, every local sub-trace j except this
                               rank's last continues from its final state over at most this many
                               rows of sub-trace j+1, stopping at the first row whose context count
                               matches j+1's first pass; the re-simulated cycles replace j+1's.
                               The first sub-trace of a rank is never corrected (:219).
                               0 = off; the paper uses 100 (:291).                              */
    uint32_t interval;      /* interval metrics (PAPER.md:310-318 [VI-E]; R20): 0 = off,
                               else 1..PSIM_MAX_INTERVAL trace rows per interval.  For every counted
                               row i (warm-up rows excluded, :197) of the first pass, interval
                               g = floor(i / interval) accumulates the Clock advance of i's step,
                               the queue entries retired in that step, those of them that are
                               stores (attribute 8), and 2^attr34 bytes if i is a load or store
                               (attributes 7, 8) whose data level (attribute 14) is 2 = memory
                               (:314).  Read with psim_get_interval_metrics.                    */
} psim_opts;

typedef struct {
    uint32_t arch;      /* PSIM_ARCH_*                                                      */
    uint32_t rows;      /* input rows, must be 112 (111 instructions + 1 zero row, R11)     */
    uint32_t features;  /* input features, must be 50                         */
    uint32_t reserved;  /* 0                                                                */
} psim_model_desc;

typedef struct {
    uint64_t k_hist[112];     /* histogram of context rows k at prediction (Fig. 14 analog) */
    uint64_t stalls;          /* ROB-full stall jumps (R5)                                  */
    uint64_t steps;           /* lockstep steps of the last simulate                        */
    uint64_t simulated;       /* instruction-simulations incl. warm-up, this rank          */
    uint64_t counted;         /* real instructions (warm-up excluded), this rank           */
    uint64_t subtraces;       /* sub-traces owned by this rank                             */
    uint64_t h2d_bytes;       /* trace bytes copied host->device by the last simulate      */
    uint64_t gpu_launches;    /* kernels launched by the last simulate                     */
    double sim_ms;            /* device time of the last simulate (CUDA events), ms        */
    double load_ms;           /* device time spent in trace loading before/while stepping  */
    int64_t local_cycles;     /* sum of this rank's sub-trace cycles                       */
    int32_t trace_mode;       /* 0 device-resident, 1 pinned host (zero-copy loader), 2 pageable */
    int32_t comm_ranks;       /* ranks of the NCCL communicator the last simulate reduced over (0: none) */
    double kernel_ms[8];      /* PSIM_PROFILE: summed device time per kernel class          */
    uint64_t kernel_launches[8]; /* launches per kernel class                               */
    uint64_t layer_m[4];      /* GEMM rows per launch of layers 0..3 (M = sub-traces x positions) */
    uint32_t layer_n[4], layer_k[4];  /* GEMM N and K of layers 0..3 (device shapes)        */
    uint64_t corrected;       /* rows re-simulated by post-error correction (0 if off)       */
    uint64_t corr_steps;      /* lockstep steps of the correction pass                      */
} psim_stats;

/* Create a context on opts->device.  world_size > 1 with nccl_id != NULL
 * initialises an NCCL communicator (collective over all ranks; every rank
 * must call it).
 * *out is NULL on failure.  PSIM_ERR_ARG for bad options. */
int psim_create(const psim_opts* opts, psim_ctx** out);

/* Free all device/host resources.  NULL-safe. */
void psim_destroy(psim_ctx* ctx);

/* Borrow an encoded trace: n_instr = L instructions in total,
 * of which this buffer holds rows [first_row, first_row + n_rows), row r at
 * attrs + (r - first_row) * row_stride, n_attr (= 47) attribute bytes each
 * (row_stride >= 48, a multiple of 16 for device buffers).  attrs may be device
 * memory (used in place: the "inputs resident in HBM" mode), pinned host
 * memory (streamed by a zero-copy loader kernel during simulate) or pageable
 * host memory (staged).  The buffer must stay valid until psim_simulate
 * returns; nothing is copied here (the trace crosses PCIe once, inside
 * simulate).  Resets a previous partition if L changes. */
int psim_load_trace(psim_ctx* ctx, const uint8_t* attrs, uint64_t n_instr, uint64_t first_row,
                    uint64_t n_rows, uint32_t n_attr, uint64_t row_stride);

/* Partition the L instructions into n_subtraces disjoint sub-traces
 * [s_j, e_j), s_j = floor(j*L/N) (Fig. 5; R8), each preceded by
 * warm-up rows [max(0, s_j - W), s_j) whose cycles are discarded (:197; R9).
 * Rank g of G owns sub-traces [floor(g*N/G), floor((g+1)*N/G)).  Errors:
 * N = 0 or N > L (ARG); the loaded rows must cover this rank's range
 * [max(0, s_first - W), e_last) (ARG). */
int psim_partition(psim_ctx* ctx, uint64_t n_subtraces, uint64_t warmup);

/* Copy the model (PyTorch layouts, fp32, layers in order: conv weight
 * [Cout][Cin][k] then bias, linear weight [out][in] then bias; FC1 columns
 * position-major, R11) to the device, repacked for the kernels.  The caller
 * may free weights on return.  ARG if n_floats does not match the arch,
 * UNSUPPORTED if the arch/precision pair is not built. */
int psim_load_model(psim_ctx* ctx, const psim_model_desc* desc, const float* weights, uint64_t n_floats);

/* Run the whole lockstep simulation of this rank's sub-traces: for every step,
 * gather -> batched CNN -> rounding -> queue update, then
 * reduce the per-sub-trace cycles and (world_size > 1) all-reduce them over
 * NCCL -- the single gather of Clocks.  Collective; blocking. */
int psim_simulate(psim_ctx* ctx);

/* Total simulated cycles summed over all sub-traces of all ranks
 * (N = 1: the final Clock).  STATE before a simulate. */
int psim_total_cycles(const psim_ctx* ctx, int64_t* out);

/* Human-readable description of the last error (valid until the next call). */
const char* psim_last_error(const psim_ctx* ctx);

/* ------------------------- diagnostics / parity -------------------------- */

/* Teacher forcing (parity stage S1): use lat3[3*i .. 3*i+2] = (f, c, s) as the
 * prediction of instruction i instead of the CNN.  lat3 covers all L rows
 * (host pointer, copied).  Pass NULL to return to CNN mode. */
int psim_force_latencies(psim_ctx* ctx, const uint16_t* lat3, uint64_t n_instr);

/* Per-instruction outputs of the last simulate for real rows [first, first+n)
 * of this rank (requires PSIM_RECORD_ROWS): (f, c, s) into out3 [n][3], the
 * context row count k into k (int32, may be NULL) and the Clock after the
 * update into clock (int64, may be NULL).  Rows outside this rank's sub-traces
 * are ARG. */
int psim_get_rows(const psim_ctx* ctx, uint64_t first, uint64_t n, uint16_t* out3, int32_t* k,
                  int64_t* clock);

/* Raw CNN outputs of the last simulate for real rows [first, first + n) of
 * this rank: out3 [n][3] fp32 (fetch, complete, store before rounding)
 * exactly as the hot path computed them (the fused bf16 C3 kernels, the
 * layer-wise GEMMs or the fp32 SIMT path -- whichever simulate ran), for the
 * step that predicted each row.  Requires PSIM_RECORD_ROWS and a CNN run
 * (a model loaded and either no teacher forcing or PSIM_FORCE_PREDICT);
 * otherwise STATE.  Rows outside this rank's sub-traces are ARG.  Parity
 * stage S2 of the hot path: with PSIM_FORCE_PREDICT and the oracle's
 * latencies forced, the inputs are the oracle's, element by element. */
int psim_get_outputs(const psim_ctx* ctx, uint64_t first, uint64_t n, float* out3);

/* Cycles of local sub-traces [first, first + n) (index relative to this
 * rank's first sub-trace) into out (int64). */
int psim_get_subtrace_cycles(const psim_ctx* ctx, uint64_t first, uint64_t n, int64_t* out);

/* Post-error correction of local sub-traces [first, first + n) (opts.correction_limit
 * > 0): corr_len[i] = rows of sub-trace first+i re-simulated by its predecessor
 * (0: not corrected), cycles1[i] = its first-pass cycles (before the
 * replacement).  Either pointer may be NULL.  STATE if correction was off. */
int psim_get_corrections(const psim_ctx* ctx, uint64_t first, uint64_t n, int32_t* corr_len, int64_t* cycles1);

/* The re-simulation's (f, c, s) and context count k of real rows
 * [first, first + n) (requires PSIM_RECORD_ROWS and correction): rows that were
 * not re-simulated get k = -1 and (f, c, s) = 0.  Rows outside this rank are ARG. */
int psim_get_corrected_rows(const psim_ctx* ctx, uint64_t first, uint64_t n, uint16_t* out3, int32_t* k);

/* This rank's sub-trace block [j0, j1) and trace rows [row_lo, row_hi). */
/* Interval metrics of the last simulate (psim_opts.interval > 0; PAPER.md:310-318,
 * DESIGN.md R20): for global intervals g = first .. first+n-1 (g < ceil(L / interval)),
 * cycles[g] (Clock advance), retired[g] (retire events), retired_st[g] (of which
 * stores) and mem_bytes[g] (data served by memory), summed over every sub-trace
 * of every rank (one ncclAllReduce when the context has a communicator, else this
 * rank's part).  CPI_g = cycles / retired, bandwidth_g = mem_bytes / cycles
 * (bytes per cycle).  Any output pointer may be NULL.  Host arrays of n int64.
 * Metrics come from the first pass (post-error correction does not change them).
 * PSIM_ERR_STATE if interval was 0 or before simulate; PSIM_ERR_ARG if out of range. */
int psim_get_interval_metrics(const psim_ctx* ctx, uint64_t first, uint64_t n, int64_t* cycles,
                              int64_t* retired, int64_t* retired_st, int64_t* mem_bytes);

int psim_rank_range(const psim_ctx* ctx, uint64_t* j0, uint64_t* j1, uint64_t* row_lo, uint64_t* row_hi);

/* Pure host helper (no context, no GPU): the sub-trace block [j0, j1), trace
 * rows [row_lo, row_hi) and lockstep step count of rank g of G for an N-way
 * partition of L rows with W warm-up (the rule of psim_partition). */
int psim_partition_range(uint64_t L, uint64_t N, uint64_t W, int rank, int world_size, uint64_t* j0,
                         uint64_t* j1, uint64_t* row_lo, uint64_t* row_hi, uint64_t* steps);

/* Statistics of the last simulate. */
int psim_get_stats(const psim_ctx* ctx, psim_stats* out);

/* Batched CNN forward on caller inputs (parity stage S2): X host [B][112][50]
 * fp32 (the instruction-major input of PAPER.md:93), Y host [B][3] fp32 raw
 * outputs before rounding.  Runs the layer-wise lowering of the loaded model
 * (gather-free: the inputs are given): per-layer tcgen05 GEMMs for bf16, SIMT
 * GEMMs for fp32.  The fused bf16 C3 kernels that simulate runs by default
 * build their inputs from the queue and cannot take caller inputs; their raw
 * outputs are read with psim_get_outputs. */
int psim_cnn_forward(psim_ctx* ctx, const float* X, uint64_t B, float* Y);

/* Name of kernel class i (0 <= i < PSIM_KC_COUNT), or NULL. */
const char* psim_kernel_class_name(int i);

/* Fill out[128] with a fresh ncclUniqueId (call on rank 0, broadcast the bytes
 * to the other ranks, pass them as psim_opts.nccl_id).  PSIM_ERR_NCCL if NCCL
 * cannot be loaded. */
int psim_nccl_unique_id(void* out128);

/* Library build string (compiler, arch, kernels). */
const char* psim_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PSIM_H */
