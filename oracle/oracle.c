/*
 * oracle.c -- plain, slow, single-threaded CPU oracle for parallel sub-trace
 * ML microarchitecture simulation (Pandey et al., SC'22).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * It shares no code, header, table or constant generator with the CUDA
 * product path (paper_conf_sc_pandeylfhl22_b200/); it is built with gcc
 * from this one file and called through ctypes (oracle/__init__.py).
 *
 * Citations are PAPER.md:<line> (/root/reference/PAPER.md, section in
 * brackets) or DESIGN.md reading R<n> (readings of silent/garbled text; the
 * same list as SURVEY.md §8c O1..O15).
 *
 * Numeric modes
 *   ORACLE_FP64 (0): everything in double; the CNN is the exact definition.
 *   ORACLE_BF16 (1): every operand of a tensor-core layer (all layers but the
 *     last linear) -- the layer input and its weights -- is rounded to bf16
 *     (IEEE round-to-nearest-even) before use; products and sums in double;
 *     bias in double.  The last linear (fc2) takes the unrounded fc1
 *     activations and fp32 weights (R16).  This fixes the same
 *     rounding points as the bf16 GPU path, not its summation order.
 *
 * Pins (tests/test_oracle_*.py): hand trace of PAPER.md:105-107 and the
 * 20-instruction table (tests/golden/hand_trace_cap4.txt), a brute-force
 * definition simulator, closed forms (N=1 identity, W>=s_j identity,
 * context-free total = sum f), shift invariance, CNN == torch.nn.functional
 * in float64, rounding special cases.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_ROWS 112     /* 111 instruction rows + 1 zero row (R11) */
#define ORACLE_FEAT 50      /* 50 entries per instruction               */
#define ORACLE_NATTR 47     /* 47 trace attributes + 3 time features (R1)             */
#define ORACLE_MAXCAP 110   /* Context_length = 111 - 1                 */
#define ORACLE_LAT_MAX 4095 /* R7 */
#define ORACLE_TIME_MAX 65535

enum { ORACLE_FP64 = 0, ORACLE_BF16 = 1 };
enum { ARCH_M2 = 1, ARCH_C3 = 2, ARCH_RB7 = 3 };

/* ------------------------------------------------------------------ */
/* bf16 rounding: IEEE binary32 -> bfloat16 round-to-nearest-even,     */
/* applied to the exact double value (R16).                            */
/* ------------------------------------------------------------------ */
static double bf16_round(double x) {
    /* bf16 has an 8-bit significand; round x to 8 significant bits, ties to
     * even, keeping binary32 exponent range (values here are far from the
     * subnormal/overflow range; both are handled by frexp/ldexp anyway). */
    if (x == 0.0 || isnan(x) || isinf(x)) return x;
    int e;
    double m = frexp(x, &e);           /* x = m * 2^e, 0.5 <= |m| < 1 */
    double scaled = ldexp(m, 8);       /* 8 significant bits in the integer part */
    double r = nearbyint(scaled);      /* default rounding mode: to nearest even */
    return ldexp(r, e - 8);
}

/* ------------------------------------------------------------------ */
/* Model: SimNet-style 1-D CNN over the 112x50 instruction matrix.     */
/* Conv1d takes features as channels and instructions as length       */
/* (the transpose SimNet performs); R11 fixes the   */
/* shapes.  Weight layout: PyTorch (conv.weight [Cout][Cin][k], bias   */
/* [Cout], linear.weight [out][in], bias [out]), layers in order.      */
/* FC1 flattens position-major: index = p*C + c (R11).                */
/* ------------------------------------------------------------------ */
typedef struct { int type, cin, cout, k, stride, pad, relu, res_begin, res_add; } layer_t;
enum { L_CONV = 0, L_LINEAR = 1 };

static int arch_layers(int arch, layer_t* L) {
    int n = 0;
    if (arch == ARCH_M2) {            /* "2-conv-layer" model, config 1 */
        L[n++] = (layer_t){L_CONV, 50, 64, 2, 2, 0, 1, 0, 0};
        L[n++] = (layer_t){L_CONV, 64, 64, 2, 2, 0, 1, 0, 0};
        L[n++] = (layer_t){L_LINEAR, 28 * 64, 256, 0, 0, 0, 1, 0, 0};
        L[n++] = (layer_t){L_LINEAR, 256, 3, 0, 0, 0, 0, 0, 0};
    } else if (arch == ARCH_C3) {     /* "3C+2F", 64 conv1 channels (:161) */
        L[n++] = (layer_t){L_CONV, 50, 64, 2, 2, 0, 1, 0, 0};
        L[n++] = (layer_t){L_CONV, 64, 128, 2, 2, 0, 1, 0, 0};
        L[n++] = (layer_t){L_CONV, 128, 128, 2, 2, 0, 1, 0, 0};
        L[n++] = (layer_t){L_LINEAR, 14 * 128, 256, 0, 0, 0, 1, 0, 0};
        L[n++] = (layer_t){L_LINEAR, 256, 3, 0, 0, 0, 0, 0, 0};
    } else if (arch == ARCH_RB7) {    /* deeper residual variant (config 5, R11) */
        L[n++] = (layer_t){L_CONV, 50, 64, 2, 2, 0, 1, 0, 0};
        for (int b = 0; b < 3; b++) {
            /* y = relu(x + conv_b(relu(conv_a(x)))) */
            L[n++] = (layer_t){L_CONV, 64, 64, 3, 1, 1, 1, 1, 0};
            L[n++] = (layer_t){L_CONV, 64, 64, 3, 1, 1, 1, 0, 1};
        }
        L[n++] = (layer_t){L_LINEAR, 56 * 64, 256, 0, 0, 0, 1, 0, 0};
        L[n++] = (layer_t){L_LINEAR, 256, 3, 0, 0, 0, 0, 0, 0};
    } else {
        return -1;
    }
    return n;
}

static long layer_nparams(const layer_t* l) {
    if (l->type == L_CONV) return (long)l->cout * l->cin * l->k + l->cout;
    return (long)l->cout * l->cin + l->cout;
}

long oracle_arch_nparams(int arch) {
    layer_t L[16];
    int n = arch_layers(arch, L);
    if (n < 0) return -1;
    long t = 0;
    for (int i = 0; i < n; i++) t += layer_nparams(&L[i]);
    return t;
}

/* Effective weights: the fp32 file values as double, rounded to bf16 for the
 * tensor-core layers in ORACLE_BF16 mode (operand rounding, R16).  Done once
 * per simulation; the same values are used for every instruction. */
static double* effective_weights(int arch, int mode, const float* weights, long n) {
    layer_t L[16];
    int nl = arch_layers(arch, L);
    double* W = (double*)malloc(sizeof(double) * (size_t)n);
    long off = 0;
    for (int li = 0; li < nl; li++) {
        long nw = layer_nparams(&L[li]) - L[li].cout;          /* weights, then bias */
        for (long t = 0; t < nw; t++) {
            double v = (double)weights[off + t];
            W[off + t] = (mode == ORACLE_BF16 && li != nl - 1) ? bf16_round(v) : v;
        }
        for (long t = nw; t < nw + L[li].cout; t++) W[off + t] = (double)weights[off + t];
        off += nw + L[li].cout;
    }
    return W;
}

/* Forward pass for one 112x50 input (row-major [row][feature]) with effective
 * weights We.  Activations are kept as act[position][channel]. */
static int forward(int arch, int mode, const double* We, const double* X, double* y_out) {
    layer_t L[16];
    int nl = arch_layers(arch, L);
    if (nl < 0) return -1;
    static double cur[ORACLE_ROWS * 256], nxt[ORACLE_ROWS * 256], skip[ORACLE_ROWS * 256];
    int len = ORACLE_ROWS, ch = ORACLE_FEAT;
    for (int i = 0; i < len * ch; i++) cur[i] = X[i];
    int flat = 0; /* after the first linear the activation is a vector */
    int skip_ch = 0;
    const double* w = We;

    for (int li = 0; li < nl; li++) {
        const layer_t* l = &L[li];
        int tensor_core = (li != nl - 1);   /* R16: every layer but the last */
        const double* Wt = w;
        const double* B = w + (l->type == L_CONV ? (long)l->cout * l->cin * l->k
                                                 : (long)l->cout * l->cin);
        w += layer_nparams(l);

        /* operand rounding of the layer input (bf16 mode) */
        if (mode == ORACLE_BF16 && tensor_core)
            for (int i = 0; i < len * ch; i++) cur[i] = bf16_round(cur[i]);

        if (l->res_begin) {                 /* remember block input x */
            for (int i = 0; i < len * ch; i++) skip[i] = cur[i];
            skip_ch = ch;
        }

        if (l->type == L_CONV) {
            /* out[p][o] = b[o] + sum_{t<k} sum_{c<Cin} W[o][c][t] * in[p*s + t - pad][c]
             * (zero outside [0, len)) -- the definition of Conv1d. */
            int olen = (len + 2 * l->pad - l->k) / l->stride + 1;
            for (int p = 0; p < olen; p++)
                for (int o = 0; o < l->cout; o++) {
                    double acc = 0.0;
                    for (int t = 0; t < l->k; t++) {
                        int r = p * l->stride + t - l->pad;
                        if (r < 0 || r >= len) continue;
                        for (int c = 0; c < l->cin; c++)
                            acc += Wt[((long)o * l->cin + c) * l->k + t] * cur[r * ch + c];
                    }
                    acc += B[o];
                    if (l->res_add) acc += skip[p * skip_ch + o];
                    if (l->relu && acc < 0.0) acc = 0.0;
                    nxt[p * l->cout + o] = acc;
                }
            len = olen; ch = l->cout;
        } else {
            /* Linear on the position-major flattening: in[i], i = p*C + c. */
            int nin = flat ? ch : len * ch;
            if (nin != l->cin) return -2;
            for (int o = 0; o < l->cout; o++) {
                double acc = 0.0;
                for (int i = 0; i < nin; i++) acc += Wt[(long)o * l->cin + i] * cur[i];
                acc += B[o];
                if (l->relu && acc < 0.0) acc = 0.0;
                nxt[o] = acc;
            }
            flat = 1; len = 1; ch = l->cout;
        }
        memcpy(cur, nxt, sizeof(double) * (size_t)len * ch);
    }
    if (ch != 3) return -3;
    for (int i = 0; i < 3; i++) y_out[i] = cur[i];
    return 0;
}

int oracle_cnn_forward(int arch, int mode, const float* weights, long n_weights,
                       const double* X, double* y_out) {
    if (oracle_arch_nparams(arch) < 0 || n_weights != oracle_arch_nparams(arch)) return -1;
    double* We = effective_weights(arch, mode, weights, n_weights);
    int rc = forward(arch, mode, We, X, y_out);
    free(We);
    return rc;
}

/* Rounding of a predicted latency (R7): the double output is taken to
 * binary32 (the precision the kernel decides in), rounded to the nearest
 * integer with ties to even (rint), clamped to [0, 4095]; NaN -> 0. */
int oracle_round_latency(double y) {
    float yf = (float)y;
    if (isnan(yf)) return 0;
    float r = nearbyintf(yf);
    if (r < 0.0f) return 0;
    if (r > (float)ORACLE_LAT_MAX) return ORACLE_LAT_MAX;
    return (int)r;
}

/* ------------------------------------------------------------------ */
/* Instruction queue (Fig. 1): entries in fetch order,    */
/* each with its retire clock; Clock starts at 0 (:91).               */
/* ------------------------------------------------------------------ */
typedef struct {
    int cap;                     /* live context entries after each step (<= 110) */
    int n;
    int64_t clock;
    int64_t stalls;
    int64_t seq[ORACLE_MAXCAP + 1];
    int64_t fetch[ORACLE_MAXCAP + 1], complete[ORACLE_MAXCAP + 1], retire[ORACLE_MAXCAP + 1];
} oracle_queue;

oracle_queue* oracle_queue_new(int cap, int64_t clock0) {
    if (cap < 1 || cap > ORACLE_MAXCAP) return NULL;
    oracle_queue* q = (oracle_queue*)calloc(1, sizeof(oracle_queue));
    q->cap = cap;
    q->clock = clock0;
    return q;
}
void oracle_queue_free(oracle_queue* q) { free(q); }
int64_t oracle_queue_clock(const oracle_queue* q) { return q->clock; }
int64_t oracle_queue_stalls(const oracle_queue* q) { return q->stalls; }
int oracle_queue_size(const oracle_queue* q) { return q->n; }
int oracle_queue_entries(const oracle_queue* q, int64_t* seq, int64_t* fetch,
                         int64_t* complete, int64_t* retire) {
    for (int i = 0; i < q->n; i++) {
        seq[i] = q->seq[i]; fetch[i] = q->fetch[i];
        complete[i] = q->complete[i]; retire[i] = q->retire[i];
    }
    return q->n;
}

static int64_t min64(int64_t a, int64_t b) { return a < b ? a : b; }
static int64_t max64(int64_t a, int64_t b) { return a > b ? a : b; }

/* Build the 112x50 input for instruction i (PAPER.md:93 concatenation,
 * :127 "current instruction is always in the first position", zero padding
 * at the tail).  Context rows newest-first (R6); time columns relative to
 * the current Clock (R2, R1).  Returns k = number of context rows. */
int oracle_build_input(const oracle_queue* q, const uint8_t* trace, long row_stride,
                       long i, double* X) {
    for (int t = 0; t < ORACLE_ROWS * ORACLE_FEAT; t++) X[t] = 0.0;
    const uint8_t* a = trace + (size_t)i * row_stride;
    for (int f = 0; f < ORACLE_NATTR; f++) X[3 + f] = (double)a[f];
    int r = 1;
    for (int e = q->n - 1; e >= 0; e--, r++) {
        double* row = X + r * ORACLE_FEAT;
        row[0] = (double)min64(ORACLE_TIME_MAX, q->clock - q->fetch[e]);
        row[1] = (double)min64(ORACLE_TIME_MAX, max64(0, q->complete[e] - q->clock));
        row[2] = (double)min64(ORACLE_TIME_MAX, q->retire[e] - q->clock);
        const uint8_t* ae = trace + (size_t)q->seq[e] * row_stride;
        for (int f = 0; f < ORACLE_NATTR; f++) row[3 + f] = (double)ae[f];
    }
    return q->n;
}

/* Remove every entry whose retire clock has elapsed ("Whenever the Clock
 * value is greater or equal to the retire clock, we remove the instruction",
 * PAPER.md:107), keeping fetch order.  Logs removals if asked. */
static void retire_elapsed(oracle_queue* q, int64_t* log_seq, int64_t* log_ret, int* n_log) {
    int w = 0;
    for (int e = 0; e < q->n; e++) {
        if (q->retire[e] <= q->clock) {
            if (log_seq) { log_seq[*n_log] = q->seq[e]; log_ret[*n_log] = q->retire[e]; }
            if (n_log) (*n_log)++;
            continue;
        }
        q->seq[w] = q->seq[e]; q->fetch[w] = q->fetch[e];
        q->complete[w] = q->complete[e]; q->retire[w] = q->retire[e];
        w++;
    }
    q->n = w;
}

/* Update after predicting (f, c, s) for instruction i:
 *   Clock += fetch latency;  retire clock = Clock_old + f + c + s (R3);
 *   push i (R4), retire everything with retire <= Clock;
 *   if more than cap entries remain: ROB-full stall, Clock = min retire,
 *   retire again (R5).
 * Returns the number of retired entries; *stalled = 1 if a stall happened. */
int oracle_queue_update(oracle_queue* q, long i, int f, int c, int s,
                        int64_t* log_seq, int64_t* log_ret, int* stalled) {
    int n_log = 0;
    q->clock += f;
    q->seq[q->n] = i;
    q->fetch[q->n] = q->clock;
    q->complete[q->n] = q->clock + c;
    q->retire[q->n] = q->clock + c + s;
    q->n++;
    retire_elapsed(q, log_seq, log_ret, &n_log);
    if (stalled) *stalled = 0;
    if (q->n > q->cap) {
        int64_t m = q->retire[0];
        for (int e = 1; e < q->n; e++) m = min64(m, q->retire[e]);
        q->clock = m;
        q->stalls++;
        if (stalled) *stalled = 1;
        retire_elapsed(q, log_seq ? log_seq : NULL, log_ret, &n_log);
    }
    return n_log;
}

/* ------------------------------------------------------------------ */
/* Partition (Fig. 5, warm-up :197; R8, R9):          */
/*   s_j = floor(j*L/N), e_j = s_{j+1}, warm-up start ws_j = max(0,s_j-W) */
/* ------------------------------------------------------------------ */
int oracle_partition(long L, long N, long W, int64_t* s, int64_t* e, int64_t* ws) {
    if (N <= 0 || N > L || W < 0) return -1;
    for (long j = 0; j < N; j++) {
        /* j*L fits int64 for L < 2^40, N < 2^23 */
        s[j] = (int64_t)(((__int128)j * L) / N);
        e[j] = (int64_t)(((__int128)(j + 1) * L) / N);
        ws[j] = s[j] - W > 0 ? s[j] - W : 0;
    }
    return 0;
}

/* ------------------------------------------------------------------ */
/* Simulate sub-traces [j0, j0+nj) of an N-way partition.              */
/*   forced_lat: uint16 [L][3] teacher-forced (f,c,s) per row, or NULL  */
/*               to use the CNN (arch, mode, weights).                 */
/*   Per real row i (s_j <= i < e_j), if the arrays are non-NULL:       */
/*     lat_out[3i..3i+2] = (f,c,s), y_out[3i..] = raw CNN outputs,      */
/*     k_out[i] = context rows at prediction, clock_out[i] = Clock after */
/*   cycles[j-j0] = Clock_end - boundary_j, boundary[j-j0] = Clock at   */
/*   the end of warm-up (clock0 if no warm-up).   */
/* Returns 0 on success.                                               */
/* ------------------------------------------------------------------ */
int oracle_simulate(int arch, int mode, const float* weights, long n_weights,
                    const uint8_t* trace, long row_stride, long L, long N, long W, int cap,
                    const uint16_t* forced_lat, long j0, long nj, int64_t clock0,
                    int64_t* cycles, int64_t* boundary, uint16_t* lat_out, float* y_out,
                    int32_t* k_out, int64_t* clock_out, int64_t* stalls_out) {
    if (N <= 0 || N > L || W < 0 || j0 < 0 || nj < 0 || j0 + nj > N) return -1;
    if (cap < 1 || cap > ORACLE_MAXCAP) return -1;
    if (!forced_lat && n_weights != oracle_arch_nparams(arch)) return -2;
    double* X = (double*)malloc(sizeof(double) * ORACLE_ROWS * ORACLE_FEAT);
    double* We = forced_lat ? NULL : effective_weights(arch, mode, weights, n_weights);
    int64_t total_stalls = 0;
    for (long j = j0; j < j0 + nj; j++) {
        int64_t s = (int64_t)(((__int128)j * L) / N);
        int64_t e = (int64_t)(((__int128)(j + 1) * L) / N);
        int64_t ws = s - W > 0 ? s - W : 0;
        oracle_queue* q = oracle_queue_new(cap, clock0);
        int64_t bnd = clock0;
        for (int64_t i = ws; i < e; i++) {
            int k = oracle_build_input(q, trace, row_stride, (long)i, X);
            int f, c, st;
            double y[3] = {0, 0, 0};
            if (forced_lat) {
                f = forced_lat[3 * i]; c = forced_lat[3 * i + 1]; st = forced_lat[3 * i + 2];
            } else {
                if (forward(arch, mode, We, X, y) != 0) {
                    free(X); free(We); oracle_queue_free(q); return -3;
                }
                f = oracle_round_latency(y[0]);
                c = oracle_round_latency(y[1]);
                st = oracle_round_latency(y[2]);
            }
            oracle_queue_update(q, (long)i, f, c, st, NULL, NULL, NULL);
            if (i == s - 1) bnd = q->clock;           /* end of warm-up */
            if (i >= s) {
                if (lat_out) { lat_out[3*i] = (uint16_t)f; lat_out[3*i+1] = (uint16_t)c; lat_out[3*i+2] = (uint16_t)st; }
                if (y_out) { y_out[3*i] = (float)y[0]; y_out[3*i+1] = (float)y[1]; y_out[3*i+2] = (float)y[2]; }
                if (k_out) k_out[i] = k;
                if (clock_out) clock_out[i] = q->clock;
            }
        }
        if (cycles) cycles[j - j0] = q->clock - bnd;
        if (boundary) boundary[j - j0] = bnd;
        total_stalls += q->stalls;
        oracle_queue_free(q);
    }
    if (stalls_out) *stalls_out = total_stalls;
    free(X);
    free(We);
    return 0;
}

/* ------------------------------------------------------------------ */
/* Post-error correction (PAPER.md:203-219 [V-B "Post-error           */
/* correction"], Fig. 9; limit :291; R19).                   */
/*                                                                     */
/* First pass: every sub-trace j in [j0, j0+nj) exactly as             */
/* oracle_simulate (warm-up is still used, :205).  Then "if this        */
/* partition is not the last one on the GPU, it will re-simulate the    */
/* following instructions, which were previously simulated by the next  */
/* partition" (:207): sub-trace j's final queue and Clock continue over */
/* rows i = s_{j+1}, s_{j+1}+1, ...  Before row i is re-simulated the    */
/* re-simulation's context count is compared with the count the first  */
/* pass of j+1 saw at row i; the re-simulation "continues until either  */
/* the number of context instructions of the re-simulation matches the */
/* prior outcomes or a user-defined resimulation limit" (:219): the     */
/* first matching row is not re-simulated (Fig. 9: partition 0          */
/* re-simulates {I4, I5}, terminating at I6), at most `limit` rows are  */
/* re-simulated, and never past e_{j+1}.  "The re-simulated cycles will */
/* replace the previously simulated ones" (:207):                       */
/*   cycles_{j+1} += (Clock_re,last - Clock_{j,end})                    */
/*                 - (Clock1_{j+1}(last re-simulated row) - bnd_{j+1}).  */
/* "We do not perform post-error correction for the first partition of */
/* each GPU" (:219): with G ranks (rank g owns [floor(gN/G),             */
/* floor((g+1)N/G))), j+1 is corrected only if j is on the same rank;   */
/* j+1 == j0 (j outside the simulated range) is not corrected either.   */
/* Sub-traces are processed in index order with j's first-pass final    */
/* state kept until j+1 has been corrected; the passes are independent  */
/* so this equals running all first passes before all corrections.      */
/*                                                                     */
/* Outputs as oracle_simulate (cycles are the CORRECTED cycles; the     */
/* per-row arrays hold the first pass), plus cycles1[j-j0] = first-pass */
/* cycles, corr_len[j-j0] = rows of sub-trace j re-simulated by j-1,    */
/* corr_lat[3i..] / corr_k[i] = the re-simulation's (f,c,s) and context */
/* count for each re-simulated row i (untouched elsewhere).             */
/* ------------------------------------------------------------------ */
static long rank_of(long j, long N, long G) {
    for (long g = 0; g < G; g++)
        if (j < (long)(((__int128)(g + 1) * N) / G)) return g;
    return G - 1;
}

/* one instruction: build input, predict (or take the forced latencies),
 * update the queue.  Returns the context count k; fills f/c/s and y. */
static int oracle_step(int arch, int mode, const double* We, double* X, oracle_queue* q,
                       const uint8_t* trace, long row_stride, const uint16_t* forced_lat, int64_t i,
                       int* lat3, double* y) {
    int k = oracle_build_input(q, trace, row_stride, (long)i, X);
    y[0] = y[1] = y[2] = 0.0;
    if (forced_lat) {
        lat3[0] = forced_lat[3 * i]; lat3[1] = forced_lat[3 * i + 1]; lat3[2] = forced_lat[3 * i + 2];
    } else {
        if (forward(arch, mode, We, X, y) != 0) return -1;
        for (int o = 0; o < 3; o++) lat3[o] = oracle_round_latency(y[o]);
    }
    oracle_queue_update(q, (long)i, lat3[0], lat3[1], lat3[2], NULL, NULL, NULL);
    return k;
}

int oracle_simulate_pec(int arch, int mode, const float* weights, long n_weights,
                        const uint8_t* trace, long row_stride, long L, long N, long W, int cap,
                        const uint16_t* forced_lat, long j0, long nj, long G, long limit,
                        int64_t* cycles, int64_t* cycles1, int64_t* boundary, int32_t* corr_len,
                        uint16_t* lat_out, int32_t* k_out, int64_t* clock_out,
                        uint16_t* corr_lat, int32_t* corr_k, int64_t* stalls_out) {
    if (N <= 0 || N > L || W < 0 || j0 < 0 || nj < 0 || j0 + nj > N) return -1;
    if (cap < 1 || cap > ORACLE_MAXCAP || G < 1 || G > N || limit < 0) return -1;
    if (!forced_lat && n_weights != oracle_arch_nparams(arch)) return -2;
    double* X = (double*)malloc(sizeof(double) * ORACLE_ROWS * ORACLE_FEAT);
    double* We = forced_lat ? NULL : effective_weights(arch, mode, weights, n_weights);
    int* k1 = (int*)malloc(sizeof(int) * (size_t)(limit + 1));          /* first pass of j: k per real row */
    int64_t* c1 = (int64_t*)malloc(sizeof(int64_t) * (size_t)(limit + 1));   /* Clock - bnd per real row */
    oracle_queue* prev = NULL;   /* final first-pass state of sub-trace j-1 */
    int64_t total_stalls = 0;
    int rc = 0;
    for (long j = j0; j < j0 + nj && rc == 0; j++) {
        int64_t s = (int64_t)(((__int128)j * L) / N);
        int64_t e = (int64_t)(((__int128)(j + 1) * L) / N);
        int64_t ws = s - W > 0 ? s - W : 0;
        /* ---- first pass of sub-trace j ---- */
        oracle_queue* q = oracle_queue_new(cap, 0);
        int64_t bnd = 0;
        for (int64_t i = ws; i < e; i++) {
            int lat3[3];
            double y[3];
            int k = oracle_step(arch, mode, We, X, q, trace, row_stride, forced_lat, i, lat3, y);
            if (k < 0) { rc = -3; break; }
            if (i == s - 1) bnd = q->clock;
            if (i >= s) {
                if (lat_out) for (int o = 0; o < 3; o++) lat_out[3 * i + o] = (uint16_t)lat3[o];
                if (k_out) k_out[i] = k;
                if (clock_out) clock_out[i] = q->clock;
                if (i - s < limit) { k1[i - s] = k; c1[i - s] = q->clock - bnd; }
            }
        }
        int64_t cyc = q->clock - bnd;
        if (cycles1) cycles1[j - j0] = cyc;
        if (boundary) boundary[j - j0] = bnd;
        total_stalls += q->stalls;
        /* ---- correction of j by j-1 ---- */
        int32_t n_re = 0;
        if (rc == 0 && prev && rank_of(j - 1, N, G) == rank_of(j, N, G)) {
            oracle_queue* r = prev;                    /* j-1's final state continues */
            const int64_t clock_start = r->clock, stalls_start = r->stalls;
            for (int64_t i = s; i < e && i - s < limit; i++) {
                if (r->n == k1[i - s]) break;          /* context counts match: stop */
                int lat3[3];
                double y[3];
                int k = oracle_step(arch, mode, We, X, r, trace, row_stride, forced_lat, i, lat3, y);
                if (k < 0) { rc = -3; break; }
                if (corr_lat) for (int o = 0; o < 3; o++) corr_lat[3 * i + o] = (uint16_t)lat3[o];
                if (corr_k) corr_k[i] = k;
                n_re++;
            }
            if (n_re > 0) cyc += (r->clock - clock_start) - c1[n_re - 1];
            total_stalls += r->stalls - stalls_start;  /* stalls of the re-simulation counted too */
        }
        if (corr_len) corr_len[j - j0] = n_re;
        if (cycles) cycles[j - j0] = cyc;
        if (prev) oracle_queue_free(prev);
        prev = q;
    }
    if (prev) oracle_queue_free(prev);
    if (stalls_out) *stalls_out = total_stalls;
    free(X); free(We); free(k1); free(c1);
    return rc;
}

/* ------------------------------------------------------------------ */
/* Interval metrics (PAPER.md:310-318 [VI-E "Predicting Other          */
/* Simulation Metrics"]; R20).                               */
/*                                                                     */
/* "the simulator tracks the instruction retire events in the          */
/* instruction queue at a certain interval ... The CPI is then computed */
/* as the ratio of the collective predicted instruction latency over   */
/* the number of retired instructions for an interval" and "store      */
/* instructions [retire out of order] ... We tracked store instructions */
/* separately" (:316).  "the memory bandwidth is the ratio of the       */
/* amount of data accessed from memory and the latency"; data counts    */
/* only for load/store instructions whose trace says the data came from */
/* memory (code 2, :314).                                               */
/*                                                                     */
/* Interval g holds the counted rows i (s_j <= i < e_j) with            */
/* floor(i / interval) == g.  For each such row, processed by the step  */
/* that predicts it:                                                   */
/*   cycles[g]   += Clock after the step - Clock before it (f + stall)  */
/*   retired[g]  += entries removed from the queue in that step         */
/*   retired_st[g] += those of them that are stores (attribute 8)       */
/*   mem_bytes[g] += 2^(attr 34) if row i is a load or store (attrs 7,8) */
/*                   with data level (attr 14) == 2, else 0             */
/* Warm-up rows contribute nothing (their cycles are discarded, :197).  */
/* CPI_g = cycles[g] / retired[g]; bandwidth_g = mem_bytes[g] /        */
/* cycles[g] (bytes per cycle).  Arrays are indexed by global interval  */
/* g in [0, ceil(L / interval)) and ADDED to (caller zeroes them).      */
/* Trace attribute indices: the row layout of SURVEY.md Appendix C     */
/* (the shared file format).                                           */
/* ------------------------------------------------------------------ */
#define ORACLE_A_LOAD 7
#define ORACLE_A_STORE 8
#define ORACLE_A_DLEVEL 14
#define ORACLE_A_LOG2SIZE 34

int oracle_simulate_metrics(int arch, int mode, const float* weights, long n_weights,
                            const uint8_t* trace, long row_stride, long L, long N, long W, int cap,
                            const uint16_t* forced_lat, long j0, long nj, long interval,
                            int64_t* cycles, int64_t* retired, int64_t* retired_st, int64_t* mem_bytes) {
    if (N <= 0 || N > L || W < 0 || j0 < 0 || nj < 0 || j0 + nj > N || interval < 1) return -1;
    if (cap < 1 || cap > ORACLE_MAXCAP) return -1;
    if (!forced_lat && n_weights != oracle_arch_nparams(arch)) return -2;
    double* X = (double*)malloc(sizeof(double) * ORACLE_ROWS * ORACLE_FEAT);
    double* We = forced_lat ? NULL : effective_weights(arch, mode, weights, n_weights);
    int64_t log_seq[2 * (ORACLE_MAXCAP + 2)], log_ret[2 * (ORACLE_MAXCAP + 2)];
    for (long j = j0; j < j0 + nj; j++) {
        int64_t s = (int64_t)(((__int128)j * L) / N);
        int64_t e = (int64_t)(((__int128)(j + 1) * L) / N);
        int64_t ws = s - W > 0 ? s - W : 0;
        oracle_queue* q = oracle_queue_new(cap, 0);
        for (int64_t i = ws; i < e; i++) {
            oracle_build_input(q, trace, row_stride, (long)i, X);
            int lat3[3];
            double y[3] = {0, 0, 0};
            if (forced_lat) {
                for (int o = 0; o < 3; o++) lat3[o] = forced_lat[3 * i + o];
            } else {
                if (forward(arch, mode, We, X, y) != 0) { free(X); free(We); oracle_queue_free(q); return -3; }
                for (int o = 0; o < 3; o++) lat3[o] = oracle_round_latency(y[o]);
            }
            const int64_t clock_before = q->clock;
            int n_ret = oracle_queue_update(q, (long)i, lat3[0], lat3[1], lat3[2], log_seq, log_ret, NULL);
            if (i < s) continue;                       /* warm-up row: discarded (:197) */
            const int64_t g = i / interval;
            cycles[g] += q->clock - clock_before;
            retired[g] += n_ret;
            for (int r = 0; r < n_ret; r++)
                if (trace[(size_t)log_seq[r] * row_stride + ORACLE_A_STORE]) retired_st[g]++;
            const uint8_t* a = trace + (size_t)i * row_stride;
            if ((a[ORACLE_A_LOAD] || a[ORACLE_A_STORE]) && a[ORACLE_A_DLEVEL] == 2)
                mem_bytes[g] += (int64_t)1 << a[ORACLE_A_LOG2SIZE];
        }
        oracle_queue_free(q);
    }
    free(X);
    free(We);
    return 0;
}
