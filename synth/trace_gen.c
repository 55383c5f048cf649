/*
 * trace_gen.c -- seeded synthetic SPEC-like instruction trace generator.
 *
 * INPUT GENERATOR shared by the oracle tests and the product benchmarks.  It
 * holds none of the method's arithmetic (no queue, no clock, no CNN): it only
 * writes encoded instruction rows, the input of PAPER.md:87-89 ("each
 * instruction ... is represented by an array of 50 entries of instruction
 * attributes ... static properties ... and dynamic processor states").
 *
 * Row layout (47 attribute bytes + 1 pad byte; the CNN
 * column of attribute a is a + 3, R1):
 *   0 op class 0..15          1..10 flags (control, cond, call, return,
 *   indirect, mispredicted, load, store, serializing, barrier)
 *   11 fetch level (0 L1I, 1 L2, 2 memory; the 0/1/2 code of PAPER.md:312)
 *   12 ITLB walk depth 0..3   13 fetch waits for writeback
 *   14 data level 0/1/2       15 DTLB walk depth    16 data waits for wb
 *   17 store->load dependency distance bucket 0..7
 *   18..25 source registers (0 none, 1..96)   26..31 destination registers
 *   32 is_microop  33 is_last_microop  34 log2 access size  35..46 reserved
 *
 * Structure: four phase profiles (int, fp, mem-bound, branchy), each with a
 * static program of 4096 instructions in basic blocks; the dynamic trace
 * walks loops (geometric trip counts, mean 20).  Randomness is counter based:
 * segment g (4096 rows) is generated from splitmix64(seed, g) alone, so any
 * row range is regenerated identically and in parallel.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define SEG 4096
#define PROG 4096
#define NPROF 4
#define EPOCH_SEGS 64 /* phase switches every 64 segments = 262,144 rows */

static inline uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
typedef struct { uint64_t s; } rng_t;
static inline uint64_t rnext(rng_t* r) { r->s += 0x9E3779B97F4A7C15ULL; return mix64(r->s); }
static inline double runif(rng_t* r) { return (double)(rnext(r) >> 11) * (1.0 / 9007199254740992.0); }
static inline int rint_(rng_t* r, int n) { return (int)(runif(r) * n); }
static inline int rgeom(rng_t* r, double mean) { /* >= 1 */
    int k = 1; double p = 1.0 / mean;
    while (runif(r) > p && k < 64) k++;
    return k;
}

typedef struct {
    double mem, fp, br_block_mean, mispredict, l1d_miss, l2_miss_frac, icache_miss;
} profile_t;
static const profile_t PROFILES[NPROF] = {
    /* int       */ {0.35, 0.03, 6.0, 0.03, 0.03, 0.20, 0.003},
    /* fp        */ {0.30, 0.40, 12.0, 0.01, 0.05, 0.25, 0.001},
    /* mem-bound */ {0.40, 0.05, 8.0, 0.03, 0.20, 0.40, 0.002},
    /* branchy   */ {0.30, 0.02, 4.5, 0.06, 0.04, 0.20, 0.010},
};

typedef struct {
    uint8_t op, ctrl, cond, call, ret, indirect, load, store, serial, barrier;
    uint8_t src[8], dst[6], micro, last_micro, log2size;
    int block_end;    /* 1 if this instruction ends its basic block */
    int loop_head;    /* static index of the loop head for the block's branch */
    int latch;        /* block-ending branch is a loop latch (taken with p = 1 - 1/20) */
} sinst_t;

typedef struct { uint64_t seed; int ready; sinst_t prog[NPROF][PROG]; } programs_t;
static programs_t* g_prog = NULL;

static void build_program(uint64_t seed, int p, sinst_t* P) {
    rng_t r = {mix64(seed * 0x9E3779B97F4A7C15ULL + 0x1000 + p)};
    const profile_t* pf = &PROFILES[p];
    int recent[16] = {0}; int nrec = 0;
    int i = 0;
    while (i < PROG) {
        int bsize = 2 + rgeom(&r, pf->br_block_mean - 2.0);   /* >= 3, mean ~ br_block_mean + 1 */
        int head = i;
        int back = rint_(&r, 4);                 /* loop body spans 1..4 blocks */
        for (int b = 0; b < back && head > 0; b++) {
            int h = head - 1;
            while (h > 0 && !P[h - 1].block_end) h--;
            head = h;
        }
        int in_micro = 0;
        for (int t = 0; t < bsize && i < PROG; t++, i++) {
            sinst_t* s = &P[i];
            memset(s, 0, sizeof(*s));
            int last = (t == bsize - 1) || (i == PROG - 1);
            double u = runif(&r);
            if (last) {
                s->op = 13; s->ctrl = 1;
                double v = runif(&r);
                if (v < 0.04) { s->call = 1; }
                else if (v < 0.08) { s->ret = 1; s->indirect = 1; }
                else if (v < 0.10) { s->indirect = 1; }
                else { s->cond = 1; s->latch = runif(&r) < 0.3; }
            } else if (u < pf->mem) {
                int isst = runif(&r) < 0.33;
                int isfp = runif(&r) < pf->fp;
                s->op = isst ? (isfp ? 12 : 10) : (isfp ? 11 : 9);
                s->load = !isst; s->store = isst;
                s->log2size = (uint8_t)(isfp ? 3 + rint_(&r, 2) : rint_(&r, 4));
            } else if (u < pf->mem + pf->fp) {
                static const uint8_t fpops[5] = {4, 5, 6, 7, 8};
                s->op = fpops[rint_(&r, 5)];
            } else {
                double v = runif(&r);
                s->op = v < 0.80 ? 1 : v < 0.92 ? 2 : v < 0.95 ? 3 : v < 0.985 ? 15 : v < 0.995 ? 0 : 14;
                if (s->op == 14) { s->serial = 1; s->barrier = runif(&r) < 0.5; }
            }
            /* sources: recently written destinations (geometric distance, mean 4) */
            int nsrc = s->op == 0 ? 0 : 1 + rint_(&r, s->store ? 3 : 2);
            for (int k = 0; k < nsrc; k++) {
                int d = rgeom(&r, 4.0);
                s->src[k] = (uint8_t)(d <= nrec ? recent[(nrec - d) % 16] : 1 + rint_(&r, 96));
            }
            int ndst = (s->store || s->ctrl || s->op == 0) ? (s->call ? 1 : 0) : 1 + (runif(&r) < 0.1);
            for (int k = 0; k < ndst; k++) {
                int reg = 1 + rint_(&r, 96);
                s->dst[k] = (uint8_t)reg;
                recent[nrec % 16] = reg; nrec++;
            }
            if (!last && !in_micro && runif(&r) < 0.05) in_micro = 2 + rint_(&r, 3);
            if (in_micro) { s->micro = 1; in_micro--; s->last_micro = (in_micro == 0); }
            s->block_end = last;
            s->loop_head = head;
        }
    }
}

static const sinst_t* programs(uint64_t seed, int p) {
    if (!g_prog) g_prog = (programs_t*)calloc(1, sizeof(programs_t));
    if (!g_prog->ready || g_prog->seed != seed) {
        for (int q = 0; q < NPROF; q++) build_program(seed, q, g_prog->prog[q]);
        g_prog->seed = seed; g_prog->ready = 1;
    }
    return g_prog->prog[p];
}

static void gen_segment(uint64_t seed, int64_t g, int64_t r0, int64_t r1, uint8_t* out,
                        long stride, int64_t out_base) {
    int phase = (int)(mix64(seed ^ (0xABCDEF12345ULL + (uint64_t)(g / EPOCH_SEGS))) % NPROF);
    const sinst_t* P = programs(seed, phase);
    const profile_t* pf = &PROFILES[phase];
    rng_t r = {mix64(seed * 0xD1B54A32D192ED03ULL ^ (uint64_t)g * 0x9E3779B97F4A7C15ULL)};
    int pc = rint_(&r, PROG);
    while (pc > 0 && !P[pc - 1].block_end) pc--;    /* start at a block head */
    int64_t row0 = g * SEG;
    for (int64_t row = row0; row < row0 + SEG && row < r1; row++) {
        const sinst_t* s = &P[pc];
        uint8_t a[48];
        memset(a, 0, sizeof(a));
        a[0] = s->op; a[1] = s->ctrl; a[2] = s->cond; a[3] = s->call; a[4] = s->ret;
        a[5] = s->indirect; a[7] = s->load; a[8] = s->store; a[9] = s->serial; a[10] = s->barrier;
        /* fetch side */
        if (runif(&r) < pf->icache_miss) a[11] = runif(&r) < 0.2 ? 2 : 1;
        if (runif(&r) < 0.002) a[12] = (uint8_t)(1 + rint_(&r, 3));
        if (a[11] && runif(&r) < 0.1) a[13] = 1;
        /* data side */
        if (s->load || s->store) {
            if (runif(&r) < pf->l1d_miss) a[14] = runif(&r) < pf->l2_miss_frac ? 2 : 1;
            if (runif(&r) < 0.005) a[15] = (uint8_t)(1 + rint_(&r, 3));
            if (a[14] && runif(&r) < 0.05) a[16] = 1;
            if (s->load && runif(&r) < 0.1) a[17] = (uint8_t)(1 + rint_(&r, 7));
        }
        for (int k = 0; k < 8; k++) a[18 + k] = s->src[k];
        for (int k = 0; k < 6; k++) a[26 + k] = s->dst[k];
        a[32] = s->micro; a[33] = s->last_micro; a[34] = s->log2size;
        /* control flow: loops (mean trip 20), calls jump, the rest fall through */
        int next = pc + 1;
        if (s->ctrl) {
            int taken;
            if (s->cond) taken = runif(&r) < (s->latch ? 1.0 - 1.0 / 20.0 : 0.5);
            else taken = 1;
            if (s->cond && runif(&r) < pf->mispredict) a[6] = 1;
            if (taken) {
                if (s->cond && s->latch) next = s->loop_head;
                else if (s->cond) {              /* forward branch: skip the next block */
                    next = pc + 1;
                    while (next < PROG && !P[next - 1].block_end) next++;
                    next++;
                    while (next < PROG && next > 0 && !P[next - 1].block_end) next++;
                }
                else {
                    next = rint_(&r, PROG);
                    while (next > 0 && !P[next - 1].block_end) next--;
                }
            }
        }
        pc = next >= PROG ? 0 : next;
        if (row >= r0) memcpy(out + (size_t)(row - out_base) * stride, a, stride < 48 ? stride : 48);
    }
}

/* Write rows [r0, r1) of the trace with the given seed into out (row r at
 * out + (r - r0) * stride, stride >= 48).  Thread-parallel over segments. */
int synth_trace(uint64_t seed, int64_t r0, int64_t r1, uint8_t* out, long stride) {
    if (r1 < r0 || stride < 48) return -1;
    if (r1 == r0) return 0;
    (void)programs(seed, 0);             /* build the static programs once */
    int64_t g0 = r0 / SEG, g1 = (r1 + SEG - 1) / SEG;
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t g = g0; g < g1; g++) gen_segment(seed, g, r0, r1, out, stride, r0);
    return 0;
}
