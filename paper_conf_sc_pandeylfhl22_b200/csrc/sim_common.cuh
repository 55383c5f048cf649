// sim_common.cuh -- the integer queue update of one sub-trace, executed by one
// warp (R3-R5, R7).  Shared by the standalone
// update kernel (sim_kernels.cu) and the fused fc1/head/update kernel
// (fused_c3.cu).  Product side only.
#pragma once
#include "internal.h"

namespace psim {

__device__ __forceinline__ int lat_round(float y) {
  // R7: nearest integer, ties to even, on the fp32 value; NaN -> 0; clamp [0, 4095]
  if (isnan(y)) return 0;
  float r = rintf(y);
  if (r < 0.f) return 0;
  if (r > (float)kLatMax) return kLatMax;
  return (int)r;
}

// Post-error correction bookkeeping after the update of row i (R19).
// First pass (k1_rec): record the context count k seen at real row s_b + t and
// Clock - bnd after it, t < limit.  Correction pass (kref): corrector b stops
// when its new count equals the first-pass count of sub-trace b+1 at the next
// row; its re-simulated cycles go to st.cycles[b] and st.e[b]
// marks the end.  Returns true if the corrector stopped.
__device__ __forceinline__ bool pec_record_or_stop(const UpdateArgs& a, uint64_t b, int64_t i, int64_t s_b,
                                                   int64_t nsteps, int k, int knew, int64_t clock, int64_t bnd) {
  if (a.k1_rec && i >= s_b && i - s_b < a.limit) {
    const uint64_t o = (uint64_t)(i - s_b) * a.st.n + b;
    a.k1_rec[o] = (uint8_t)k;
    a.c1_rec[o] = (uint32_t)(clock - bnd);
  }
  if (a.kref) {
    const int64_t t1 = a.step + 1;
    if (t1 < nsteps && knew == (int)a.kref[(uint64_t)t1 * a.st.n + b + 1]) {
      a.st.cycles[b] = clock - bnd;
      a.st.e[b] = i + 1;
      return true;
    }
  }
  return false;
}

// Interval metrics after the update of counted row i (PAPER.md:310-318 [VI-E];
// DESIGN.md R20): the sub-trace keeps {retired, retired stores, Clock lo at the
// start of its current interval segment} in macc[b] and adds them to interval
// i / I when the segment ends (last row of the interval or of the sub-trace).
// Memory bytes are rare (memory-served loads/stores) and added at once.
// Segment Clock advance < 2^32 for I <= PSIM_MAX_INTERVAL (<= 12285 per row).
__device__ __forceinline__ void metrics_row(const UpdateArgs& a, uint64_t b, int64_t i, int64_t s_b,
                                            int64_t nsteps, uint32_t clo_before, uint32_t clo_after, int nret,
                                            int nst, uint32_t code) {
  if (!a.macc || i < s_b) return;
  const int64_t I = a.interval;
  const int64_t g = i / I;
  const int64_t r = i - g * I;
  uint4 acc = (i == s_b || r == 0) ? make_uint4(0u, 0u, clo_before, 0u) : a.macc[b];
  acc.x += (uint32_t)nret;
  acc.y += (uint32_t)nst;
  unsigned long long* o = a.mout + (uint64_t)g * 4;
  const uint32_t lb = code & 0x7Fu;
  if (lb) atomicAdd(o + 3, 1ull << (lb - 1));
  if (r == I - 1 || a.step == nsteps - 1) {
    atomicAdd(o, (unsigned long long)(uint32_t)(clo_after - acc.z));
    if (acc.x) atomicAdd(o + 1, (unsigned long long)acc.x);
    if (acc.y) atomicAdd(o + 2, (unsigned long long)acc.y);
  } else {
    a.macc[b] = acc;
  }
}

// Warp-cooperative update of sub-trace b at lockstep step a.step (caller has
// checked the sub-trace is active).  y: the CNN's raw outputs (nullptr when
// teacher-forced without prediction).  Returns the new context count (all lanes).
// Lane l owns entries l, l+32, l+64, l+96 in registers; stable compaction by
// ballot + popc keeps fetch order.
__device__ __forceinline__ int update_subtrace(const UpdateArgs& a, uint64_t b, int64_t ws, int64_t s_b,
                                               int64_t nsteps, bool has_y, float y0, float y1, float y2,
                                               int lane) {
  const unsigned lt_mask = (1u << lane) - 1u;
  const int64_t i = ws + a.step;
  int f, c, s;                    // latencies that drive the update
  int pf = 0, pc = 0, ps = 0;     // the CNN's rounded prediction (recorded)
  if (has_y) { pf = lat_round(y0); pc = lat_round(y1); ps = lat_round(y2); }
  if (a.forced) {
    const uint16_t* p = a.forced + (i - a.row_lo) * 3;
    f = p[0]; c = p[1]; s = p[2];
    if (!has_y) { pf = f; pc = c; ps = s; }
  } else {
    f = pf; c = pc; s = ps;
  }
  int64_t clock = a.st.clock[b];
  const int k = a.st.count[b];
  const uint64_t qn = a.st.qn ? a.st.qn : a.st.n;        // entry stride (entry-major layout)
  uint4* qb = a.st.q + b;
  const uint32_t code = a.mrow ? a.mrow[i - a.row_lo] : 0u;   // metrics tag of row i (R20)
  const uint32_t clo_before = (uint32_t)clock;

  clock += f;
  const uint32_t clo_push = (uint32_t)clock;
  uint32_t eseq[4], efet[4], ecs[4], ew[4] = {0u, 0u, 0u, 0u};
  bool valid[4];
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const int ent = lane + 32 * m;
    valid[m] = ent < k;
    if (valid[m]) { const uint4 v = qb[ent * qn]; eseq[m] = v.x; efet[m] = v.y; ecs[m] = v.z; ew[m] = v.w; }
    if (ent == k) {                                      // push the predicted instruction (R4)
      valid[m] = true;
      eseq[m] = (uint32_t)i; efet[m] = clo_push; ecs[m] = (uint32_t)c | ((uint32_t)s << 16); ew[m] = code >> 7;
    }
  }
  __syncwarp();
  // retire: keep iff retire > Clock  <=>  c + s - age > 0
  auto live = [&](int m, uint32_t clo) -> bool {
    if (!valid[m]) return false;
    const int cs_sum = (int)(ecs[m] & 0xFFFF) + (int)(ecs[m] >> 16);
    return cs_sum - (int)(clo - efet[m]) > 0;
  };
  bool keep[4];
  int kept = 0;
  uint32_t clo = (uint32_t)clock;
#pragma unroll
  for (int m = 0; m < 4; ++m) { keep[m] = live(m, clo); kept += __popc(__ballot_sync(0xffffffffu, keep[m])); }
  if (kept > a.cap) {                                    // ROB-full stall: Clock = min retire (R5)
    int dmin = 0x7fffffff;
#pragma unroll
    for (int m = 0; m < 4; ++m)
      if (keep[m]) dmin = min(dmin, (int)(ecs[m] & 0xFFFF) + (int)(ecs[m] >> 16) - (int)(clo - efet[m]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) dmin = min(dmin, __shfl_xor_sync(0xffffffffu, dmin, o));
    clock += dmin;
    clo = (uint32_t)clock;
    kept = 0;
#pragma unroll
    for (int m = 0; m < 4; ++m) { keep[m] = live(m, clo); kept += __popc(__ballot_sync(0xffffffffu, keep[m])); }
    if (lane == 0) atomicAdd(a.st.stalls, 1ull);
  }
  int base = 0, nst = 0;
#pragma unroll
  for (int m = 0; m < 4; ++m) {
    const unsigned bal = __ballot_sync(0xffffffffu, keep[m]);
    if (keep[m]) {
      const uint64_t pos = (uint64_t)(base + __popc(bal & lt_mask)) * qn;
      qb[pos] = make_uint4(eseq[m], efet[m], ecs[m], ew[m]);
    }
    base += __popc(bal);
    if (a.macc) nst += __popc(__ballot_sync(0xffffffffu, valid[m] && !keep[m] && (ew[m] & 1u)));
  }
  if (lane == 0) {
    a.st.count[b] = base;
    a.st.clock[b] = clock;
    int64_t bnd = a.st.bnd[b];
    if (i == s_b - 1) { bnd = clock; a.st.bnd[b] = bnd; }   // end of warm-up
    if (a.step == nsteps - 1) a.st.cycles[b] = clock - bnd;
    pec_record_or_stop(a, b, i, s_b, nsteps, k, base, clock, bnd);
    metrics_row(a, b, i, s_b, nsteps, clo_before, (uint32_t)clock, k + 1 - base, nst, code);
    atomicAdd(a.st.k_hist + k, 1ull);
    if (i >= s_b) {
      const int64_t r = i - a.row_lo;
      if (a.rec_lat) { a.rec_lat[3 * r] = (uint16_t)pf; a.rec_lat[3 * r + 1] = (uint16_t)pc; a.rec_lat[3 * r + 2] = (uint16_t)ps; }
      if (a.rec_k) a.rec_k[r] = k;
      if (a.rec_clock) a.rec_clock[r] = clock;
      if (a.rec_y) { a.rec_y[3 * r] = y0; a.rec_y[3 * r + 1] = y1; a.rec_y[3 * r + 2] = y2; }
    }
  }
  return base;
}

}  // namespace psim

namespace psim {

// Thread-per-sub-trace variant of the same update (used by the fused
// fc1/head/update kernel, where one epilogue thread owns one sub-trace row of
// the tile).  Streams the fetch-ordered entries with 16-byte loads and
// compacts in place (write index <= read index); the rare ROB-full stall
// (R5) re-filters the compacted entries once.  Returns the new count.
// hist: per-CTA shared histogram of k (flushed by the caller).
struct QBatch { uint32_t s[8], f[8], c[8], w[8]; };

// 16-byte global store executed only if `pred` (a predicated instruction, no branch)
__device__ __forceinline__ void st_v4_if(uint4* p, uint4 v, bool pred) {
  asm volatile(
      "{\n"
      ".reg .pred q;\n"
      "setp.ne.u32 q, %5, 0;\n"
      "@q st.global.v4.u32 [%0], {%1, %2, %3, %4};\n"
      "}\n" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"((uint32_t)pred)
      : "memory");
}

// first 8 entries of sub-trace b (entry-major layout), to be prefetched early
__device__ __forceinline__ void load_qbatch(const SimState& st, uint64_t b, int k, QBatch& q) {
  const uint64_t qn = st.qn ? st.qn : st.n;
#pragma unroll
  for (int t = 0; t < 8; ++t)
    if (t < k) { const uint4 v = st.q[t * qn + b]; q.s[t] = v.x; q.f[t] = v.y; q.c[t] = v.z; q.w[t] = v.w; }
}

__device__ __forceinline__ int update_subtrace_thread(const UpdateArgs& a, uint64_t b, int64_t ws, int64_t s_b,
                                                      int64_t nsteps, int k, int64_t& clock, uint32_t rmin,
                                                      const QBatch& first, bool has_y, float y0, float y1, float y2,
                                                      unsigned int* hist, bool* stopped = nullptr,
                                                      long long* ts = nullptr) {   // timing builds: clock64 stamps
  if (ts) ts[0] = clock64();
  const int64_t i = ws + a.step;
  int f, c, s;
  int pf = 0, pc = 0, ps = 0;
  if (has_y) { pf = lat_round(y0); pc = lat_round(y1); ps = lat_round(y2); }
  if (a.forced) {
    const uint16_t* p = a.forced + (i - a.row_lo) * 3;
    f = p[0]; c = p[1]; s = p[2];
    if (!has_y) { pf = f; pc = c; ps = s; }
  } else {
    f = pf; c = pc; s = ps;
  }
  const uint64_t qn = a.st.qn ? a.st.qn : a.st.n;          // entry-major: entry e at [e * qn + b]
  uint4* qb = a.st.q + b;
  const uint32_t code = a.mrow ? a.mrow[i - a.row_lo] : 0u;   // metrics tag of row i (R20)
  const uint32_t clo_before = (uint32_t)clock;
  clock += f;
  uint32_t clo = (uint32_t)clock;
  // push the predicted instruction (R4) as entry k, then retire.
  // Entries are streamed in batches of 8 with all loads of a batch in flight;
  // consecutive threads (sub-traces) access consecutive words (coalesced).
  const uint32_t push_s = (uint32_t)i, push_f = clo, push_c = (uint32_t)c | ((uint32_t)s << 16),
                 push_w = code >> 7;
  const int n_in = k + 1;
  int w = 0, nst = 0;
  int dmin = 0x7fffffff;   // min (retire - Clock) over kept entries
  uint4* wp = qb;          // write position of the scan: entry w
  const bool new_live = (c + s) > 0;                       // retire = Clock + c + s > Clock
  // Fast path: if the smallest retire Clock of the old entries is still ahead of the new
  // Clock, none of them retires; only the pushed entry is appended (or retires at once).
  // The result is the same set removal as the scan below.
  if (k == 0 || (int)(rmin - clo) > 0) {
    if (k + (new_live ? 1 : 0) <= a.cap) {
      if (new_live) qb[(uint64_t)k * qn] = make_uint4(push_s, push_f, push_c, push_w);
      w = k + (new_live ? 1 : 0);
      nst = new_live ? 0 : (int)(push_w & 1u);
      const uint32_t rnew = clo + (uint32_t)(c + s);
      rmin = (k == 0 || (int)(rnew - rmin) < 0) ? rnew : rmin;
      goto done;
    }
  }
  if (ts) ts[1] = clock64();
  for (int e0 = 0; e0 < n_in; e0 += 8) {
    if (ts && e0 <= 32) ts[2 + e0 / 4] = clock64();
    uint32_t vs[8], vf[8], vc[8], vw[8];
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      const int e = e0 + t;
      if (e < k) {
        if (e0 == 0) { vs[t] = first.s[t]; vf[t] = first.f[t]; vc[t] = first.c[t]; vw[t] = first.w[t]; }   // prefetched
        else { const uint4 v = qb[e * qn]; vs[t] = v.x; vf[t] = v.y; vc[t] = v.z; vw[t] = v.w; }
      } else { vs[t] = push_s; vf[t] = push_f; vc[t] = push_c; vw[t] = push_w; }   // e == k: the pushed entry
    }
    // Branch-free: the retire tests of the 8 entries are independent; the only serial chain
    // is the write pointer (one predicated 16-B store and one conditional add per entry).
    // A branch per entry cost ~140 cycles per entry (divergence + reconvergence + the
    // rematerialised w * qn address; PSIM_TIMING stamps: a batch of 8 prefetched entries
    // 1.14k -> 0.71k cycles).  Skipping the stores of entries that do not move: no gain.
#pragma unroll
    for (int t = 0; t < 8; ++t) {
      const bool val = e0 + t < n_in;
      const int rem = (int)(vc[t] & 0xFFFF) + (int)(vc[t] >> 16) - (int)(clo - vf[t]);   // retire - Clock
      const bool kp = val && rem > 0;
      st_v4_if(wp, make_uint4(vs[t], vf[t], vc[t], vw[t]), kp);
      wp += kp ? qn : 0;
      w += kp ? 1 : 0;
      dmin = kp ? min(dmin, rem) : dmin;
      nst += (val && !kp) ? (int)(vw[t] & 1u) : 0;
    }
    if (ts && e0 <= 32) ts[3 + e0 / 4] = clock64();
  }
  if (w > a.cap) {                                         // ROB-full stall: Clock = min retire (R5)
    clock += dmin;
    clo = (uint32_t)clock;
    const int n2 = w;
    w = 0;
    dmin = 0x7fffffff;
    for (int e = 0; e < n2; ++e) {
      const uint4 v = qb[e * qn];
      const int rem = (int)(v.z & 0xFFFF) + (int)(v.z >> 16) - (int)(clo - v.y);
      if (rem > 0) {
        qb[w * qn] = v; ++w;
        dmin = min(dmin, rem);
      } else {
        nst += (int)(v.w & 1u);
      }
    }
    atomicAdd(a.st.stalls, 1ull);
  }
  rmin = clo + (uint32_t)dmin;                             // (unused when w == 0)
done:
  if (ts) ts[12] = clock64();
  a.st.count[b] = w;
  a.st.clock[b] = clock;
  a.st.rmin[b] = rmin;
  int64_t bnd = a.st.bnd[b];
  if (i == s_b - 1) { bnd = clock; a.st.bnd[b] = bnd; }   // end of warm-up
  if (a.step == nsteps - 1) a.st.cycles[b] = clock - bnd;
  const bool stop = pec_record_or_stop(a, b, i, s_b, nsteps, k, w, clock, bnd);
  if (stopped) *stopped = stop;
  metrics_row(a, b, i, s_b, nsteps, clo_before, (uint32_t)clock, k + 1 - w, nst, code);
  atomicAdd(hist + k, 1u);
  if (i >= s_b) {
    const int64_t r = i - a.row_lo;
    if (a.rec_lat) { a.rec_lat[3 * r] = (uint16_t)pf; a.rec_lat[3 * r + 1] = (uint16_t)pc; a.rec_lat[3 * r + 2] = (uint16_t)ps; }
    if (a.rec_k) a.rec_k[r] = k;
    if (a.rec_clock) a.rec_clock[r] = clock;
    if (a.rec_y) { a.rec_y[3 * r] = y0; a.rec_y[3 * r + 1] = y1; a.rec_y[3 * r + 2] = y2; }
  }
  return w;
}

}  // namespace psim
