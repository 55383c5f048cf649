// sim_kernels.cu -- the integer side of the lockstep step (sm_100a):
//   gather   (context construction, PAPER.md:93 steps 2.1-2.3, :123-127)
//   update   (rounding + Clock advance + retire/compact/push, :99, :105-107)
//   reduce   (per-sub-trace cycles -> local total, :107, :181)
// One warp per sub-trace; state is structure-of-arrays in HBM (internal.h).
//
// Time features: every live entry satisfies retire > Clock (R4), and
// retire - fetch = c + s <= 8190, so age = Clock - fetch < 8191 is computed
// exactly from the low 32 bits of the clocks (q_fetch) whatever the absolute
// Clock; the 65535 clamp of R7 is kept for completeness.
#include "internal.h"
#include "sim_common.cuh"

namespace psim {

template <typename T>
__device__ __forceinline__ void store2(T* p, float a, float b);
template <>
__device__ __forceinline__ void store2<float>(float* p, float a, float b) {
  *reinterpret_cast<float2*>(p) = make_float2(a, b);
}
template <>
__device__ __forceinline__ void store2<__nv_bfloat16>(__nv_bfloat16* p, float a, float b) {
  *reinterpret_cast<__nv_bfloat162*>(p) = __floats2bfloat162_rn(a, b);  // RNE, as the oracle's bf16 mode
}

// X[b][r][c]: row 0 = current instruction (time columns 0), rows 1..k = live
// entries newest first (R6), rows > k zero (PAPER.md:93 zero padding); the item's
// extra pad rows (RB7 layout: item_rows = 116, row_off = 2) are zero.
// Eight threads per (sub-trace, item row), thread c of a row building features 8c .. 8c + 7:
// the whole input of a sub-trace is built in parallel (independent loads of the queue entry
// and of two aligned 8-byte words of the trace row), and a warp stores four consecutive
// rows as one contiguous 512-byte (bf16) / 1 KB (fp32) span.
template <typename T>
__global__ void __launch_bounds__(256) gather_kernel(GatherArgs a, T* __restrict__ x) {
  const uint64_t total = a.n * (uint64_t)a.item_rows * 8;
  const bool aligned8 = ((a.stride | reinterpret_cast<uintptr_t>(a.trace)) & 7) == 0;
  for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < total; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t rr = t >> 3;                                        // global item row
    const int ch = (int)(t & 7);                                       // 8-feature chunk of the row
    const uint64_t b = rr / (uint64_t)a.item_rows;
    const int r = (int)(rr - b * (uint64_t)a.item_rows) - a.row_off;  // input row (PAPER.md:93 order)
    const int64_t ws = a.ws[b];
    if (a.step >= a.e[b] - ws) continue;                               // sub-trace finished
    const int k = a.count[b];
    float v[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) v[c] = 0.f;
    if (r >= 0 && r <= k && r < kRows && ch < 7) {                    // features 56..63 are zero
      int64_t row;
      if (r == 0) {
        row = ws + a.step;                                             // current instruction first
      } else {
        const uint4 en = a.q[(uint64_t)(k - r) * (a.qn ? a.qn : a.n) + b];   // newest first (R6)
        row = en.x;
        if (ch == 0) {                                                 // R2 time features, clamped (R7)
          const uint32_t clo = (uint32_t)a.clock[b];
          const int c = en.z & 0xFFFF, s = en.z >> 16;
          const int age = (int)(clo - en.y);
          v[0] = (float)min(age, kTimeMax);
          v[1] = (float)min(max(0, c - age), kTimeMax);
          v[2] = (float)min(c + s - age, kTimeMax);
        }
      }
      // feature f = 8 ch + i (i < 8) is attribute f - 3 for 3 <= f < 50: trace bytes 8 ch - 3 .. 8 ch + 4
      const uint8_t* ar = a.trace + (row - a.row_lo) * a.stride;
      if (aligned8) {
        const uint2 lo = ch > 0 ? __ldg(reinterpret_cast<const uint2*>(ar) + ch - 1) : make_uint2(0u, 0u);
        // bytes 8 ch .. 8 ch + 7 (chunk 6 needs only bytes 45, 46 of lo: its hi word would lie
        // past the 47 attributes, past the buffer for the last row)
        const uint2 hi = ch < 6 ? __ldg(reinterpret_cast<const uint2*>(ar) + ch) : make_uint2(0u, 0u);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int f = 8 * ch + i;
          if (f < 3 || f >= kFeat) continue;
          const int byte = f - 3 - 8 * (ch - 1);                       // offset within [lo | hi]
          const uint32_t w = byte < 4 ? lo.x : byte < 8 ? lo.y : byte < 12 ? hi.x : hi.y;
          v[i] = (float)((w >> ((byte & 3) * 8)) & 0xFFu);
        }
      } else {
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const int f = 8 * ch + i;
          if (f >= 3 && f < kFeat) v[i] = (float)__ldg(ar + (f - 3));
        }
      }
    }
    T* xr = x + rr * kFeatPad + 8 * ch;
    if constexpr (sizeof(T) == 2) {
      uint32_t p[4];
#pragma unroll
      for (int h = 0; h < 4; ++h) {
        __nv_bfloat162 h2 = __floats2bfloat162_rn(v[2 * h], v[2 * h + 1]);   // RNE (oracle bf16 mode)
        p[h] = *reinterpret_cast<uint32_t*>(&h2);
      }
      *reinterpret_cast<uint4*>(xr) = make_uint4(p[0], p[1], p[2], p[3]);
    } else {
      reinterpret_cast<float4*>(xr)[0] = make_float4(v[0], v[1], v[2], v[3]);
      reinterpret_cast<float4*>(xr)[1] = make_float4(v[4], v[5], v[6], v[7]);
    }
  }
}

static int grid_for(uint64_t warps, int block = 256) {
  uint64_t blocks = (warps * 32 + block - 1) / block;
  if (blocks > 148ull * 64) blocks = 148ull * 64;
  if (blocks < 1) blocks = 1;
  return (int)blocks;
}

static int grid_rows(uint64_t rows) {   // threads -> CTAs of 256, at most 148 x 16
  uint64_t blocks = (rows + 255) / 256;
  if (blocks > 148ull * 16) blocks = 148ull * 16;
  return (int)std::max<uint64_t>(blocks, 1);
}
void launch_gather_f32(const GatherArgs& a, float* x, cudaStream_t st) {
  gather_kernel<float><<<grid_rows(a.n * (uint64_t)a.item_rows * 8), 256, 0, st>>>(a, x);
}
void launch_gather_bf16(const GatherArgs& a, __nv_bfloat16* x, cudaStream_t st) {
  gather_kernel<__nv_bfloat16><<<grid_rows(a.n * (uint64_t)a.item_rows * 8), 256, 0, st>>>(a, x);
}

// ---------------------------------------------------------------------------
// update: round (R7), Clock += f, push, retire every entry with retire <= Clock
// (PAPER.md:107), ROB-full stall if more than cap entries remain (R5),
// boundary / cycles bookkeeping, per-row records (parity).
// Lane l owns entries l, l+32, l+64, l+96 in registers; stable compaction by
// ballot + popc keeps fetch order.
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(256) update_kernel(UpdateArgs a) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (gridDim.x * (uint64_t)blockDim.x) >> 5;
  for (uint64_t b = warp; b < a.st.n; b += nwarps) {
    const int64_t ws = a.st.ws[b], s_b = a.st.s[b], e_b = a.st.e[b];
    const int64_t nsteps = e_b - ws;
    if (a.step >= nsteps) continue;
    const bool has_y = a.y != nullptr;
    update_subtrace(a, b, ws, s_b, nsteps, has_y, has_y ? a.y[b * 3] : 0.f, has_y ? a.y[b * 3 + 1] : 0.f,
                    has_y ? a.y[b * 3 + 2] : 0.f, lane);
  }
}

void launch_update(const UpdateArgs& a, cudaStream_t st) {
  update_kernel<<<grid_for(a.st.n), 256, 0, st>>>(a);
}

// per-row metric code (R20; trace attribute layout of SURVEY.md Appendix C):
// bit 7 = store (attr 8); bits 0..6 = 1 + log2 access size (attr 34) if the row is a
// load or store (attrs 7, 8) whose data came from memory (attr 14 == 2)
__device__ __forceinline__ uint8_t metric_code(uint32_t load, uint32_t store, uint32_t dlevel, uint32_t log2size) {
  const uint32_t mem = ((load | store) != 0u && dlevel == 2u) ? min(log2size, 62u) + 1u : 0u;
  return (uint8_t)((store ? 0x80u : 0u) | mem);
}
__global__ void mrow_kernel(const uint8_t* __restrict__ trace, int64_t stride, int64_t rows, uint8_t* __restrict__ out) {
  const int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (r >= rows) return;
  const uint8_t* a = trace + r * stride;
  out[r] = metric_code(a[7], a[8], a[14], a[34]);
}
void launch_mrow(const uint8_t* trace, int64_t stride, int64_t rows, uint8_t* out, cudaStream_t st) {
  if (rows > 0) mrow_kernel<<<(unsigned)((rows + 255) / 256), 256, 0, st>>>(trace, stride, rows, out);
}

__global__ void state_init_kernel(SimState s) {
  const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (t < s.n) {
    s.clock[t] = 0; s.bnd[t] = 0; s.cycles[t] = 0; s.count[t] = 0;
    if (s.rmin) s.rmin[t] = 0;   // meaningful only when count > 0; defined for the sanitizer (initcheck)
  }
  if (t < 112) s.k_hist[t] = 0;
  if (t == 0) { *s.stalls = 0; *s.total = 0; *s.ptile_sum = 0; }
}
void launch_state_init(const SimState& s, cudaStream_t st) {
  uint64_t n = s.n > 112 ? s.n : 112;
  state_init_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(s);
}

// ---- post-error correction (PAPER.md:203-219 [V-B]; R19) ----
// corrector b (every local sub-trace but the last) continues from its final
// state over rows [s_{b+1}, s_{b+1} + len) of sub-trace b+1; it does not start
// if its count already equals b+1's first-pass count at s_{b+1}.
__global__ void pec_init_kernel(SimState s, Pec p) {
  const uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (b >= s.n) return;
  p.cycles1[b] = s.cycles[b];
  p.len[b] = 0;
  int64_t r0 = 0, len = 0;
  if (b + 1 < s.n) {
    r0 = s.s[b + 1];
    len = min((int64_t)p.limit, s.e[b + 1] - r0);
    if (len > 0 && s.count[b] == (int)p.k1[b + 1]) len = 0;
  }
  p.ws[b] = r0; p.s[b] = r0; p.e[b] = r0 + len;
  p.bnd[b] = s.clock[b];
  p.cyc[b] = 0;
  if (b == 0) *p.corrected = 0;
}
void launch_pec_init(const SimState& s, const Pec& p, cudaStream_t st) {
  if (s.n) pec_init_kernel<<<(unsigned)((s.n + 255) / 256), 256, 0, st>>>(s, p);
}

// "The re-simulated cycles will replace the previously simulated ones"
__global__ void pec_apply_kernel(SimState s, Pec p) {
  const uint64_t b = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (b + 1 >= s.n) return;
  const int64_t len = p.e[b] - p.ws[b];
  if (len <= 0) return;
  s.cycles[b + 1] = p.cycles1[b + 1] - (int64_t)p.c1[(uint64_t)(len - 1) * s.n + b + 1] + p.cyc[b];
  p.len[b + 1] = (int32_t)len;
  atomicAdd(p.corrected, (unsigned long long)len);
}
void launch_pec_apply(const SimState& s, const Pec& p, cudaStream_t st) {
  if (s.n > 1) pec_apply_kernel<<<(unsigned)((s.n + 255) / 256), 256, 0, st>>>(s, p);
}

// total = sum_j cycles_j (int64, exact and order independent)
__global__ void __launch_bounds__(1024) reduce_kernel(SimState s) {
  long long acc = 0;
  for (uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; t < s.n; t += (uint64_t)gridDim.x * blockDim.x)
    acc += s.cycles[t];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  __shared__ long long part[32];
  if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x < 32) {
    acc = threadIdx.x < (blockDim.x >> 5) ? part[threadIdx.x] : 0;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (threadIdx.x == 0) atomicAdd((unsigned long long*)s.total, (unsigned long long)acc);
  }
}
void launch_reduce_cycles(const SimState& s, cudaStream_t st) {
  unsigned blocks = (unsigned)((s.n + 1023) / 1024);
  if (blocks > 148) blocks = 148;
  if (blocks < 1) blocks = 1;
  reduce_kernel<<<blocks, 1024, 0, st>>>(s);
}

// head (fc2, fp32 on CUDA cores): y[b][o] = b[o] + sum_i h[b][i] w[o][i]
__global__ void __launch_bounds__(256) head_kernel(const float* __restrict__ h, const float* __restrict__ w,
                                                   const float* __restrict__ bias, int in,
                                                   float* __restrict__ y, uint64_t n) {
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (gridDim.x * (uint64_t)blockDim.x) >> 5;
  for (uint64_t b = warp; b < n; b += nwarps) {
    float a0 = 0.f, a1 = 0.f, a2 = 0.f;
    for (int t = lane; t < in; t += 32) {
      const float v = h[b * in + t];
      a0 = fmaf(v, __ldg(w + t), a0);
      a1 = fmaf(v, __ldg(w + in + t), a1);
      a2 = fmaf(v, __ldg(w + 2 * in + t), a2);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      a0 += __shfl_xor_sync(0xffffffffu, a0, o);
      a1 += __shfl_xor_sync(0xffffffffu, a1, o);
      a2 += __shfl_xor_sync(0xffffffffu, a2, o);
    }
    if (lane == 0) {
      y[b * 3 + 0] = a0 + bias[0];
      y[b * 3 + 1] = a1 + bias[1];
      y[b * 3 + 2] = a2 + bias[2];
    }
  }
}
void launch_head(const float* h, const float* w, const float* b, int in, float* y, uint64_t n,
                 cudaStream_t st) {
  head_kernel<<<grid_for(n), 256, 0, st>>>(h, w, b, in, y, n);
}

__global__ void pad_inputs_kernel(const float* __restrict__ X, uint64_t B, void* x, bool bf16, int item_rows,
                                  int row_off) {
  const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const uint64_t total = B * item_rows * kFeatPad;
  if (t >= total) return;
  const int c = (int)(t % kFeatPad);
  const uint64_t br = t / kFeatPad;
  const uint64_t b = br / item_rows;
  const int r = (int)(br % item_rows) - row_off;   // pad rows outside [0, kRows) are zero
  const float v = (c < kFeat && r >= 0 && r < kRows) ? X[(b * kRows + r) * kFeat + c] : 0.f;
  if (bf16) reinterpret_cast<__nv_bfloat16*>(x)[t] = __float2bfloat16_rn(v);
  else reinterpret_cast<float*>(x)[t] = v;
}
void launch_pad_inputs(const float* X, uint64_t B, void* x, bool bf16, cudaStream_t st, int item_rows, int row_off) {
  const uint64_t total = B * item_rows * kFeatPad;
  pad_inputs_kernel<<<(unsigned)((total + 255) / 256), 256, 0, st>>>(X, B, x, bf16, item_rows, row_off);
}

}  // namespace psim
