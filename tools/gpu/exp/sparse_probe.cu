// Experiment: tcgen05.mma.sp (2:4 structured sparse A) kind::f16, M = 128, N = 64,
// K = 32 logical per instruction.  Establishes, by probing, how the compressed A operand
// (16 stored bf16 per row per instruction, SW128 K-major smem) and the metadata (TMEM)
// map to logical K positions: with B = identity (B[n][k] = (n == k)) the accumulator row
// m is the decompressed A row m itself.
//
// Per run (host argv): meta word pattern per lane quarter, sparse_id2, number of K steps,
// TMEM metadata column step between K steps.  Prints D rows 0, 1, 33, 64, 127 and a
// consistency summary.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../../../paper_conf_sc_pandeylfhl22_b200/csrc/tc_common.cuh"
using namespace psim::tc;

__device__ __forceinline__ void tmem_st1(uint32_t taddr, uint32_t v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(v) : "memory");
}
__device__ __forceinline__ void mma_sp(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t tmem_e,
                                       uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.sp.cta_group::1.kind::f16 [%0], %1, %2, [%5], %3, p;\n}\n" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(acc), "r"(tmem_e));
}

// A: compressed [128 rows][64 stored] bf16 (4 K steps x 16), B: [64 N][128 K logical]
// meta: [ksteps][128 lanes] u32
__global__ void k(const __nv_bfloat16* A, const __nv_bfloat16* B, const uint32_t* meta, int ksteps, int id2,
                  int col_step, float* D) {
  __shared__ __align__(1024) uint8_t sA[128 * 128];
  __shared__ __align__(1024) uint8_t sB[2 * 64 * 128];   // 2 atoms: K 0..63, 64..127
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  for (int idx = tid; idx < 128 * 8; idx += blockDim.x) {
    const int r = idx / 8, c = idx % 8;
    st_sw128(sA, r, c, reinterpret_cast<const uint4*>(A)[idx]);
  }
  for (int idx = tid; idx < 64 * 16; idx += blockDim.x) {
    const int r = idx / 16, c = idx % 16;
    st_sw128(sB + (c >> 3) * 64 * 128, r, c & 7, reinterpret_cast<const uint4*>(B)[idx]);
  }
  if (tid == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  if (warp == 0) tmem_alloc(&slot, 256);
  fence_async_smem();
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = slot;
  const uint32_t ecol = 128;
  // col_step < 0: step s's metadata in column ecol + s, addressed as column ecol + (s & ~1)
  // with sparse_id2 = s & 1 (the id2-selects-the-odd-column hypothesis)
  for (int s = 0; s < ksteps; ++s)
    tmem_st1(tmem + ((uint32_t)(warp * 32) << 16) + ecol + (col_step < 0 ? s : s * col_step),
             meta[s * 128 + warp * 32 + lane]);
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  fence_before();
  __syncthreads();
  fence_after();
  if (tid == 0) {
    for (int s = 0; s < ksteps; ++s) {
      const uint32_t idesc = idesc_bf16(128, 64) | (1u << 2) | (uint32_t)((col_step < 0 ? (s & 1) : id2) & 3);
      const uint32_t ecs = col_step < 0 ? (uint32_t)(s & ~1) : (uint32_t)(s * col_step);
      // A: 16 stored elements (32 B) per step; B: 32 logical K (64 B) per step
      const uint64_t da = sw128_desc(smem_u32(sA) + s * 32);
      const int kb = s * 32;
      const uint64_t db = sw128_desc(smem_u32(sB) + (kb >> 6) * 64 * 128 + (kb & 63) * 2);
      mma_sp(tmem, da, db, idesc, tmem + ecol + ecs, s > 0);
    }
    mma_commit(&bar);
  }
  __syncwarp();
  mbar_wait(&bar, 0);
  fence_after();
  uint32_t r[32];
  tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16), r);
  tmem_wait_ld();
  for (int i = 0; i < 32; ++i) D[(warp * 32 + lane) * 64 + i] = __uint_as_float(r[i]);
  tmem_ld32_nowait(tmem + ((uint32_t)(warp * 32) << 16) + 32, r);
  tmem_wait_ld();
  for (int i = 0; i < 32; ++i) D[(warp * 32 + lane) * 64 + 32 + i] = __uint_as_float(r[i]);
  fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 256);
}

// valid 2:4 nibbles (idx0 < idx1, idx0 in bits 0-1, idx1 in bits 2-3)
static const uint32_t kPat[6] = {0x4, 0x8, 0xC, 0x9, 0xD, 0xE};
static int pat_of(const float* g4) {   // positions of the two nonzeros in a group of 4 -> pattern index
  int i0 = -1, i1 = -1;
  for (int i = 0; i < 4; ++i)
    if (g4[i] != 0.f) { if (i0 < 0) i0 = i; else i1 = i; }
  if (i0 < 0 || i1 < 0) return -1;
  const uint32_t nib = (uint32_t)i0 | ((uint32_t)i1 << 2);
  for (int p = 0; p < 6; ++p) if (kPat[p] == nib) return p;
  return -2;
}

int main(int argc, char** argv) {
  // decode mode: metadata set by formula, five runs decode (lane, nibble) of every (row, group)
  const int ksteps = argc > 1 ? atoi(argv[1]) : 1;
  const int col_step = argc > 2 ? atoi(argv[2]) : 2;
  const int id2 = argc > 3 ? atoi(argv[3]) : 0;
  std::vector<__nv_bfloat16> A(128 * 64), B(64 * 128);
  for (int m = 0; m < 128; ++m)
    for (int j = 0; j < 64; ++j) A[m * 64 + j] = __float2bfloat16((float)(j + 1));
  for (int n = 0; n < 64; ++n)
    for (int kk = 0; kk < 128; ++kk) B[n * 128 + kk] = __float2bfloat16(n == kk ? 1.f : 0.f);
  __nv_bfloat16 *dA, *dB;
  uint32_t* dM;
  float* dD;
  cudaMalloc(&dA, A.size() * 2); cudaMalloc(&dB, B.size() * 2); cudaMalloc(&dM, 4 * 128 * 4);
  cudaMalloc(&dD, 128 * 64 * 4);
  cudaMemcpy(dA, A.data(), A.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 2, cudaMemcpyHostToDevice);
  const int G = 8 * ksteps;   // groups per row
  std::vector<int> dig[5];
  for (int mode = 0; mode < 5; ++mode) {
    std::vector<uint32_t> meta(4 * 128);
    for (int s = 0; s < 4; ++s)
      for (int l = 0; l < 128; ++l) {
        uint32_t w = 0;
        for (int j = 0; j < 8; ++j) {
          int v = 0;
          switch (mode) {
            case 0: v = l % 6; break;
            case 1: v = (l / 6) % 6; break;
            case 2: v = (l / 36) % 6; break;
            case 3: v = (j + 8 * s) % 6; break;
            case 4: v = ((j + 8 * s) / 6) % 6; break;
          }
          w |= kPat[v] << (4 * j);
        }
        meta[s * 128 + l] = w;
      }
    cudaMemcpy(dM, meta.data(), meta.size() * 4, cudaMemcpyHostToDevice);
    cudaMemset(dD, 0, 128 * 64 * 4);
    k<<<1, 128>>>(dA, dB, dM, ksteps, id2, col_step, dD);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("mode %d: %s\n", mode, cudaGetErrorString(e)); return 1; }
    std::vector<float> D(128 * 64);
    cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost);
    dig[mode].resize(128 * G);
    for (int m = 0; m < 128; ++m)
      for (int g = 0; g < G; ++g) dig[mode][m * G + g] = pat_of(&D[m * 64 + 4 * g]);
  }
  printf("ksteps %d col_step %d id2 %d: (row, group) -> (lane, step*8+nibble)\n", ksteps, col_step, id2);
  for (int m = 0; m < 128; ++m) {
    printf("row %3d:", m);
    for (int g = 0; g < G; ++g) {
      const int a0 = dig[0][m * G + g], a1 = dig[1][m * G + g], a2 = dig[2][m * G + g];
      const int b0 = dig[3][m * G + g], b1 = dig[4][m * G + g];
      if (a0 < 0 || a1 < 0 || a2 < 0 || b0 < 0 || b1 < 0) { printf(" ?"); continue; }
      int lane = -1;
      for (int l = 0; l < 128; ++l) if (l % 6 == a0 && (l / 6) % 6 == a1 && (l / 36) % 6 == a2) lane = l;
      int nib = -1;
      for (int j = 0; j < 32; ++j) if (j % 6 == b0 && (j / 6) % 6 == b1) nib = j;
      printf(" %d:%d", lane, nib);
    }
    printf("\n");
  }
  return 0;
}
