// Experiment: TMA tile::gather4 into a SWIZZLE_128B tile at 512-B offsets (sm_100a).
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void k(const __grid_constant__ CUtensorMap tm, const int* rows, uint16_t* out, int off_rows) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su(&bar)), "r"(1));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (int i = threadIdx.x; i < 16384 / 4; i += blockDim.x) ((uint32_t*)sm)[i] = 0xFFFFFFFFu;
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar)), "r"(128 * 96) : "memory");
    for (int g = 0; g < 32; ++g) {
      const int m = g * 4;
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
          ::"r"(su(sm + (m + off_rows) % 128 * 128)), "l"((uint64_t)&tm), "r"(0), "r"(rows[m]), "r"(rows[m + 1]), "r"(rows[m + 2]),
            "r"(rows[m + 3]), "r"(su(&bar)) : "memory");
    }
  }
  asm volatile("{\n.reg .pred P1;\nW: mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n@!P1 bra W;\n}\n" ::"r"(su(&bar)), "r"(0) : "memory");
  for (int i = threadIdx.x; i < 16384 / 2; i += blockDim.x) out[i] = ((uint16_t*)sm)[i];
}
int main(int argc, char** argv) {
  const int R = 1000, C = 48;
  std::vector<uint16_t> h(R * C);
  for (int r = 0; r < R; ++r) for (int c = 0; c < C; ++c) h[r * C + c] = (uint16_t)(r * 64 + c);
  uint16_t* d; cudaMalloc(&d, h.size() * 2); cudaMemcpy(d, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
  std::vector<int> rows(128); for (int i = 0; i < 128; ++i) rows[i] = (i * 37 + 11) % R;
  int* drows; cudaMalloc(&drows, 512); cudaMemcpy(drows, rows.data(), 512, cudaMemcpyHostToDevice);
  uint16_t* dout; cudaMalloc(&dout, 16384);
  void* p = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  EncodeTiledFn fn = (EncodeTiledFn)p;
  for (int boxr : {1}) {
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)C, (cuuint64_t)R}; cuuint64_t str[1] = {C * 2};
    cuuint32_t box[2] = {48, (cuuint32_t)boxr}; cuuint32_t es[2] = {1, 1};
    CUresult cr = fn(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("box rows %d encode %d\n", boxr, (int)cr);
    if (cr) continue;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 20000);
    for (int off : {0, 4}) {
      cudaMemset(dout, 0, 16384);
      k<<<1, 128, 20000>>>(tm, drows, dout, off);
      cudaError_t e = cudaDeviceSynchronize();
      if (e) { printf("  off %d: kernel error %s\n", off, cudaGetErrorString(e)); return 1; }
      std::vector<uint16_t> o(8192); cudaMemcpy(o.data(), dout, 16384, cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int m = 0; m < 128; ++m) {
        const int srow = rows[((m - off) % 128 + 128) % 128];
        for (int c = 0; c < 64; ++c) {
          const int chunk = c / 8, e8 = c % 8;
          const int pos = m * 64 + ((chunk ^ (m & 7)) * 8) + e8;   // SW128 K-major layout, 128-B row pitch
          const uint16_t want = c < 48 ? (uint16_t)(srow * 64 + c) : (uint16_t)0xFFFF;   // chunks 6,7 untouched
          if (o[pos] != want) { if (bad < 4) printf("    m %d c %d got %d want %d\n", m, c, o[pos], want); ++bad; }
        }
      }
      printf("  off %d: mismatches vs SW128 layout: %d\n", off, bad);
    }
  }
  return 0;
}
