// Microbenchmark: H2D of one streaming chunk (65536 sub-traces x 64 rows x 48 B, one 3 KB
// piece per sub-trace at a ~73 KB stride in a pinned host trace) by
//   (a) cudaMemcpyBatchAsync (copy engines, one descriptor per piece),
//   (b) a zero-copy kernel (16-B loads of the pinned host memory, 256 CTAs x 128 threads),
//   (c) one contiguous cudaMemcpyAsync of the same byte count (the PCIe ceiling).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
__global__ void zc(const uint4* __restrict__ host, uint4* __restrict__ dev, int n, int64_t pitch16, int per16) {
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x, nt = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = tid; i < (int64_t)n * per16; i += nt) {
    const int64_t b = i / per16, o = i - b * per16;
    dev[i] = host[b * pitch16 + o];
  }
}
int main() {
  const int n = 65536, rows = 64, rb = 48;
  const int64_t len = 1526, piece = (int64_t)rows * rb, pitch = len * rb;
  const size_t host_bytes = (size_t)n * pitch;
  uint8_t* host; cudaMallocHost(&host, host_bytes);
  for (size_t i = 0; i < host_bytes; i += 4096) host[i] = (uint8_t)i;
  uint8_t* dev; cudaMalloc(&dev, (size_t)n * piece);
  cudaStream_t st; cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  std::vector<void*> dsts(n), srcs(n); std::vector<size_t> sizes(n, piece);
  for (int b = 0; b < n; ++b) { dsts[b] = dev + (size_t)b * piece; srcs[b] = host + (size_t)b * pitch + 100 * rb; }
  cudaMemcpyAttributes attr = {};
  attr.srcAccessOrder = cudaMemcpySrcAccessOrderStream;
  attr.flags = cudaMemcpyFlagPreferOverlapWithCompute;
  size_t attrIdx = 0, fail = 0;
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(e0, st);
    cudaError_t r = cudaMemcpyBatchAsync(dsts.data(), srcs.data(), sizes.data(), n, &attr, &attrIdx, 1, &fail, st);
    cudaEventRecord(e1, st); cudaStreamSynchronize(st); cudaEventElapsedTime(&ms, e0, e1);
    printf("batch copy:   %s  %.3f ms  %.1f GB/s\n", cudaGetErrorString(r), ms, n * piece / ms / 1e6);
  }
  const uint4* hdev = nullptr; cudaHostGetDevicePointer((void**)&hdev, host, 0);
  for (int grid : {148, 296, 1184}) {
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(e0, st);
      zc<<<grid, 128, 0, st>>>(hdev, (uint4*)dev, n, pitch / 16, piece / 16);
      cudaEventRecord(e1, st); cudaStreamSynchronize(st); cudaEventElapsedTime(&ms, e0, e1);
    }
    printf("zero-copy %4d CTAs: %.3f ms  %.1f GB/s  %s\n", grid, ms, n * piece / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
  }
  for (int rep = 0; rep < 2; ++rep) {
    cudaEventRecord(e0, st);
    cudaMemcpyAsync(dev, host, (size_t)n * piece, cudaMemcpyHostToDevice, st);
    cudaEventRecord(e1, st); cudaStreamSynchronize(st); cudaEventElapsedTime(&ms, e0, e1);
  }
  printf("contiguous memcpy: %.3f ms  %.1f GB/s\n", ms, n * piece / ms / 1e6);
  return 0;
}
