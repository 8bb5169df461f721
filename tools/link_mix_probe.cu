// Host-link probe (round 2): can SM loads/stores of mapped pinned host memory
// add bandwidth on top of a copy-engine transfer in the same direction?
//
// For each direction, over G GiB of pinned host memory (cudaHostAlloc,
// mapped) and a device buffer:
//   ce   : cudaMemcpyAsync in 64 MiB pieces on one stream (the library's path)
//   sm   : a grid-stride kernel that moves the bytes with 16-B loads/stores
//          through the host mapping (zero-copy)
//   mix f: the first (1-f) of the bytes by the copy engine and the rest by the
//          kernel, concurrently on two streams
// Reports GB/s of bytes moved per wall time between events bracketing both.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/link_mix_probe tools/link_mix_probe.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <vector>

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e = (x);                                                       \
    if (e != cudaSuccess) {                                                    \
      printf("%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e)); \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

__global__ void zc_copy(const uint4* __restrict__ in, uint4* __restrict__ out, uint64_t n) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n; i += 4 * stride) {
    uint4 a = in[i], b = in[i + stride], c = in[i + 2 * stride], d = in[i + 3 * stride];
    out[i] = a;
    out[i + stride] = b;
    out[i + 2 * stride] = c;
    out[i + 3 * stride] = d;
  }
  for (; i < n; i += stride) out[i] = in[i];
}

int main(int argc, char** argv) {
  const uint64_t bytes = (argc > 1 ? atoll(argv[1]) : 8) << 30;
  const int grid_ctas = argc > 2 ? atoi(argv[2]) : 148 * 4;
  uint8_t *h, *d, *hd;
  CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped));
  CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  CK(cudaMalloc(&d, bytes));
  CK(cudaMemset(d, 7, bytes));
  memset(h, 3, bytes);
  cudaStream_t s1, s2;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, e2;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreate(&e2));
  const uint64_t piece = 64ull << 20;
  auto run = [&](bool d2h, double f) {
    // bytes [0, ce_end) by the copy engine, [ce_end, bytes) by the kernel
    uint64_t ce_end = (uint64_t)((1.0 - f) * bytes) / piece * piece;
    float best = 1e30f;
    for (int rep = 0; rep < 3; ++rep) {
      CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(e0, s1));
      CK(cudaStreamWaitEvent(s2, e0, 0));
      for (uint64_t a = 0; a < ce_end; a += piece) {
        if (d2h) CK(cudaMemcpyAsync(h + a, d + a, piece, cudaMemcpyDeviceToHost, s1));
        else CK(cudaMemcpyAsync(d + a, h + a, piece, cudaMemcpyHostToDevice, s1));
      }
      if (ce_end < bytes) {
        uint64_t n = (bytes - ce_end) / 16;
        if (d2h) zc_copy<<<grid_ctas, 256, 0, s2>>>((const uint4*)(d + ce_end), (uint4*)(hd + ce_end), n);
        else zc_copy<<<grid_ctas, 256, 0, s2>>>((const uint4*)(hd + ce_end), (uint4*)(d + ce_end), n);
        CK(cudaGetLastError());
      }
      CK(cudaEventRecord(e2, s2));
      CK(cudaStreamWaitEvent(s1, e2, 0));
      CK(cudaEventRecord(e1, s1));
      CK(cudaEventSynchronize(e1));
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      best = std::min(best, ms);
    }
    printf("%s  kernel share %.2f  %7.2f GB/s  (%.1f ms for %.2f GB)\n", d2h ? "D2H" : "H2D", f,
           bytes / (best * 1e-3) / 1e9, best, bytes / 1e9);
    fflush(stdout);
  };
  printf("link_mix_probe: %.2f GB, kernel grid %d x 256\n", bytes / 1e9, grid_ctas);
  for (int d2h = 1; d2h >= 0; --d2h)
    for (double f : {0.0, 1.0, 0.05, 0.1, 0.2, 0.3, 0.5})
      run(d2h, f);
  return 0;
}
