// Probe (tools only): does the ~45 us per-launch penalty that a concurrent
// copy-engine D2H adds to K2 (profiles/r01_kbench.txt) depend on the size of
// the kernel's by-value parameters?  Hypothesis: launch commands and their
// inline parameters are fetched from the pushbuffer in host memory; those
// reads queue behind the D2H's posted writes on the PCIe link, so a larger
// parameter block costs more fetch latency per launch.
//
// The same streaming kernel (256 MiB copy, grid = 148 x 8, 256 threads) is
// launched with a 16-byte and with a 608-byte (LaunchRanges-sized) parameter
// block, alone and next to a 4 GiB D2H on another stream; CUDA events per
// launch, best of 3.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 tools/param_probe.cu -o tools/param_probe
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e_ = (x);                                                      \
    if (e_ != cudaSuccess) {                                                   \
      printf("%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

struct Big {
  uint64_t src, dst, n;
  uint64_t pad[73];  // 608 bytes in all, like jitc::LaunchRanges + the other K2 arguments
};

__device__ __forceinline__ void body(const uint4* __restrict__ s, uint4* __restrict__ d, uint64_t n) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    d[i] = s[i];
}
__global__ void copy_small(const uint4* s, uint4* d, uint64_t n) { body(s, d, n); }
__global__ void copy_big(Big b) {
  body(reinterpret_cast<const uint4*>(b.src), reinterpret_cast<uint4*>(b.dst), b.n + b.pad[72]);
}
__global__ void empty_small(int) {}
__global__ void empty_big(Big b) {
  if (b.pad[72] == 12345) printf("x");
}

int main(int argc, char** argv) {
  const uint64_t bytes = (uint64_t)(argc > 1 ? atoll(argv[1]) : 256) << 20;
  const int nl = 32;
  uint8_t *a, *b, *big;
  CK(cudaMalloc(&a, bytes));
  CK(cudaMalloc(&b, bytes));
  CK(cudaMalloc(&big, 4ull << 30));
  CK(cudaMemset(a, 1, bytes));
  uint8_t* host;
  CK(cudaHostAlloc(&host, 4ull << 30, cudaHostAllocDefault));
  cudaStream_t s, s2;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t ev[2 * nl];
  for (auto& e : ev) CK(cudaEventCreate(&e));
  Big P{};
  P.src = (uint64_t)a;
  P.dst = (uint64_t)b;
  P.n = bytes / 16;
  const int grid = 148 * 8;
  printf("param_probe: %d launches of %llu MiB copies, grid %d x 256; sizeof(Big) = %zu B\n", nl,
         (unsigned long long)(bytes >> 20), grid, sizeof(Big));
  auto timed = [&](const char* name, int kind, bool d2h) {
    double best = 1e30;
    for (int rep = 0; rep < 3; ++rep) {
      if (d2h) CK(cudaMemcpyAsync(host, big, 4ull << 30, cudaMemcpyDeviceToHost, s2));
      for (int j = 0; j < nl; ++j) {
        CK(cudaEventRecord(ev[2 * j], s));
        switch (kind) {
          case 0: copy_small<<<grid, 256, 0, s>>>((const uint4*)a, (uint4*)b, bytes / 16); break;
          case 1: copy_big<<<grid, 256, 0, s>>>(P); break;
          case 2: empty_small<<<grid, 256, 0, s>>>(0); break;
          default: empty_big<<<grid, 256, 0, s>>>(P); break;
        }
        CK(cudaEventRecord(ev[2 * j + 1], s));
      }
      CK(cudaStreamSynchronize(s));
      CK(cudaStreamSynchronize(s2));
      double sum = 0;
      for (int j = 0; j < nl; ++j) {
        float ms;
        CK(cudaEventElapsedTime(&ms, ev[2 * j], ev[2 * j + 1]));
        sum += ms;
      }
      best = sum / nl < best ? sum / nl : best;
    }
    printf("%-34s %s %8.1f us/launch\n", name, d2h ? "+D2H" : "    ", best * 1e3);
  };
  for (int d2h = 0; d2h < 2; ++d2h) {
    timed("copy, 24 B params", 0, d2h);
    timed("copy, 608 B params", 1, d2h);
    timed("empty, 4 B params", 2, d2h);
    timed("empty, 608 B params", 3, d2h);
  }
  // Is it the launches or the timing events?  32 launches bracketed by ONE
  // event pair (mode 0), by a timing event pair each (mode 1), or by a
  // non-timing event each plus one timing pair (mode 2).
  cudaEvent_t nt[2 * nl], t0, t1;
  for (auto& e : nt) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  CK(cudaEventCreate(&t0));
  CK(cudaEventCreate(&t1));
  auto batch = [&](const char* name, bool copy, int mode, bool d2h) {
    double best = 1e30;
    for (int rep = 0; rep < 3; ++rep) {
      if (d2h) CK(cudaMemcpyAsync(host, big, 4ull << 30, cudaMemcpyDeviceToHost, s2));
      CK(cudaEventRecord(t0, s));
      for (int j = 0; j < nl; ++j) {
        if (mode == 1) CK(cudaEventRecord(ev[2 * j], s));
        if (mode == 2) CK(cudaEventRecord(nt[2 * j], s));
        if (copy) copy_small<<<grid, 256, 0, s>>>((const uint4*)a, (uint4*)b, bytes / 16);
        else empty_small<<<grid, 256, 0, s>>>(0);
        if (mode == 1) CK(cudaEventRecord(ev[2 * j + 1], s));
        if (mode == 2) CK(cudaEventRecord(nt[2 * j + 1], s));
      }
      CK(cudaEventRecord(t1, s));
      CK(cudaStreamSynchronize(s));
      CK(cudaStreamSynchronize(s2));
      float ms;
      CK(cudaEventElapsedTime(&ms, t0, t1));
      best = ms / nl < best ? ms / nl : best;
    }
    printf("%-50s %s %8.1f us/launch (one pair around all %d)\n", name, d2h ? "+D2H" : "    ", best * 1e3, nl);
  };
  for (int d2h = 0; d2h < 2; ++d2h) {
    batch("empty, no per-launch events", false, 0, d2h);
    batch("empty, timing event pair per launch", false, 1, d2h);
    batch("empty, non-timing event pair per launch", false, 2, d2h);
    batch("copy 256 MiB, no per-launch events", true, 0, d2h);
    batch("copy 256 MiB, timing event pair per launch", true, 1, d2h);
    batch("copy 256 MiB, non-timing event pair per launch", true, 2, d2h);
  }
  return 0;
}
