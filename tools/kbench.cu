// Kernel micro-benchmark for K1/K2/K3 (tools only; links libjitc.so and calls
// its internal launcher).  Measures per-launch time of the pack kernel over
// a synthetic segment table under controlled conditions:
//   a) back-to-back launches, one event pair around all of them
//   b) an event pair around every launch (what JITC_F_TIME_KERNELS does)
//   c) b) with a concurrent D2H of pinned memory on another stream
//   d) b) with the source moving through a large arena (fresh pages per launch)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//   -I paper_conf_eurosys_guptakkvgkrs24_b200/csrc tools/kbench.cu \
//   -L paper_conf_eurosys_guptakkvgkrs24_b200 -l:libjitc.so \
//   -Xlinker -rpath=$PWD/paper_conf_eurosys_guptakkvgkrs24_b200 -o tools/kbench
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#include "jitc_internal.h"

using namespace jitc;

#define CK(x)                                                               \
  do {                                                                      \
    cudaError_t e = (x);                                                    \
    if (e != cudaSuccess) {                                                 \
      printf("%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e)); \
      exit(1);                                                              \
    }                                                                       \
  } while (0)

int main(int argc, char** argv) {
  const uint64_t launch_bytes = (argc > 1 ? atoll(argv[1]) : 256) << 20;
  const uint64_t arena_bytes = (argc > 2 ? atoll(argv[2]) : 8192ull) << 20;
  const int mode = argc > 3 ? atoi(argv[3]) : 2;
  const uint32_t seg_bytes = kMaxSegBytes;
  uint8_t *src, *stage;
  CK(cudaMalloc(&src, arena_bytes));
  CK(cudaMalloc(&stage, launch_bytes));
  CK(cudaMemset(src, 1, arena_bytes));
  uint64_t C = 1 << 20;
  std::vector<Seg> segs;
  for (uint64_t off = 0; off < arena_bytes; off += seg_bytes) {
    Seg s{};
    s.src = (uint64_t)(src + off);
    s.img_off = off;
    s.data_bytes = seg_bytes;
    s.pad_bytes = 0;
    s.chunk = (uint32_t)(off / C);
    s.flags = kSegAligned16 | kSegAligned8;
    segs.push_back(s);
  }
  Seg* d_segs;
  CK(cudaMalloc(&d_segs, segs.size() * sizeof(Seg)));
  CK(cudaMemcpy(d_segs, segs.data(), segs.size() * sizeof(Seg), cudaMemcpyHostToDevice));
  uint64_t* dig;
  CK(cudaMalloc(&dig, (arena_bytes / C + 1) * 8));
  CK(cudaMemset(dig, 0, (arena_bytes / C + 1) * 8));
  cudaStream_t s, s2;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  uint8_t* host;
  CK(cudaHostAlloc(&host, 4ull << 30, cudaHostAllocDefault));
  int grid = segment_grid(0);
  uint32_t* work;
  CK(cudaMalloc(&work, 64));
  CK(cudaMemset(work, 0, 64));
  uint32_t per = (uint32_t)(launch_bytes / seg_bytes);
  uint32_t nl = (uint32_t)(arena_bytes / launch_bytes);
  std::vector<cudaEvent_t> ev(2 * nl + 2);
  for (auto& evt : ev) CK(cudaEventCreate(&evt));
  auto run = [&](bool fresh, bool each, bool d2h, const char* name) {
    if (d2h) CK(cudaMemcpyAsync(host, src, 4ull << 30, cudaMemcpyDeviceToHost, s2));
    CK(cudaEventRecord(ev[0], s));
    for (uint32_t j = 0; j < nl; ++j) {
      uint32_t base = fresh ? j * per : 0;
      LaunchRanges r{};
      r.n = 1;
      r.seg_begin[0] = base;
      r.seg_end[0] = base + per;
      r.prefix[1] = per;
      r.base[0] = (uint64_t)stage;
      r.base_off[0] = (uint64_t)base * seg_bytes;
      if (each) CK(cudaEventRecord(ev[2 + 2 * j], s));
      CK(launch_segments(mode, d_segs, r, dig, grid, work, s, nullptr, nullptr));
      if (each) CK(cudaEventRecord(ev[3 + 2 * j], s));
    }
    CK(cudaEventRecord(ev[1], s));
    CK(cudaStreamSynchronize(s));
    CK(cudaStreamSynchronize(s2));
    float tot;
    CK(cudaEventElapsedTime(&tot, ev[0], ev[1]));
    double sum = 0;
    if (each)
      for (uint32_t j = 0; j < nl; ++j) {
        float ms;
        CK(cudaEventElapsedTime(&ms, ev[2 + 2 * j], ev[3 + 2 * j]));
        sum += ms;
      }
    double rw = mode == kDigest ? 1 : 2;
    printf("%-34s launches %u  span/launch %7.1f us (%6.0f GB/s)  event/launch %7.1f us\n", name, nl,
           1e3 * tot / nl, rw * launch_bytes / (tot / nl * 1e-3) / 1e9, each ? 1e3 * sum / nl : 0.0);
  };
  printf("mode %d launch %llu MiB arena %llu MiB grid %d seg %u B\n", mode, (unsigned long long)(launch_bytes >> 20),
         (unsigned long long)(arena_bytes >> 20), grid, seg_bytes);
  run(false, false, false, "same src, back-to-back");
  run(false, false, false, "same src, back-to-back");
  run(true, false, false, "fresh src, back-to-back");
  run(true, true, false, "fresh src, events each");
  run(true, true, true, "fresh src, events each, +D2H");
  run(false, true, true, "same src, events each, +D2H");
  return 0;
}
