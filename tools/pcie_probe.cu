// PCIe copy-engine probe: D2H / H2D throughput into different host buffers
// (cudaHostAlloc, shm mmap + cudaHostRegister, malloc + cudaHostRegister)
// with 1, 2 or 4 concurrent copy streams, 4 GiB per measurement.
#include <cuda_runtime.h>
#include <fcntl.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <unistd.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
int main() {
  const size_t N = 4ull << 30;
  uint8_t* d; CK(cudaMalloc(&d, N)); CK(cudaMemset(d, 1, N));
  uint8_t* hb[3];
  CK(cudaHostAlloc(&hb[0], N, cudaHostAllocDefault));
  int fd = open("/dev/shm/pcie_probe", O_RDWR | O_CREAT, 0600); if (ftruncate(fd, N)) return 1;
  hb[1] = (uint8_t*)mmap(nullptr, N, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0); close(fd);
  CK(cudaHostRegister(hb[1], N, cudaHostRegisterMapped | cudaHostRegisterPortable));
  hb[2] = (uint8_t*)aligned_alloc(1 << 21, N); memset(hb[2], 0, N);
  CK(cudaHostRegister(hb[2], N, cudaHostRegisterPortable));
  const char* names[3] = {"cudaHostAlloc", "shm+register", "malloc+register"};
  cudaStream_t s[4]; for (auto& x : s) CK(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  for (int b = 0; b < 3; ++b)
    for (int dir = 0; dir < 2; ++dir)
      for (int ns : {1, 2, 4}) {
        for (int rep = 0; rep < 2; ++rep) {
          CK(cudaDeviceSynchronize());
          CK(cudaEventRecord(e0, s[0]));
          for (int i = 1; i < ns; ++i) CK(cudaStreamWaitEvent(s[i], e0, 0));
          size_t piece = 256ull << 20;
          for (size_t off = 0, j = 0; off < N; off += piece, ++j) {
            cudaStream_t st = s[j % ns];
            if (dir == 0) CK(cudaMemcpyAsync(hb[b] + off, d + off, piece, cudaMemcpyDeviceToHost, st));
            else CK(cudaMemcpyAsync(d + off, hb[b] + off, piece, cudaMemcpyHostToDevice, st));
          }
          for (int i = 1; i < ns; ++i) { cudaEvent_t ev; CK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)); CK(cudaEventRecord(ev, s[i])); CK(cudaStreamWaitEvent(s[0], ev, 0)); }
          CK(cudaEventRecord(e1, s[0])); CK(cudaEventSynchronize(e1));
          float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
          if (rep) printf("%-16s %s streams=%d  %.1f GB/s\n", names[b], dir ? "H2D" : "D2H", ns, N / (ms * 1e-3) / 1e9);
        }
      }
  unlink("/dev/shm/pcie_probe");
  return 0;
}
