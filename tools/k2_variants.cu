// K2 (pack + JF64) variant sweep (tools only; round 2 experiment).
//
// Same work as the library's K2 over an 8 GiB launch of 32 KiB aligned
// segments (1 MiB chunks): read the tensor bytes, hash every 8-byte word,
// store 16-byte vectors into the staging image, one atomic per warp per
// chunk.  Variants change only the streaming core: threads per CTA, vectors
// in flight per thread, whether the loads are forced ahead of the hashing
// (asm volatile), occupancy hint, and store flavour.  Also timed: the
// library's own launch_segments(kPack) and a D2D cudaMemcpyAsync, on the same
// buffers, so all numbers come from one box in one process.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//   -I paper_conf_eurosys_guptakkvgkrs24_b200/csrc tools/k2_variants.cu \
//   -L paper_conf_eurosys_guptakkvgkrs24_b200 -l:libjitc.so \
//   -Xlinker -rpath=$PWD/paper_conf_eurosys_guptakkvgkrs24_b200 -o tools/k2_variants
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <functional>
#include <vector>

#include "jitc_internal.h"

#ifdef K2V_INCLUDE_LIB
// the library's kernels compiled into this translation unit (no libjitc.so)
#include "../paper_conf_eurosys_guptakkvgkrs24_b200/csrc/jitc_kernels.cu"
namespace jitc {
void set_error(const std::string&) {}
}
#endif

using namespace jitc;

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e = (x);                                                         \
    if (e != cudaSuccess) {                                                      \
      printf("%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e));   \
      exit(1);                                                                   \
    }                                                                            \
  } while (0)

constexpr uint64_t K2V_PHI = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t k2v_dmix(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

template <int LDV>
__device__ __forceinline__ uint4 ldv(const uint4* p) {
  uint4 v;
  if (LDV == 0)
    asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
        : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  else if (LDV == 1)
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  return v;
}
template <int STV>
__device__ __forceinline__ void stv(uint4* p, uint4 v) {
  if (STV == 3) return;  // K1: digest only
  if (STV == 0) __stcs(p, v);
  else if (STV == 1) *p = v;
  else
    asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
                 "r"(v.w) : "memory");
}

__device__ __forceinline__ uint64_t k2v_warp_sum(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Aligned-segment K2 core.  HASH=0: plain copy with the same work split.
template <int T, int U, int MINB, int LDV, int STV, int HASH, int BATCH>
__global__ void __launch_bounds__(T, MINB) k2v(const Seg* __restrict__ segs, uint32_t total, uint8_t* img_base,
                                               unsigned long long* __restrict__ dig, unsigned int* __restrict__ work) {
  const uint32_t nbatch = (total + BATCH - 1) / BATCH;
  const int tid = threadIdx.x, lane = tid & 31;
  __shared__ uint32_t s_batch;
  uint64_t acc = 0;
  uint32_t cur = 0xFFFFFFFFu;
  for (;;) {
    if (tid == 0) s_batch = atomicAdd(work, 1u);
    __syncthreads();
    const uint32_t b = s_batch;
    __syncthreads();
    if (b >= nbatch) break;
    const uint32_t v0 = b * BATCH, v1 = min(total, v0 + BATCH);
    Seg nx = segs[v0];
    for (uint32_t v = v0; v < v1; ++v) {
      const Seg sg = nx;
      if (v + 1 < v1) nx = segs[v + 1];
      if (HASH && sg.chunk != cur) {
        if (cur != 0xFFFFFFFFu) {
          uint64_t a = k2v_warp_sum(acc);
          if (lane == 0) atomicAdd(dig + cur, (unsigned long long)a);
        }
        acc = 0;
        cur = sg.chunk;
      }
      const uint4* in = reinterpret_cast<const uint4*>(sg.src);
      uint4* out = reinterpret_cast<uint4*>(img_base + sg.img_off);
      const uint32_t nvec = sg.data_bytes >> 4;
      uint32_t i = tid;
      uint64_t key = ((sg.img_off >> 3) + 2ull * i + 1ull) * K2V_PHI;
      const uint64_t kstep = 2ull * T * K2V_PHI;
      for (; i + (U - 1) * T < nvec; i += U * T) {
        uint4 x[U];
#pragma unroll
        for (int u = 0; u < U; ++u) x[u] = ldv<LDV>(in + i + u * T);
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (HASH) {
            acc += k2v_dmix(((uint64_t)x[u].x | ((uint64_t)x[u].y << 32)) ^ key);
            acc += k2v_dmix(((uint64_t)x[u].z | ((uint64_t)x[u].w << 32)) ^ (key + K2V_PHI));
            key += kstep;
          }
          stv<STV>(out + i + u * T, x[u]);
        }
      }
      for (; i < nvec; i += T) {
        uint4 x = ldv<LDV>(in + i);
        if (HASH) {
          acc += k2v_dmix(((uint64_t)x.x | ((uint64_t)x.y << 32)) ^ key);
          acc += k2v_dmix(((uint64_t)x.z | ((uint64_t)x.w << 32)) ^ (key + K2V_PHI));
          key += kstep;
        }
        stv<STV>(out + i, x);
      }
    }
  }
  if (HASH && cur != 0xFFFFFFFFu) {
    uint64_t a = k2v_warp_sum(acc);
    if (lane == 0) atomicAdd(dig + cur, (unsigned long long)a);
  }
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(work + 1, 1u) == gridDim.x - 1) {
      work[0] = 0;
      work[1] = 0;
      __threadfence();
    }
  }
}

// Flat grid-stride copy (no segments), the simplest possible streaming kernel.
template <int U>
__global__ void __launch_bounds__(256) flat_copy(const uint4* __restrict__ in, uint4* __restrict__ out, uint64_t n) {
  uint64_t stride = (uint64_t)gridDim.x * 256;
  uint64_t i = blockIdx.x * 256ull + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 x[U];
#pragma unroll
    for (int u = 0; u < U; ++u) x[u] = ldv<1>(in + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) __stcs(out + i + u * stride, x[u]);
  }
  for (; i < n; i += stride) __stcs(out + i, ldv<1>(in + i));
}

struct Bench {
  uint8_t *src, *stage;
  uint64_t bytes;
  Seg* d_segs;
  uint32_t nseg;
  unsigned long long* dig;
  unsigned int* work;
  cudaStream_t s;
  cudaEvent_t e0, e1;
  int sms;
  int reps;
  uint64_t want_dig_sum = 0;
  bool have_want = false;

  template <class F>
  void time(const char* name, double rw, F launch) {
    CK(cudaMemsetAsync(dig, 0, (bytes >> 20) * 8 + 8, s));
    launch();  // warm-up + digest check
    CK(cudaStreamSynchronize(s));
    CK(cudaGetLastError());
    std::vector<unsigned long long> h((bytes >> 20) + 1);
    CK(cudaMemcpy(h.data(), dig, h.size() * 8, cudaMemcpyDeviceToHost));
    uint64_t sum = 0;
    for (auto x : h) sum = sum * 31 + x;
    std::vector<float> ms;
    for (int r = 0; r < reps; ++r) {
      CK(cudaEventRecord(e0, s));
      launch();
      CK(cudaEventRecord(e1, s));
      CK(cudaEventSynchronize(e1));
      float t;
      CK(cudaEventElapsedTime(&t, e0, e1));
      ms.push_back(t);
    }
    std::sort(ms.begin(), ms.end());
    double med = ms[ms.size() / 2], best = ms[0];
    printf("%-44s median %8.3f ms  %7.0f GB/s   best %7.0f GB/s   digsum %016llx\n", name, med,
           rw * bytes / (med * 1e-3) / 1e9, rw * bytes / (best * 1e-3) / 1e9, (unsigned long long)sum);
  }
};

template <int T, int U, int MINB, int LDV, int STV, int HASH, int BATCH>
void run_variant(Bench& B, const char* name, int per_sm) {
  int per = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k2v<T, U, MINB, LDV, STV, HASH, BATCH>, T, 0));
  if (per_sm > 0) per = std::min(per, per_sm);
  int grid = B.sms * per;
  cudaFuncAttributes fa;
  CK(cudaFuncGetAttributes(&fa, k2v<T, U, MINB, LDV, STV, HASH, BATCH>));
  char full[160];
  snprintf(full, sizeof full, "%s r%d g%d", name, fa.numRegs, grid);
  B.time(full, 2.0, [&] {
    k2v<T, U, MINB, LDV, STV, HASH, BATCH><<<grid, T, 0, B.s>>>(B.d_segs, B.nseg, B.stage, B.dig, B.work);
  });
}

int main(int argc, char** argv) {
  Bench B{};
  B.bytes = (argc > 1 ? atoll(argv[1]) : 8192ull) << 20;
  B.reps = argc > 2 ? atoi(argv[2]) : 10;
  CK(cudaDeviceGetAttribute(&B.sms, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaMalloc(&B.src, B.bytes));
  CK(cudaMalloc(&B.stage, B.bytes));
  // non-trivial contents (digests differ per word)
  {
    std::vector<uint64_t> h(1 << 20);
    for (size_t i = 0; i < h.size(); ++i) h[i] = mix64(i * 0x1234567ull + 99);
    for (uint64_t off = 0; off < B.bytes; off += h.size() * 8)
      CK(cudaMemcpy(B.src + off, h.data(), std::min<uint64_t>(h.size() * 8, B.bytes - off), cudaMemcpyHostToDevice));
  }
  std::vector<Seg> segs;
  const uint32_t seg_bytes = getenv("K2V_SEG_KIB") ? (uint32_t)atoi(getenv("K2V_SEG_KIB")) << 10 : kMaxSegBytes;
  for (uint64_t off = 0; off < B.bytes; off += seg_bytes) {
    Seg sg{};
    sg.src = (uint64_t)(B.src + off);
    sg.img_off = off;
    sg.data_bytes = seg_bytes;
    sg.chunk = (uint32_t)(off >> 20);
    sg.flags = kSegAligned16 | kSegAligned8;
    segs.push_back(sg);
  }
  B.nseg = (uint32_t)segs.size();
  CK(cudaMalloc(&B.d_segs, segs.size() * sizeof(Seg)));
  CK(cudaMemcpy(B.d_segs, segs.data(), segs.size() * sizeof(Seg), cudaMemcpyHostToDevice));
  CK(cudaMalloc(&B.dig, ((B.bytes >> 20) + 1) * 8));
  CK(cudaMalloc(&B.work, 64));
  CK(cudaMemset(B.work, 0, 64));
  CK(cudaStreamCreateWithFlags(&B.s, cudaStreamNonBlocking));
  CK(cudaEventCreate(&B.e0));
  CK(cudaEventCreate(&B.e1));
  printf("K2 variants: %llu MiB per launch, %u segments of %u B, %d SMs, %d reps\n",
         (unsigned long long)(B.bytes >> 20), B.nseg, seg_bytes, B.sms, B.reps);

  if (getenv("K2V_SWEEP1")) {
    B.time("cudaMemcpyAsync D2D (copy, no hash)", 2.0, [&] {
      CK(cudaMemcpyAsync(B.stage, B.src, B.bytes, cudaMemcpyDeviceToDevice, B.s));
    });
    run_variant<256, 4, 1, 0, 0, 1, 8>(B, "K2 T256 U4 (= library)", 0);
    run_variant<512, 4, 1, 1, 0, 1, 8>(B, "K2 T512 U4 volatile-ld", 0);
    return 0;
  }
  // Round-robin sweep: every variant once per pass, so clock / power drift
  // over the run hits all of them alike; report the median over passes.
  struct V {
    const char* name;
    double rw;
    std::function<void()> go;
    std::vector<float> ms;
  };
  std::vector<V> vs;
  LaunchRanges lr{};
  lr.n = 1;
  lr.seg_end[0] = B.nseg;
  lr.prefix[1] = B.nseg;
  lr.base[0] = (uint64_t)B.stage;
  const int lib_grid = segment_grid(0);
  vs.push_back({"cudaMemcpyAsync D2D (copy, no hash)", 2.0,
                [&] { CK(cudaMemcpyAsync(B.stage, B.src, B.bytes, cudaMemcpyDeviceToDevice, B.s)); }, {}});
  vs.push_back({"libjitc K2 (library build)", 2.0,
                [&] { CK(launch_segments(kPack, B.d_segs, lr, (uint64_t*)B.dig, lib_grid, B.work, B.s, nullptr)); }, {}});
  vs.push_back({"libjitc K1 (read only)", 1.0,
                [&] { CK(launch_segments(kDigest, B.d_segs, lr, (uint64_t*)B.dig, lib_grid, B.work, B.s, nullptr)); }, {}});
#define VAR(T, U, B_, MINB, LDV, STV, name)                                                            \
  {                                                                                                    \
    int per = 0;                                                                                       \
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k2v<T, U, MINB, LDV, STV, 1, B_>, T, 0));   \
    cudaFuncAttributes fa;                                                                             \
    CK(cudaFuncGetAttributes(&fa, k2v<T, U, MINB, LDV, STV, 1, B_>));                                 \
    int grid = B.sms * per;                                                                            \
    vs.push_back({name, STV == 3 ? 1.0 : 2.0, [&B, grid] {                                             \
                    k2v<T, U, MINB, LDV, STV, 1, B_><<<grid, T, 0, B.s>>>(B.d_segs, B.nseg, B.stage, B.dig, B.work); \
                  }, {}});                                                                             \
    printf("%-36s grid %d regs %d local %d\n", name, grid, fa.numRegs, (int)fa.localSizeBytes);        \
  }
  if (getenv("K2V_SWEEP3")) {
    VAR(512, 4, 4, 1, 1, 0, "K2 T512 U4 b4");
    VAR(512, 4, 2, 1, 1, 0, "K2 T512 U4 b2");
    VAR(512, 4, 1, 1, 1, 0, "K2 T512 U4 b1");
    VAR(256, 4, 8, 1, 1, 3, "K1 T256 U4 b8 (read only)");
    VAR(256, 4, 4, 1, 1, 3, "K1 T256 U4 b4 (read only)");
    VAR(256, 4, 2, 1, 1, 3, "K1 T256 U4 b2 (read only)");
    VAR(256, 8, 2, 1, 1, 3, "K1 T256 U8 b2 (read only)");
  } else if (getenv("K2V_SWEEP2")) {
    VAR(512, 4, 4, 1, 1, 0, "K2 T512 U4 b4");
    VAR(512, 4, 4, 2, 1, 0, "K2 T512 U4 b4 minB2");
    VAR(512, 4, 4, 3, 1, 0, "K2 T512 U4 b4 minB3");
    VAR(512, 4, 6, 1, 1, 0, "K2 T512 U4 b6");
    VAR(512, 4, 3, 1, 1, 0, "K2 T512 U4 b3");
    VAR(512, 4, 4, 1, 0, 0, "K2 T512 U4 b4 nonvolatile-ld");
    VAR(512, 4, 4, 1, 2, 0, "K2 T512 U4 b4 L2::256B");
    VAR(512, 4, 4, 1, 1, 2, "K2 T512 U4 b4 st.na");
    VAR(512, 2, 4, 1, 1, 0, "K2 T512 U2 b4");
    VAR(256, 8, 4, 1, 1, 0, "K2 T256 U8 b4");
    VAR(256, 8, 4, 4, 1, 0, "K2 T256 U8 b4 minB4");
    VAR(256, 8, 2, 1, 1, 0, "K2 T256 U8 b2");
    VAR(128, 16, 2, 1, 1, 0, "K2 T128 U16 b2");
    VAR(512, 4, 4, 1, 1, 3, "K1 T512 U4 b4 (read only)");
    VAR(256, 4, 8, 1, 1, 3, "K1 T256 U4 b8 (read only)");
    VAR(512, 4, 8, 1, 1, 3, "K1 T512 U4 b8 (read only)");
    VAR(512, 8, 4, 2, 1, 3, "K1 T512 U8 b4 minB2 (read only)");
  } else {
    VAR(256, 4, 8, 1, 1, 0, "K2 T256 U4 b8");
    VAR(256, 4, 4, 1, 1, 0, "K2 T256 U4 b4");
    VAR(256, 8, 4, 1, 1, 0, "K2 T256 U8 b4");
    VAR(512, 4, 8, 1, 1, 0, "K2 T512 U4 b8");
    VAR(512, 4, 4, 1, 1, 0, "K2 T512 U4 b4");
    VAR(512, 4, 2, 1, 1, 0, "K2 T512 U4 b2");
    VAR(384, 4, 4, 1, 1, 0, "K2 T384 U4 b4");
  }
  for (auto& v : vs) {  // warm-up
    v.go();
    CK(cudaStreamSynchronize(B.s));
  }
  for (int pass = 0; pass < B.reps; ++pass)
    for (auto& v : vs) {
      CK(cudaEventRecord(B.e0, B.s));
      v.go();
      CK(cudaEventRecord(B.e1, B.s));
      CK(cudaEventSynchronize(B.e1));
      float t;
      CK(cudaEventElapsedTime(&t, B.e0, B.e1));
      v.ms.push_back(t);
    }
  CK(cudaGetLastError());
  for (auto& v : vs) {
    std::sort(v.ms.begin(), v.ms.end());
    double med = v.ms[v.ms.size() / 2];
    printf("%-40s median %8.3f ms  %7.0f GB/s  (min..max %7.0f..%7.0f)\n", v.name, med, v.rw * B.bytes / (med * 1e-3) / 1e9,
           v.rw * B.bytes / (v.ms.back() * 1e-3) / 1e9, v.rw * B.bytes / (v.ms[0] * 1e-3) / 1e9);
  }
  return 0;
}
