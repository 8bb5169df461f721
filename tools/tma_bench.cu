// Experiment (tools only, not product): is a TMA-staged K2 faster than the
// LDG.128 K2 of libjitc?  DESIGN.md §7 "TMA" records the outcome.
//
// tma_pack: persistent CTAs, 16 KiB tiles moved global -> shared by
// cp.async.bulk (TMA bulk copy, mbarrier complete_tx), hashed from shared
// memory (JF64, the same definition as K2), and written shared -> global
// staging by cp.async.bulk bulk_group stores; an S-stage ring keeps S-1 loads
// and up to 2 stores in flight per CTA.  The arena is the kbench one: 32 KiB
// aligned segments laid out contiguously, so tile t of a launch is image
// bytes [t*16K, (t+1)*16K) and never crosses a 1 MiB chunk.
//
// Both kernels run over the same launches, with and without a concurrent D2H
// on another stream (the live capture condition), and the TMA kernel's staging
// bytes and digests are checked against seg_kernel<kPack>'s.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//   -I paper_conf_eurosys_guptakkvgkrs24_b200/csrc tools/tma_bench.cu \
//   -L paper_conf_eurosys_guptakkvgkrs24_b200 -l:libjitc.so \
//   -Xlinker -rpath=$PWD/paper_conf_eurosys_guptakkvgkrs24_b200 -o tools/tma_bench
// Run:   tools/tma_bench [launch_MiB=4096] [arena_MiB=16384]
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <vector>

#include "jitc_internal.h"

using namespace jitc;

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e_ = (x);                                                      \
    if (e_ != cudaSuccess) {                                                   \
      printf("%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e_)); \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

constexpr int kT = 256;            // threads per CTA
constexpr uint32_t kTile = 16384;  // bytes per TMA tile
constexpr int kStages = 4;         // smem ring: 4 x 16 KiB = 64 KiB per CTA
constexpr uint64_t kPhi = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* m, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(m)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* m, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(m)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* m, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(m)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* m) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(m))
      : "memory");
}
__device__ __forceinline__ void bulk_store(void* dst, const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(smem_u32(src)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// src: contiguous tensor bytes of the launch; dst: staging; img0: image byte
// offset of tile 0 (for the JF64 keys); C: chunk bytes.
__global__ void __launch_bounds__(kT) tma_pack(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                               uint64_t ntiles, uint64_t img0, uint64_t C,
                                               unsigned long long* __restrict__ dig) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[kStages];
  const int tid = threadIdx.x, lane = tid & 31;
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // this CTA's tiles: blockIdx.x + i * gridDim.x, i = 0 .. n-1
  const uint64_t n = blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  auto tile_of = [&](uint64_t i) { return blockIdx.x + i * gridDim.x; };
  if (tid == 0)
    for (uint64_t i = 0; i < (uint64_t)(kStages - 1) && i < n; ++i) {
      mbar_expect_tx(&full[i], kTile);
      bulk_load(smem + i * kTile, src + tile_of(i) * kTile, kTile, &full[i]);
    }
  for (uint64_t i = 0; i < n; ++i) {
    const int s = (int)(i % kStages);
    mbar_wait(&full[s], (uint32_t)((i / kStages) & 1));
    const uint64_t t = tile_of(i);
    const uint64_t off = img0 + t * kTile;
    const uint4* in = reinterpret_cast<const uint4*>(smem + s * kTile);
    uint64_t acc = 0;
#pragma unroll
    for (int u = 0; u < (int)(kTile / 16 / kT); ++u) {
      const uint32_t v = tid + u * kT;
      const uint4 x = in[v];
      const uint64_t key = ((off >> 3) + 2ull * v + 1ull) * kPhi;
      acc += mix(((uint64_t)x.x | ((uint64_t)x.y << 32)) ^ key);
      acc += mix(((uint64_t)x.z | ((uint64_t)x.w << 32)) ^ (key + kPhi));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) atomicAdd(dig + off / C, (unsigned long long)acc);
    __syncthreads();  // every thread is done reading stage s
    if (tid == 0) {
      bulk_store(dst + t * kTile, smem + s * kTile, kTile);
      bulk_commit();
      // refill the stage freed by tile i-1 (its store must have finished reading)
      const uint64_t nx = i + kStages - 1;
      if (nx < n) {
        bulk_wait_read<1>();
        const int s2 = (int)(nx % kStages);
        mbar_expect_tx(&full[s2], kTile);
        bulk_load(smem + s2 * kTile, src + tile_of(nx) * kTile, kTile, &full[s2]);
      }
    }
  }
  if (tid == 0) bulk_wait_all();
}

// tma_pack_warp: the same pipeline per WARP instead of per CTA -- every warp
// owns a private S-stage ring of W-byte tiles in shared memory, lane 0 issues
// its bulk loads/stores, and the only synchronisation is __syncwarp and the
// warp's own mbarriers (no CTA-wide barrier per tile).
template <uint32_t W, int S>
__global__ void __launch_bounds__(kT) tma_pack_warp(const uint8_t* __restrict__ src, uint8_t* __restrict__ dst,
                                                    uint64_t ntiles, uint64_t img0, uint64_t C,
                                                    unsigned long long* __restrict__ dig) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t full[kT / 32][S];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint8_t* ring = smem + (size_t)wid * S * W;
  if (lane == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&full[wid][s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const uint64_t nw = (uint64_t)gridDim.x * (kT / 32);
  const uint64_t gw = (uint64_t)blockIdx.x * (kT / 32) + wid;
  const uint64_t n = gw < ntiles ? (ntiles - gw + nw - 1) / nw : 0;
  auto tile_of = [&](uint64_t i) { return gw + i * nw; };
  if (lane == 0)
    for (uint64_t i = 0; i < (uint64_t)(S - 1) && i < n; ++i) {
      mbar_expect_tx(&full[wid][i], W);
      bulk_load(ring + i * W, src + tile_of(i) * W, W, &full[wid][i]);
    }
  for (uint64_t i = 0; i < n; ++i) {
    const int s = (int)(i % S);
    mbar_wait(&full[wid][s], (uint32_t)((i / S) & 1));
    const uint64_t t = tile_of(i);
    const uint64_t off = img0 + t * W;
    const uint4* in = reinterpret_cast<const uint4*>(ring + s * W);
    uint64_t acc = 0;
#pragma unroll
    for (int u = 0; u < (int)(W / 16 / 32); ++u) {
      const uint32_t v = lane + u * 32;
      const uint4 x = in[v];
      const uint64_t key = ((off >> 3) + 2ull * v + 1ull) * kPhi;
      acc += mix(((uint64_t)x.x | ((uint64_t)x.y << 32)) ^ key);
      acc += mix(((uint64_t)x.z | ((uint64_t)x.w << 32)) ^ (key + kPhi));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) {
      atomicAdd(dig + off / C, (unsigned long long)acc);
      bulk_store(dst + t * W, ring + s * W, W);
      bulk_commit();
      const uint64_t nx = i + S - 1;
      if (nx < n) {
        bulk_wait_read<1>();
        const int s2 = (int)(nx % S);
        mbar_expect_tx(&full[wid][s2], W);
        bulk_load(ring + s2 * W, src + tile_of(nx) * W, W, &full[wid][s2]);
      }
    }
    __syncwarp();
  }
  if (lane == 0) bulk_wait_all();
}

struct Variant {
  const char* name;
  const void* fn;
  size_t smem;
  uint32_t tile;
};

int main(int argc, char** argv) {
  const uint64_t launch_bytes = (uint64_t)(argc > 1 ? atoll(argv[1]) : 4096) << 20;
  const uint64_t arena_bytes = (uint64_t)(argc > 2 ? atoll(argv[2]) : 16384) << 20;
  const uint32_t seg_bytes = kMaxSegBytes;
  const uint64_t C = 1 << 20;
  uint8_t *src, *stage_a, *stage_b;
  CK(cudaMalloc(&src, arena_bytes));
  CK(cudaMalloc(&stage_a, launch_bytes));
  CK(cudaMalloc(&stage_b, launch_bytes));
  // non-trivial contents (a fixed byte pattern would let a wrong key cancel)
  {
    std::vector<uint64_t> h(1 << 20);
    uint64_t z = 12345;
    for (auto& x : h) {
      z += kPhi;
      uint64_t y = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
      x = y ^ (y >> 27);
    }
    for (uint64_t o = 0; o < arena_bytes; o += h.size() * 8)
      CK(cudaMemcpy(src + o, h.data(), h.size() * 8, cudaMemcpyHostToDevice));
  }
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
  const uint64_t nch = arena_bytes / C;
  uint64_t *dig_a, *dig_b;
  CK(cudaMalloc(&dig_a, nch * 8));
  CK(cudaMalloc(&dig_b, nch * 8));
  cudaStream_t s, s2;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  uint8_t* host;
  CK(cudaHostAlloc(&host, 4ull << 30, cudaHostAllocDefault));
  uint32_t* work;
  CK(cudaMalloc(&work, 64));
  CK(cudaMemset(work, 0, 64));
  const int seg_grid = segment_grid(0);
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const uint32_t nl = (uint32_t)(arena_bytes / launch_bytes);
  const uint32_t per = (uint32_t)(launch_bytes / seg_bytes);
  printf("launch %llu MiB, arena %llu MiB, %u launches; seg_kernel grid %d\n",
         (unsigned long long)(launch_bytes >> 20), (unsigned long long)(arena_bytes >> 20), nl, seg_grid);

  std::vector<Variant> vs = {
      {"tma_pack CTA ring 4 x 16 KiB", (const void*)tma_pack, kStages * kTile, kTile},
      {"tma_pack_warp 4 x 4 KiB per warp", (const void*)tma_pack_warp<4096, 4>, 8 * 4 * 4096, 4096},
      {"tma_pack_warp 6 x 4 KiB per warp", (const void*)tma_pack_warp<4096, 6>, 8 * 6 * 4096, 4096},
      {"tma_pack_warp 3 x 8 KiB per warp", (const void*)tma_pack_warp<8192, 3>, 8 * 3 * 8192, 8192},
      {"tma_pack_warp 8 x 2 KiB per warp", (const void*)tma_pack_warp<2048, 8>, 8 * 8 * 2048, 2048},
      {"tma_pack_warp 12 x 2 KiB per warp", (const void*)tma_pack_warp<2048, 12>, 8 * 12 * 2048, 2048},
  };
  std::vector<int> grids;
  for (auto& v : vs) {
    CK(cudaFuncSetAttribute(v.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)v.smem));
    int per_sm = 0;
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, v.fn, kT, v.smem));
    grids.push_back(sms * per_sm);
    printf("  %-36s smem %6zu B  %d CTA/SM  grid %d\n", v.name, v.smem, per_sm, sms * per_sm);
  }

  auto launch_seg = [&](uint32_t j) {
    LaunchRanges r{};
    r.n = 1;
    r.seg_begin[0] = j * per;
    r.seg_end[0] = (j + 1) * per;
    r.prefix[1] = per;
    r.base[0] = (uint64_t)stage_a;
    r.base_off[0] = (uint64_t)j * launch_bytes;
    CK(launch_segments(kPack, d_segs, r, dig_a, seg_grid, work, s, nullptr, nullptr));
  };
  auto launch_var = [&](int k, uint32_t j) {
    const uint8_t* a0 = src + (uint64_t)j * launch_bytes;
    uint8_t* a1 = stage_b;
    uint64_t a2 = launch_bytes / vs[k].tile, a3 = (uint64_t)j * launch_bytes, a4 = C;
    unsigned long long* a5 = (unsigned long long*)dig_b;
    void* args[] = {&a0, &a1, &a2, &a3, &a4, &a5};
    CK(cudaLaunchKernel(vs[k].fn, dim3(grids[k]), dim3(kT), args, vs[k].smem, s));
  };

  // correctness of every variant: all digests and the last launch's staging bytes
  bool all_ok = true;
  CK(cudaMemset(dig_a, 0, nch * 8));
  for (uint32_t j = 0; j < nl; ++j) launch_seg(j);
  CK(cudaStreamSynchronize(s));
  std::vector<uint64_t> da(nch), db(nch);
  CK(cudaMemcpy(da.data(), dig_a, nch * 8, cudaMemcpyDeviceToHost));
  std::vector<uint8_t> sa(64 << 20), sb(64 << 20);
  for (size_t k = 0; k < vs.size(); ++k) {
    CK(cudaMemset(dig_b, 0, nch * 8));
    CK(cudaMemset(stage_b, 0, launch_bytes));
    for (uint32_t j = 0; j < nl; ++j) launch_var((int)k, j);
    CK(cudaStreamSynchronize(s));
    CK(cudaMemcpy(db.data(), dig_b, nch * 8, cudaMemcpyDeviceToHost));
    const bool dig_ok = da == db;
    bool img_ok = true;
    for (uint64_t o = 0; o < launch_bytes; o += sa.size()) {
      CK(cudaMemcpy(sa.data(), stage_a + o, sa.size(), cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(sb.data(), stage_b + o, sb.size(), cudaMemcpyDeviceToHost));
      img_ok &= memcmp(sa.data(), sb.data(), sa.size()) == 0;
    }
    printf("%-36s == seg_kernel<kPack>: digests %s, staging bytes %s\n", vs[k].name, dig_ok ? "equal" : "DIFFER",
           img_ok ? "equal" : "DIFFER");
    all_ok &= dig_ok && img_ok;
  }

  std::vector<cudaEvent_t> ev(2 * nl);
  for (auto& e : ev) CK(cudaEventCreate(&e));
  const uint64_t d2h_bytes = 4ull << 30;   // from the (>= 4 GiB) source arena
  auto timed = [&](const char* name, int k, bool d2h) {
    double best = 1e30;
    for (int rep = 0; rep < 3; ++rep) {
      if (d2h) CK(cudaMemcpyAsync(host, src, d2h_bytes, cudaMemcpyDeviceToHost, s2));
      for (uint32_t j = 0; j < nl; ++j) {
        CK(cudaEventRecord(ev[2 * j], s));
        k < 0 ? launch_seg(j) : launch_var(k, j);
        CK(cudaEventRecord(ev[2 * j + 1], s));
      }
      CK(cudaStreamSynchronize(s));
      CK(cudaStreamSynchronize(s2));
      double sum = 0;
      for (uint32_t j = 0; j < nl; ++j) {
        float ms;
        CK(cudaEventElapsedTime(&ms, ev[2 * j], ev[2 * j + 1]));
        sum += ms;
      }
      best = sum / nl < best ? sum / nl : best;
    }
    printf("%-36s %s %8.1f us/launch  %7.0f GB/s (read+write)\n", name, d2h ? "+D2H" : "    ", best * 1e3,
           2.0 * launch_bytes / (best * 1e-3) / 1e9);
  };
  for (int d2h = 0; d2h < 2; ++d2h) {
    timed("seg_kernel<kPack> (LDG.128/STG.128)", -1, d2h);
    for (size_t k = 0; k < vs.size(); ++k) timed(vs[k].name, (int)k, d2h);
  }
  return all_ok ? 0 : 2;
}
