// sm_100a kernels of libjitc.so.
//
//  K1 digest        : JF64 chunk digests of live tensors (reads L from HBM)
//  K2 pack+digest   : gather tensors -> contiguous image bytes (staging slot in
//                     HBM, or mapped pinned host memory), JF64 in the same pass
//  K3 unpack+verify : image bytes (staging slot / mapped host) -> scatter into
//                     the tensors, JF64 of the bytes read
//  K5 pull+verify   : (F1 fusion) the writers' tensors read directly over
//                     NVLink through CUDA IPC mappings -> the local tensors,
//                     JF64 in the same pass: transfer and verification in one
//                     kernel, no staging and no writer-side kernel
//  K4 (harness)     : counter-based synthetic state, optimizer-update and
//                     bit-flip injectors
//
// JF64 (reading R2; PAPER.md:162 names only "checksums"): for image word g
// (8 bytes, little-endian) term(g) = fmix64(w ^ (g+1)*PHI); d[chunk] is the
// wrap-around sum of its terms.  The sum is order-free, so every CTA adds its
// partial into d[chunk] with a 64-bit atomic and the result is deterministic.
//
// Work unit: one Seg = one piece (<= 128 KiB) of one tensor that never crosses
// a chunk boundary.  CTAs of a persistent grid grab batches of consecutive
// segments from an atomic counter; inside a segment every thread streams 16-byte vectors (4 or 8 loads in flight
// before any use), hashes both words, optionally stores, and the warp reduces its
// partial with shuffles before one atomicAdd per warp per chunk it touched.  Pure HBM
// (or PCIe) streaming: no tensor cores, no shared-memory reuse (every byte is
// touched once), so the design targets coalescing, MLP and a grid sized to
// the SM count.
//
// CTA shape per mode (round 2, tools/k2_variants.cu sweeps on B200,
// profiles/r02c_k2_variants.txt).  Work grabs of 128-256 KiB and enough loads
// in flight per SM are what matter; the per-segment bookkeeping (descriptor,
// range lookup, tail test) is amortised over 128 KiB segments:
//  * read+write kernels (K2, K3, K5): 512 threads x 4 vectors (32 KiB per
//    unrolled step), 2 CTAs per SM, one segment per grab.  6.84 TB/s vs
//    6.29 TB/s for round 1's 256-thread, 8-CTA, 32-register shape with 32 KiB
//    segments on the same box (a D2D cudaMemcpy: 6.5-6.6 TB/s);
//  * read-only K1: 256 threads x 8 vectors, 4 CTAs per SM, two segments per
//    grab: 7.34 vs 6.83 TB/s; with no stores in flight it needs more loads
//    per thread to cover the read latency.
#include <cuda_runtime.h>
#include <stdint.h>

#include <string.h>

#include <atomic>
#include <string>

#include "jitc_internal.h"

namespace jitc {

namespace {

// threads per CTA, vectors in flight per thread, resident CTAs per SM (the
// register budget given to ptxas: without it ptxas picks 32 registers and
// serialises the loads of a step), and segments per work grab, by mode
// (see the header)
template <int MODE> struct Shape { static constexpr int T = 512, U = 4, MINB = 2, B = 1; };
template <> struct Shape<kDigest> { static constexpr int T = 256, U = 8, MINB = 4, B = 2; };
constexpr uint64_t PHI = 0x9E3779B97F4A7C15ull;

__device__ __forceinline__ uint64_t dmix(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

// Loads are asm volatile so that all kUnroll loads of a step issue before
// the hashing that consumes them (measured +1-2% over letting ptxas interleave).
__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}
__device__ __forceinline__ uint4 ld_plain(const uint4* p) {
  uint4 v;
  asm volatile("ld.global.cs.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p));
  return v;
}
__device__ __forceinline__ void st_stream(uint4* p, uint4 v) { __stcs(p, v); }
__device__ __forceinline__ uint64_t lo64(uint4 v) { return (uint64_t)v.x | ((uint64_t)v.y << 32); }
__device__ __forceinline__ uint64_t hi64(uint4 v) { return (uint64_t)v.z | ((uint64_t)v.w << 32); }

// Assemble the little-endian word made of bytes [b, b+8) of a tensor piece
// whose first `data` bytes come from `src` (any alignment) and the rest are 0.
__device__ __forceinline__ uint64_t load_word_bytes(const uint8_t* src, uint64_t b, uint64_t data,
                                                    bool al8) {
  if (al8 && b + 8 <= data) return *reinterpret_cast<const uint64_t*>(src + b);
  uint64_t w = 0;
#pragma unroll
  for (int i = 7; i >= 0; --i) {
    uint64_t bi = b + i;
    uint64_t byte = bi < data ? (uint64_t)src[bi] : 0ull;
    w = (w << 8) | byte;
  }
  return w;
}

__device__ __forceinline__ void store_word_bytes(uint8_t* dst, uint64_t b, uint64_t data, uint64_t w,
                                                 bool al8) {
  if (al8 && b + 8 <= data) {
    *reinterpret_cast<uint64_t*>(dst + b) = w;
    return;
  }
#pragma unroll
  for (int i = 0; i < 8; ++i)
    if (b + i < data) dst[b + i] = (uint8_t)(w >> (8 * i));
}

__device__ __forceinline__ uint64_t warp_sum(uint64_t v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Segment v of the launch's virtual concatenation of ranges.
__device__ __forceinline__ const Seg* seg_at(const Seg* segs, const LaunchRanges& R, uint32_t v, int* r) {
  int k = 0;
  while (v >= R.prefix[k + 1]) ++k;
  *r = k;
  return segs + R.seg_begin[k] + (v - R.prefix[k]);
}

// Warp-reduce the partial digest and add it to the chunk's digest.
__device__ __forceinline__ void flush(unsigned long long* dig, uint32_t chunk, uint64_t acc, int lane) {
  acc = warp_sum(acc);
  if (lane == 0) atomicAdd(dig + chunk, (unsigned long long)acc);
}

// Dynamic work distribution: CTAs grab batches of Shape<MODE>::B consecutive
// segments (<= 256 KiB) from a global counter, so SMs that stream faster take
// more work and no CTA idles at the tail.  Inside a batch the next
// descriptor is prefetched while the current segment streams, and the
// partial digest stays in registers until the chunk changes.  The counter
// pair (next batch, finished CTAs) resets itself: the last CTA to finish
// zeroes it for the next launch on the stream.
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// span (optional, timing diagnostics; zeroed before the launch): span[0] =
// ~(first CTA start), span[1] = last CTA end, in %globaltimer nanoseconds
// (the start is stored inverted so that both ends are an atomicMax).
template <int MODE>
__global__ void __launch_bounds__(Shape<MODE>::T, Shape<MODE>::MINB) seg_kernel(const Seg* __restrict__ segs, LaunchRanges R,
                                                       unsigned long long* __restrict__ dig,
                                                       unsigned int* __restrict__ work,
                                                       const uint64_t* __restrict__ remote,
                                                       unsigned long long* __restrict__ span) {
  constexpr int kThreads = Shape<MODE>::T;
  constexpr int kUnroll = Shape<MODE>::U;
  constexpr uint32_t kBatch = Shape<MODE>::B;
  if (span && threadIdx.x == 0) atomicMax(span, ~gtimer());
  const uint32_t total = R.prefix[R.n];
  const uint32_t nbatch = (total + kBatch - 1) / kBatch;
  const int tid = threadIdx.x;
  const int lane = tid & 31;
  __shared__ uint32_t s_batch;
  uint64_t acc = 0;
  uint32_t cur_chunk = 0xFFFFFFFFu;
  for (;;) {
    if (tid == 0) s_batch = atomicAdd(work, 1u);
    __syncthreads();
    const uint32_t bidx = s_batch;
    __syncthreads();
    if (bidx >= nbatch) break;
    const uint32_t v0 = bidx * kBatch, v1 = min(total, v0 + kBatch);
    int r;
    Seg next = *seg_at(segs, R, v0, &r);
    int next_r = r;
    for (uint32_t v = v0; v < v1; ++v) {
      const Seg sg = next;
      r = next_r;
      if (v + 1 < v1) next = *seg_at(segs, R, v + 1, &next_r);
      if (sg.chunk != cur_chunk) {
        if (cur_chunk != 0xFFFFFFFFu) flush(dig, cur_chunk, acc, lane);
        acc = 0;
        cur_chunk = sg.chunk;
      }
      const uint64_t rel = sg.img_off - R.base_off[r];
      uint8_t* img = reinterpret_cast<uint8_t*>(R.base[r]) + rel;  // 16-B aligned (staging / host image)
      uint8_t* ten = reinterpret_cast<uint8_t*>(sg.src);
      // kPull: the same bytes in a peer's tensor, read over NVLink (CUDA IPC mapping)
      const uint8_t* peer = MODE == kPull ? reinterpret_cast<const uint8_t*>(remote[R.seg_begin[r] + (v - R.prefix[r])])
                                          : nullptr;
      const uint64_t data = sg.data_bytes;
      const uint64_t words = (data + sg.pad_bytes) >> 3;
      const uint64_t g0 = sg.img_off >> 3;
      uint64_t body_words = 0;
      const bool vec = MODE == kPull ? (((uint64_t)peer | sg.src) & 15) == 0 : (sg.flags & kSegAligned16) != 0;

      if (vec) {
        const uint32_t nvec = (uint32_t)(data >> 4);
        body_words = 2ull * nvec;
        const uint4* in = MODE == kUnpack ? reinterpret_cast<const uint4*>(img)
                        : MODE == kPull   ? reinterpret_cast<const uint4*>(peer)
                                          : reinterpret_cast<const uint4*>(ten);
        uint4* out = MODE == kPack ? reinterpret_cast<uint4*>(img)
                   : (MODE == kUnpack || MODE == kPull) ? reinterpret_cast<uint4*>(ten) : nullptr;
        uint32_t i = tid;
        // key of word 2i is (g0 + 2i + 1) * PHI; the step between a thread's
        // consecutive vectors is 2 * kThreads words.
        uint64_t key = (g0 + 2ull * i + 1ull) * PHI;
        const uint64_t kstep = 2ull * kThreads * PHI;
        for (; i + (kUnroll - 1) * kThreads < nvec; i += kUnroll * kThreads) {
          uint4 x[kUnroll];
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) x[u] = MODE == kUnpack ? ld_plain(in + i + u * kThreads)
                                                                   : ld_stream(in + i + u * kThreads);
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) {
            acc += dmix(lo64(x[u]) ^ key);
            acc += dmix(hi64(x[u]) ^ (key + PHI));
            key += kstep;
            if (MODE != kDigest) st_stream(out + i + u * kThreads, x[u]);
          }
        }
        for (; i < nvec; i += kThreads) {
          uint4 x = MODE == kUnpack ? ld_plain(in + i) : ld_stream(in + i);
          acc += dmix(lo64(x) ^ key);
          acc += dmix(hi64(x) ^ (key + PHI));
          key += kstep;
          if (MODE != kDigest) st_stream(out + i, x);
        }
      }
      // Remaining words: unaligned tensors (all of them), the < 16-byte data
      // tail, and the zero padding that closes the tensor's image slot.
      const bool al8 = MODE == kPull ? (((uint64_t)peer | sg.src) & 7) == 0 : (sg.flags & kSegAligned8) != 0;
      for (uint64_t w = body_words + tid; w < words; w += kThreads) {
        const uint64_t b = 8 * w;
        uint64_t x;
        if (MODE == kUnpack) {
          x = *reinterpret_cast<const uint64_t*>(img + b);
          if (b < data) store_word_bytes(ten, b, data, x, al8);
        } else if (MODE == kPull) {
          x = load_word_bytes(peer, b, data, al8);
          if (b < data) store_word_bytes(ten, b, data, x, al8);
        } else {
          x = load_word_bytes(ten, b, data, al8);
          if (MODE == kPack) *reinterpret_cast<uint64_t*>(img + b) = x;
        }
        acc += dmix(x ^ ((g0 + w + 1ull) * PHI));
      }
    }
  }
  if (cur_chunk != 0xFFFFFFFFu) flush(dig, cur_chunk, acc, lane);
  if (span) {
    __syncthreads();
    if (tid == 0) atomicMax(span + 1, gtimer());
  }
  // the last CTA out resets the counters for the next launch on this stream
  if (tid == 0) {
    __threadfence();
    if (atomicAdd(work + 1, 1u) == gridDim.x - 1) {
      work[0] = 0;
      work[1] = 0;
      __threadfence();
    }
  }
}

__global__ void phase_write_kernel(volatile uint64_t* slot, uint64_t value) {
  *slot = value;
  __threadfence_system();
}

// ----------------------------------------------------------------- K4 (harness)
__device__ __forceinline__ uint64_t dsplitmix(uint64_t z) {
  z += PHI;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint32_t gen_bits(uint64_t key, uint64_t seed, uint64_t j, uint32_t lo,
                                             uint32_t span, int pos) {
  uint64_t x = dsplitmix(seed ^ key ^ j);
  uint32_t sign = pos ? 0u : (uint32_t)(x >> 63);
  uint32_t e = lo + (uint32_t)(((x >> 32) & 0xFFFFull) % span);
  return (sign << 31) | (e << 23) | (uint32_t)(x & 0x7FFFFFull);
}
__device__ __forceinline__ uint16_t to_bf16_rne(uint32_t u) {
  return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}

__global__ void gen_kernel(uint8_t* out, uint32_t dtype, uint64_t numel, uint64_t seed, uint64_t key,
                           uint32_t lo, uint32_t span, int pos) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t j = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; j < numel; j += stride) {
    switch (dtype) {
      case 0: {  // u8: byte b = byte (b % 4) of fp32 word (b / 4)
        uint32_t w = gen_bits(key, seed, j >> 2, lo, span, pos);
        out[j] = (uint8_t)(w >> (8 * (j & 3)));
        break;
      }
      case 1:
        reinterpret_cast<uint16_t*>(out)[j] = to_bf16_rne(gen_bits(key, seed, j, lo, span, pos));
        break;
      case 2:
        reinterpret_cast<uint32_t*>(out)[j] = gen_bits(key, seed, j, lo, span, pos);
        break;
      case 3:
        out[j] = 0;
        break;
      default:
        out[j] = 0xFF;
        break;
    }
  }
}

__global__ void update_kernel(uint32_t* x, uint64_t e0, uint64_t count, uint64_t tid_key, uint64_t vkey) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += stride) {
    uint64_t j = e0 + i;
    uint64_t h = dmix((tid_key ^ j) ^ vkey);
    x[j] ^= (uint32_t)(h & 0xFFFFull);
  }
}

__global__ void rne_kernel(const uint32_t* m, uint16_t* p, uint64_t count) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count; i += stride)
    p[i] = to_bf16_rne(m[i]);
}

__global__ void bitflip_kernel(uint8_t* p, uint8_t mask) { *p ^= mask; }

// Emulated hung collective: spins on a DEVICE-memory flag (as NCCL kernels
// spin on flags their peers write over NVLink), released by release_kernel
// launched on a separate non-blocking stream.
__global__ void hang_kernel(volatile uint32_t* flag) {
  if (threadIdx.x == 0)
    while (*flag == 0) __nanosleep(2000);
  __syncthreads();
}
__global__ void release_kernel(uint32_t* flag, uint32_t v) {
  *reinterpret_cast<volatile uint32_t*>(flag) = v;
  __threadfence_system();
}

uint32_t* g_hang_d = nullptr;  // 64 device release flags
cudaStream_t g_hang_s = nullptr;

// Computed once, read by every launch (any thread: the watchdog's action
// launches too), hence atomics; a racing first computation stores the same value.
std::atomic<int> g_sms[64];
std::atomic<int> g_per[8];  // resident CTAs per SM, by mode

template <int MODE>
int per_sm() {
  int v = g_per[MODE].load(std::memory_order_relaxed);
  if (!v) {
    int per = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, seg_kernel<MODE>, Shape<MODE>::T, 0);
    v = per > 0 ? per : 1;
    g_per[MODE].store(v, std::memory_order_relaxed);
  }
  return v;
}

}  // namespace

// SM count of the device; launch_segments sizes each mode's persistent grid
// as this x the mode's resident CTAs per SM.
int segment_grid(int device) {
  if (device < 0 || device >= 64) return 148;
  int v = g_sms[device].load(std::memory_order_relaxed);
  if (!v) {
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device);
    v = sms > 0 ? sms : 148;
    g_sms[device].store(v, std::memory_order_relaxed);
  }
  return v;
}

// Force-load every kernel of this module.  With CUDA lazy loading
// (CUDA_MODULE_LOADING=LAZY, the default) a kernel's first launch loads its
// code, and that load waits behind work already running on the device -- e.g.
// a collective hung on a dead peer -- so a first launch inside the failure
// path would deadlock (measured: tools/debug/wd_debug*.py).  jitc_create calls this.
cudaError_t preload_kernels() {
  cudaFuncAttributes fa;
  const void* fns[] = {(const void*)seg_kernel<kDigest>, (const void*)seg_kernel<kPack>,
                       (const void*)seg_kernel<kUnpack>, (const void*)seg_kernel<kPull>,
                       (const void*)phase_write_kernel,
                       (const void*)gen_kernel, (const void*)update_kernel, (const void*)rne_kernel,
                       (const void*)bitflip_kernel, (const void*)hang_kernel, (const void*)release_kernel};
  for (const void* f : fns) {
    cudaError_t e = cudaFuncGetAttributes(&fa, f);
    if (e != cudaSuccess) return e;
  }
  // the grid sizes too, so that no launch in the failure path queries the device
  per_sm<kDigest>();
  per_sm<kPack>();
  per_sm<kUnpack>();
  per_sm<kPull>();
  return cudaGetLastError();
}

cudaError_t device_check(int device, std::string* why) {
  cudaDeviceProp p;
  cudaError_t e = cudaGetDeviceProperties(&p, device);
  if (e != cudaSuccess) {
    *why = std::string("cudaGetDeviceProperties: ") + cudaGetErrorString(e);
    return e;
  }
  if (p.major != 10) {
    *why = "device " + std::to_string(device) + " is sm_" + std::to_string(p.major) + std::to_string(p.minor) +
           "; libjitc is built for sm_100a only";
    return cudaErrorNoKernelImageForDevice;
  }
  e = preload_kernels();
  if (e != cudaSuccess) *why = std::string("sm_100a kernels not loadable: ") + cudaGetErrorString(e);
  return e;
}

cudaError_t launch_segments(int mode, const Seg* d_segs, const LaunchRanges& r, uint64_t* d_dig, int grid,
                            uint32_t* d_work, cudaStream_t s, const uint64_t* d_remote, unsigned long long* d_span) {
  uint32_t total = r.prefix[r.n];
  if (total == 0) return cudaSuccess;
  auto* dig = reinterpret_cast<unsigned long long*>(d_dig);
  // grid = SMs x resident CTAs of this mode, or fewer when there are fewer batches
  auto size = [&](int per, uint32_t batch) {
    uint32_t nbatch = (total + batch - 1) / batch, full = (uint32_t)grid * (uint32_t)per;
    return (int)(nbatch < full ? nbatch : full);
  };
  switch (mode) {
    case kDigest:
      seg_kernel<kDigest><<<size(per_sm<kDigest>(), Shape<kDigest>::B), Shape<kDigest>::T, 0, s>>>(
          d_segs, r, dig, d_work, nullptr, d_span);
      break;
    case kPack:
      seg_kernel<kPack><<<size(per_sm<kPack>(), Shape<kPack>::B), Shape<kPack>::T, 0, s>>>(d_segs, r, dig, d_work,
                                                                                          nullptr, d_span);
      break;
    case kUnpack:
      seg_kernel<kUnpack><<<size(per_sm<kUnpack>(), Shape<kUnpack>::B), Shape<kUnpack>::T, 0, s>>>(
          d_segs, r, dig, d_work, nullptr, d_span);
      break;
    case kPull:
      if (!d_remote) return cudaErrorInvalidValue;
      seg_kernel<kPull><<<size(per_sm<kPull>(), Shape<kPull>::B), Shape<kPull>::T, 0, s>>>(d_segs, r, dig, d_work,
                                                                                          d_remote, d_span);
      break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_phase_write(uint64_t* dev_slot, uint64_t value, cudaStream_t s) {
  phase_write_kernel<<<1, 1, 0, s>>>(dev_slot, value);
  return cudaGetLastError();
}

}  // namespace jitc

using namespace jitc;

static uint64_t host_mix(uint64_t x) { return jitc::mix64(x); }

extern "C" {

jitc_status jitc_gen_fill(void* dptr, uint32_t dtype, uint64_t numel, uint64_t seed, uint32_t group,
                          uint32_t gen_id, uint32_t exp_lo, uint32_t exp_hi, int32_t force_pos, void* stream) {
  if (!dptr && numel) { set_error("jitc_gen_fill: null pointer"); return JITC_EINVAL; }
  if (dtype > 4 || exp_hi < exp_lo || exp_hi > 254) { set_error("jitc_gen_fill: bad dtype/range"); return JITC_EINVAL; }
  if (!numel) return JITC_OK;
  uint64_t key = host_mix(((uint64_t)group << 48) ^ ((uint64_t)gen_id << 32));
  int grid = 148 * 8;
  gen_kernel<<<grid, 256, 0, (cudaStream_t)stream>>>((uint8_t*)dptr, dtype, numel, seed, key, exp_lo,
                                                     exp_hi - exp_lo + 1, force_pos);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { set_error(std::string("jitc_gen_fill: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

jitc_status jitc_inject_update(void* dptr, uint64_t e0, uint64_t count, uint32_t gen_id, uint64_t v, void* stream) {
  if (!dptr && count) { set_error("jitc_inject_update: null pointer"); return JITC_EINVAL; }
  if (!count) return JITC_OK;
  update_kernel<<<148 * 8, 256, 0, (cudaStream_t)stream>>>((uint32_t*)dptr, e0, count, (uint64_t)gen_id << 40,
                                                            v * PHI);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { set_error(std::string("jitc_inject_update: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

jitc_status jitc_inject_rne(const void* master, void* param, uint64_t count, void* stream) {
  if ((!master || !param) && count) { set_error("jitc_inject_rne: null pointer"); return JITC_EINVAL; }
  if (!count) return JITC_OK;
  rne_kernel<<<148 * 8, 256, 0, (cudaStream_t)stream>>>((const uint32_t*)master, (uint16_t*)param, count);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { set_error(std::string("jitc_inject_rne: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

jitc_status jitc_inject_bitflip(void* dptr, uint64_t byte, uint32_t bit, void* stream) {
  if (!dptr || bit > 7) { set_error("jitc_inject_bitflip: bad argument"); return JITC_EINVAL; }
  bitflip_kernel<<<1, 1, 0, (cudaStream_t)stream>>>((uint8_t*)dptr + byte, (uint8_t)(1u << bit));
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { set_error(std::string("jitc_inject_bitflip: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

jitc_status jitc_inject_hang(void* stream, int32_t n_ctas, uint32_t slot) {
  if (n_ctas <= 0 || slot >= 64) { set_error("jitc_inject_hang: bad argument"); return JITC_EINVAL; }
  cudaError_t e = cudaSuccess;
  if (!g_hang_d) {
    e = cudaMalloc(&g_hang_d, 64 * sizeof(uint32_t));
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&g_hang_s, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaMemset(g_hang_d, 0, 64 * sizeof(uint32_t));
    if (e != cudaSuccess) { set_error(std::string("jitc_inject_hang: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  }
  release_kernel<<<1, 1, 0, (cudaStream_t)stream>>>(g_hang_d + slot, 0u);   // arm, in stream order
  hang_kernel<<<n_ctas, 32, 0, (cudaStream_t)stream>>>(g_hang_d + slot);
  e = cudaGetLastError();
  if (e != cudaSuccess) { set_error(std::string("jitc_inject_hang: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

jitc_status jitc_inject_release(uint32_t slot) {
  if (!g_hang_d || slot >= 64) { set_error("jitc_inject_release: no hang injected"); return JITC_EINVAL; }
  release_kernel<<<1, 1, 0, g_hang_s>>>(g_hang_d + slot, 1u);
  cudaError_t e = cudaStreamSynchronize(g_hang_s);
  if (e != cudaSuccess) { set_error(std::string("jitc_inject_release: ") + cudaGetErrorString(e)); return JITC_ECUDA; }
  return JITC_OK;
}

}  // extern "C"
