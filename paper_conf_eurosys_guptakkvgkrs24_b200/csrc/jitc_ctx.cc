// libjitc.so context: registration, phase words, fingerprint, capture,
// commit, restore, verify, and the library-owned NCCL communicator.
//
// Method: PAPER.md §3 (user-level JIT checkpointing) -- healthy DP replicas
// save their GPU state after a peer fails, on side streams
// (:134), to rank-dependent locations with metadata written last (:136); the
// restore loads any consistent replica and discards corrupted ones (:140);
// the state may be at minibatch i or i+1 (:148); a replica's state can be
// copied straight to a reset GPU (:174, :184).
#include <cuda.h>
#include <errno.h>
#include <fcntl.h>
#include <nccl.h>
#include <stdio.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/types.h>
#include <unistd.h>

#include <algorithm>
#include <chrono>
#include <condition_variable>
#include <mutex>
#include <thread>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include "jitc_internal.h"

using namespace jitc;

namespace {

struct GroupState {
  uint32_t id = 0;
  int policy = JITC_REQUIRED;
  std::vector<int32_t> members;
  bool held = false;
  int slot = -1;  // phase-word slot
  // layout (held groups)
  std::vector<std::string> names;
  std::vector<jitc_tensor> t;
  std::vector<uint64_t> off;
  uint64_t C = 0, L = 0, n_c = 0, layout_hash = 0;
  std::vector<Seg> segs;
  Seg* d_segs = nullptr;
  uint64_t* d_dig = nullptr;   // K1 digests
  uint64_t* d_dig2 = nullptr;  // K2 / K3 digests
  // last fingerprint
  bool has_fp = false;
  std::vector<uint64_t> fp;
  uint64_t fp_root = 0, fp_version = 0;
  int fp_phase = 0;
  // last capture
  bool captured = false;
  uint64_t cap_v = 0;
  // manifest digests (after commit / restore) for jitc_verify
  bool has_man = false;
  std::vector<uint64_t> man_d;
  uint64_t man_root = 0;
  // host image
  uint8_t* img_h = nullptr;
  uint8_t* img_d = nullptr;  // device alias of the mapped host image
  size_t img_bytes = 0;
  bool img_shm = false;
  std::string img_path;
  std::vector<uint8_t> man_priv, commit_priv;  // private-memory manifest / commit
};

typedef CUresult (*PFN_writeValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);

}  // namespace

struct jitc_ctx {
  jitc_config cfg{};
  std::string image_dir;
  int device = 0;
  cudaStream_t s_comp = nullptr, s_copy = nullptr;
  bool own_streams = false;
  uint8_t* staging = nullptr;
  uint64_t staging_bytes = 0, slot_bytes = 0;
  bool own_staging = false;
  static constexpr int kSlots = 8;
  cudaEvent_t ev_ready[kSlots]{}, ev_free[kSlots]{};
  cudaEvent_t ev_t0 = nullptr, ev_t1 = nullptr, ev_join = nullptr;
  std::vector<cudaEvent_t> kev;  // kernel timing pairs
  std::vector<int> kev_kind;
  std::vector<uint64_t> kev_bytes;
  size_t kev_used = 0;
  uint64_t* phase_h = nullptr;
  uint64_t* phase_d = nullptr;
  int phase_used = 0;
  PFN_writeValue64 write_value64 = nullptr;
  std::map<uint32_t, GroupState> groups;
  uint64_t* h_dig = nullptr;  // pinned digest scratch
  size_t h_dig_n = 0;
  int grid = 0;
  // communicator
  ncclComm_t comm = nullptr;
  int comm_n = 0, comm_rank = -1;
  std::vector<int32_t> comm_job;  // comm rank -> job rank
  uint64_t* d_small = nullptr;    // 64 B device scratch for size exchange / barrier
  uint32_t* d_work = nullptr;     // K1/K2/K3 batch counters (self-resetting)
  uint64_t* h_small = nullptr;    // pinned
  // watchdog (NEXT-1): explicit event watch-list polled by a native thread
  struct Watch {
    cudaEvent_t ev;
    uint64_t tag;
    double t_added;
  };
  std::mutex wmu;
  std::condition_variable wcv;
  std::vector<Watch> watches;
  std::thread wthread;
  bool wrun = false, fired = false, action_done = false;
  uint64_t fired_tag = 0;
  double detect_ms = 0, waited_ms = 0, action_ms = 0;
  uint32_t timeout_ms = 0;
  int action = 0;
  jitc_hang_fn hang_fn = nullptr;
  void* hang_user = nullptr;
  jitc_status action_status = JITC_OK;
  jitc_stats action_stats{};
  // counters
  jitc_kernel_counter kc[4]{};
  uint64_t launches_in_call = 0;
  double kernel_ms_in_call = 0;
};

// ----------------------------------------------------------------- helpers
namespace {

jitc_status fail(jitc_status st, const std::string& msg) {
  set_error(msg);
  return st;
}

#define CU(call)                                                                                  \
  do {                                                                                            \
    cudaError_t e_ = (call);                                                                      \
    if (e_ != cudaSuccess)                                                                        \
      return fail(JITC_ECUDA, std::string(__func__) + ": " #call ": " + cudaGetErrorString(e_)); \
  } while (0)
#define NC(call)                                                                                  \
  do {                                                                                            \
    ncclResult_t r_ = (call);                                                                     \
    if (r_ != ncclSuccess)                                                                        \
      return fail(JITC_ENCCL, std::string(__func__) + ": " #call ": " + ncclGetErrorString(r_));  \
  } while (0)

double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

struct CallTimer {
  jitc_ctx* c;
  double t0;
  explicit CallTimer(jitc_ctx* ctx) : c(ctx), t0(now_ms()) {
    c->launches_in_call = 0;
    c->kernel_ms_in_call = 0;
    c->kev_used = 0;
  }
};

// Kernel launch with optional event bracketing (JITC_F_TIME_KERNELS).
jitc_status run_segments(jitc_ctx* c, GroupState& g, int mode, const LaunchRanges& r, uint64_t* dig,
                         uint64_t bytes) {
  bool timed = (c->cfg.flags & JITC_F_TIME_KERNELS) && c->kev_used + 2 <= c->kev.size();
  if (timed) CU(cudaEventRecord(c->kev[c->kev_used], c->s_comp));
  CU(launch_segments(mode, g.d_segs, r, dig, c->grid, c->d_work, c->s_comp));
  if (timed) {
    CU(cudaEventRecord(c->kev[c->kev_used + 1], c->s_comp));
    c->kev_kind[c->kev_used / 2] = mode;
    c->kev_bytes[c->kev_used / 2] = bytes;
    c->kev_used += 2;
  }
  c->launches_in_call++;
  c->kc[mode].launches++;
  c->kc[mode].bytes += bytes;
  return JITC_OK;
}

// After the call's work has completed: harvest kernel timings into counters.
void harvest(jitc_ctx* c) {
  for (size_t i = 0; i + 1 < c->kev_used; i += 2) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, c->kev[i], c->kev[i + 1]) == cudaSuccess) {
      c->kc[c->kev_kind[i / 2]].ms += ms;
      c->kernel_ms_in_call += ms;
    }
  }
  c->kev_used = 0;
}

void finish_stats(jitc_ctx* c, const CallTimer& t, jitc_stats* st, bool device_span) {
  harvest(c);
  if (!st) return;
  st->ms_host = now_ms() - t.t0;
  st->ms_kernel = c->kernel_ms_in_call;
  st->kernel_launches = c->launches_in_call;
  if (device_span) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, c->ev_t0, c->ev_t1) == cudaSuccess) st->ms_device = ms;
  }
}

// Segments whose image offset lies in [a, b) (segments never straddle a chunk
// boundary and rounds are chunk-aligned, so this is exact).
void seg_span(const GroupState& g, uint64_t a, uint64_t b, uint32_t* lo, uint32_t* hi) {
  auto cmp = [](const Seg& s, uint64_t v) { return s.img_off < v; };
  *lo = (uint32_t)(std::lower_bound(g.segs.begin(), g.segs.end(), a, cmp) - g.segs.begin());
  *hi = (uint32_t)(std::lower_bound(g.segs.begin(), g.segs.end(), b, cmp) - g.segs.begin());
}

LaunchRanges one_range(uint32_t lo, uint32_t hi, const void* base, uint64_t base_off) {
  LaunchRanges r{};
  r.n = 1;
  r.seg_begin[0] = lo;
  r.seg_end[0] = hi;
  r.prefix[0] = 0;
  r.prefix[1] = hi - lo;
  r.base[0] = (uint64_t)base;
  r.base_off[0] = base_off;
  return r;
}

void add_range(LaunchRanges& r, uint32_t lo, uint32_t hi, const void* base, uint64_t base_off) {
  r.seg_begin[r.n] = lo;
  r.seg_end[r.n] = hi;
  r.base[r.n] = (uint64_t)base;
  r.base_off[r.n] = base_off;
  r.prefix[r.n + 1] = r.prefix[r.n] + (hi - lo);
  r.n++;
}

jitc_status ensure_h_dig(jitc_ctx* c, size_t n) {
  if (n <= c->h_dig_n) return JITC_OK;
  if (c->h_dig) cudaFreeHost(c->h_dig);
  c->h_dig = nullptr;
  c->h_dig_n = 0;
  CU(cudaHostAlloc(&c->h_dig, std::max<size_t>(n, 1) * 8, cudaHostAllocDefault));
  c->h_dig_n = n;
  return JITC_OK;
}

void free_group(GroupState& g) {
  if (g.d_segs) cudaFree(g.d_segs);
  if (g.d_dig) cudaFree(g.d_dig);
  if (g.d_dig2) cudaFree(g.d_dig2);
  if (g.img_h) {
    if (g.img_shm) {
      cudaHostUnregister(g.img_h);
      munmap(g.img_h, g.img_bytes);
    } else {
      cudaFreeHost(g.img_h);
    }
  }
  g.d_segs = nullptr;
  g.d_dig = g.d_dig2 = nullptr;
  g.img_h = g.img_d = nullptr;
}

std::string gpath(const jitc_ctx* c, uint32_t g, const char* ext) {
  return c->image_dir + "/g" + std::to_string(g) + ext;
}

std::vector<TopoEntry> topology(const jitc_ctx* c) {
  std::vector<TopoEntry> t;
  for (auto& kv : c->groups) t.push_back(TopoEntry{kv.first, kv.second.policy, kv.second.members});
  return t;
}

int comm_rank_of(const jitc_ctx* c, int32_t job) {
  for (int i = 0; i < c->comm_n; ++i)
    if (c->comm_job[i] == job) return i;
  return -1;
}

bool write_file_atomic(const std::string& path, const uint8_t* p, size_t n) {
  std::string tmp = path + ".tmp";
  FILE* f = fopen(tmp.c_str(), "wb");
  if (!f) return false;
  bool ok = fwrite(p, 1, n, f) == n;
  ok = (fflush(f) == 0) && ok;
  ok = (fsync(fileno(f)) == 0) && ok;
  fclose(f);
  return ok && rename(tmp.c_str(), path.c_str()) == 0;
}

bool read_file(const std::string& path, std::vector<uint8_t>* out) {
  FILE* f = fopen(path.c_str(), "rb");
  if (!f) return false;
  fseek(f, 0, SEEK_END);
  long n = ftell(f);
  fseek(f, 0, SEEK_SET);
  out->resize(n > 0 ? (size_t)n : 0);
  bool ok = n <= 0 || fread(out->data(), 1, (size_t)n, f) == (size_t)n;
  fclose(f);
  return ok;
}

jitc_status barrier(jitc_ctx* c) {
  if (!c->comm) return JITC_OK;
  NC(ncclAllReduce(c->d_small, c->d_small + 1, 1, ncclUint64, ncclSum, c->comm, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  return JITC_OK;
}

}  // namespace

// =====================================================================
extern "C" {

const char* jitc_last_error(const jitc_ctx*) { return get_error().c_str(); }

jitc_status jitc_create(const jitc_config* cfg, jitc_ctx** out) {
  if (!cfg || !out) return fail(JITC_EINVAL, "jitc_create: null argument");
  *out = nullptr;
  uint64_t C = cfg->chunk_bytes ? cfg->chunk_bytes : (1ull << 20);
  if ((C & (C - 1)) || C < 4096 || C > (64ull << 20))
    return fail(JITC_EINVAL, "jitc_create: chunk_bytes must be a power of two in [4 KiB, 64 MiB]");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || cfg->device < 0 || cfg->device >= ndev)
    return fail(JITC_ECUDA, std::string("jitc_create: no CUDA device ") + std::to_string(cfg->device) + ": " +
                                cudaGetErrorString(e));
  CU(cudaSetDevice(cfg->device));
  std::string why;
  if (device_check(cfg->device, &why) != cudaSuccess) return fail(JITC_ECUDA, "jitc_create: " + why);

  std::unique_ptr<jitc_ctx> c(new jitc_ctx());
  c->cfg = *cfg;
  c->cfg.chunk_bytes = C;
  c->device = cfg->device;
  if (cfg->image_dir) c->image_dir = cfg->image_dir;
  c->cfg.image_dir = nullptr;
  if (cfg->streams[0] && cfg->streams[1]) {
    c->s_comp = (cudaStream_t)cfg->streams[0];
    c->s_copy = (cudaStream_t)cfg->streams[1];
  } else {
    CU(cudaStreamCreateWithFlags(&c->s_comp, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&c->s_copy, cudaStreamNonBlocking));
    c->own_streams = true;
  }
  c->staging_bytes = cfg->staging_bytes ? cfg->staging_bytes : (1ull << 30);
  if (cfg->staging) {
    c->staging = (uint8_t*)cfg->staging;
  } else {
    CU(cudaMalloc(&c->staging, c->staging_bytes));
    c->own_staging = true;
  }
  if ((uint64_t)c->staging % 256) return fail(JITC_EINVAL, "jitc_create: staging must be 256-byte aligned");
  uint64_t slot = cfg->slot_bytes ? cfg->slot_bytes : (256ull << 20);
  slot = std::max<uint64_t>(slot / C * C, C);
  while (slot > C && slot * 2 > c->staging_bytes) slot = std::max<uint64_t>(slot / 2 / C * C, C);
  if (slot > c->staging_bytes) return fail(JITC_EINVAL, "jitc_create: staging smaller than one chunk");
  c->slot_bytes = slot;
  for (int i = 0; i < jitc_ctx::kSlots; ++i) {
    CU(cudaEventCreateWithFlags(&c->ev_ready[i], cudaEventDisableTiming));
    CU(cudaEventCreateWithFlags(&c->ev_free[i], cudaEventDisableTiming));
  }
  CU(cudaEventCreate(&c->ev_t0));
  CU(cudaEventCreate(&c->ev_t1));
  CU(cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  if (c->cfg.flags & JITC_F_TIME_KERNELS) {
    c->kev.resize(2 * 2048);
    for (auto& ev : c->kev) CU(cudaEventCreate(&ev));
    c->kev_kind.resize(2048);
    c->kev_bytes.resize(2048);
  }
  CU(cudaHostAlloc(&c->phase_h, kMaxPhaseSlots * 8, cudaHostAllocMapped | cudaHostAllocPortable));
  memset(c->phase_h, 0, kMaxPhaseSlots * 8);
  CU(cudaHostGetDevicePointer((void**)&c->phase_d, c->phase_h, 0));
  CU(cudaMalloc(&c->d_small, 64));
  CU(cudaMemset(c->d_small, 0, 64));
  CU(cudaMalloc(&c->d_work, 64));
  CU(cudaMemset(c->d_work, 0, 64));
  CU(cudaHostAlloc(&c->h_small, 64, cudaHostAllocDefault));
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuStreamWriteValue64", &fn, cudaEnableDefault, &q) == cudaSuccess &&
      q == cudaDriverEntryPointSuccess)
    c->write_value64 = (PFN_writeValue64)fn;
  cudaGetLastError();
  c->grid = segment_grid(c->device);
  *out = c.release();
  return JITC_OK;
}

void jitc_destroy(jitc_ctx* c) {
  if (!c) return;
  jitc_watchdog_stop(c);
  cudaSetDevice(c->device);
  if (c->s_comp) cudaStreamSynchronize(c->s_comp);
  if (c->s_copy) cudaStreamSynchronize(c->s_copy);
  if (c->comm) ncclCommDestroy(c->comm);
  for (auto& kv : c->groups) free_group(kv.second);
  for (int i = 0; i < jitc_ctx::kSlots; ++i) {
    if (c->ev_ready[i]) cudaEventDestroy(c->ev_ready[i]);
    if (c->ev_free[i]) cudaEventDestroy(c->ev_free[i]);
  }
  for (auto& ev : c->kev) cudaEventDestroy(ev);
  if (c->ev_t0) cudaEventDestroy(c->ev_t0);
  if (c->ev_t1) cudaEventDestroy(c->ev_t1);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->phase_h) cudaFreeHost(c->phase_h);
  if (c->h_dig) cudaFreeHost(c->h_dig);
  if (c->h_small) cudaFreeHost(c->h_small);
  if (c->d_small) cudaFree(c->d_small);
  if (c->d_work) cudaFree(c->d_work);
  if (c->own_staging && c->staging) cudaFree(c->staging);
  if (c->own_streams) {
    cudaStreamDestroy(c->s_comp);
    cudaStreamDestroy(c->s_copy);
  }
  delete c;
}

// ------------------------------------------------------------ registration
static jitc_status declare(jitc_ctx* c, uint32_t group, int32_t policy, const int32_t* members, int32_t n_members,
                           bool held) {
  if (policy != JITC_REQUIRED && policy != JITC_OPTIONAL) return fail(JITC_EINVAL, "policy must be REQUIRED/OPTIONAL");
  if (n_members <= 0 || !members) return fail(JITC_EINVAL, "a group needs >= 1 member");
  if (group == JITC_ALL_GROUPS) return fail(JITC_EINVAL, "group id reserved");
  std::vector<int32_t> m(members, members + n_members);
  std::sort(m.begin(), m.end());
  if (std::adjacent_find(m.begin(), m.end()) != m.end()) return fail(JITC_EINVAL, "duplicate member");
  bool mine = std::binary_search(m.begin(), m.end(), c->cfg.rank);
  if (held && !mine) return fail(JITC_EINVAL, "jitc_register: this rank is not a member of the group");
  if (!held && mine) return fail(JITC_EINVAL, "jitc_declare_group: this rank is a member; use jitc_register");
  auto it = c->groups.find(group);
  if (it != c->groups.end()) {
    free_group(it->second);
    c->groups.erase(it);
  }
  GroupState& g = c->groups[group];
  g.id = group;
  g.policy = policy;
  g.members = m;
  g.held = held;
  if (held) {
    if (c->phase_used >= kMaxPhaseSlots) return fail(JITC_EINVAL, "too many groups");
    g.slot = c->phase_used++;
    c->phase_h[g.slot] = 0;
  }
  return JITC_OK;
}

jitc_status jitc_declare_group(jitc_ctx* c, uint32_t group, int32_t policy, const int32_t* members,
                               int32_t n_members) {
  if (!c) return fail(JITC_EINVAL, "jitc_declare_group: null ctx");
  return declare(c, group, policy, members, n_members, false);
}

jitc_status jitc_register(jitc_ctx* c, uint32_t group, int32_t policy, const int32_t* members, int32_t n_members,
                          const jitc_tensor* t, size_t n, uint64_t* layout_hash, uint64_t* image_bytes) {
  if (!c || (n && !t)) return fail(JITC_EINVAL, "jitc_register: null argument");
  CU(cudaSetDevice(c->device));
  for (size_t i = 0; i < n; ++i)
    if (t[i].nbytes && !t[i].ptr) return fail(JITC_EINVAL, "jitc_register: tensor " + std::to_string(i) + " has no pointer");
  jitc_status st = declare(c, group, policy, members, n_members, true);
  if (st) return st;
  GroupState& g = c->groups[group];
  g.C = c->cfg.chunk_bytes;
  g.names.resize(n);
  g.t.assign(t, t + n);
  for (size_t i = 0; i < n; ++i) {
    g.names[i] = t[i].name ? t[i].name : "";
    g.t[i].name = g.names[i].c_str();
  }
  g.off.resize(n);
  st = jitc_layout(g.t.data(), n, g.C, g.off.data(), &g.layout_hash, &g.L);
  if (st) return st;
  g.n_c = (g.L + g.C - 1) / g.C;
  // segment table: pieces <= kMaxSegBytes that never cross a chunk boundary
  g.segs.clear();
  for (size_t i = 0; i < n; ++i) {
    uint64_t nb = t[i].nbytes, base = (uint64_t)t[i].ptr;
    uint64_t end_img = align_up(g.off[i] + nb, kAlign);
    uint64_t p = 0;
    while (p < nb) {
      uint64_t img = g.off[i] + p;
      uint64_t to_chunk = (img / g.C + 1) * g.C - img;
      uint64_t len = std::min<uint64_t>({nb - p, to_chunk, (uint64_t)kMaxSegBytes});
      Seg s{};
      s.src = base + p;
      s.img_off = img;
      s.data_bytes = (uint32_t)len;
      s.pad_bytes = (p + len == nb) ? (uint32_t)(end_img - (img + len)) : 0u;
      s.chunk = (uint32_t)(img / g.C);
      s.flags = ((s.src % 16) == 0 ? kSegAligned16 : 0u) | ((s.src % 8) == 0 ? kSegAligned8 : 0u);
      g.segs.push_back(s);
      p += len;
    }
  }
  if (g.n_c > 0xFFFFFFFFull || g.segs.size() > 0xFFFFFFFFull) return fail(JITC_EINVAL, "jitc_register: group too large");
  CU(cudaMalloc(&g.d_segs, std::max<size_t>(g.segs.size(), 1) * sizeof(Seg)));
  if (!g.segs.empty())
    CU(cudaMemcpyAsync(g.d_segs, g.segs.data(), g.segs.size() * sizeof(Seg), cudaMemcpyHostToDevice, c->s_comp));
  CU(cudaMalloc(&g.d_dig, std::max<uint64_t>(g.n_c, 1) * 8));
  CU(cudaMalloc(&g.d_dig2, std::max<uint64_t>(g.n_c, 1) * 8));
  CU(cudaStreamSynchronize(c->s_comp));
  st = ensure_h_dig(c, g.n_c);
  if (st) return st;
  // host image: shared /dev/shm file (survives the process) or private pinned
  g.img_bytes = std::max<uint64_t>(align_up(g.L, 4096), 4096);
  if (!c->image_dir.empty()) {
    mkdir(c->image_dir.c_str(), 0700);
    g.img_path = gpath(c, group, ".img");
    int fd = open(g.img_path.c_str(), O_RDWR | O_CREAT, 0600);
    if (fd < 0) return fail(JITC_EIO, "jitc_register: open " + g.img_path + ": " + strerror(errno));
    struct stat sb;
    if (fstat(fd, &sb) != 0 || ((uint64_t)sb.st_size != g.img_bytes && ftruncate(fd, (off_t)g.img_bytes) != 0)) {
      close(fd);
      return fail(JITC_EIO, "jitc_register: size " + g.img_path + ": " + strerror(errno));
    }
    void* p = mmap(nullptr, g.img_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    close(fd);
    if (p == MAP_FAILED) return fail(JITC_EIO, "jitc_register: mmap " + g.img_path + ": " + strerror(errno));
    cudaError_t e = cudaHostRegister(p, g.img_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
    if (e != cudaSuccess) {
      munmap(p, g.img_bytes);
      return fail(JITC_ENOMEM, std::string("jitc_register: cudaHostRegister: ") + cudaGetErrorString(e));
    }
    g.img_h = (uint8_t*)p;
    g.img_shm = true;
  } else {
    cudaError_t e = cudaHostAlloc(&g.img_h, g.img_bytes, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) {
      g.img_h = nullptr;
      return fail(JITC_ENOMEM, std::string("jitc_register: cudaHostAlloc: ") + cudaGetErrorString(e));
    }
  }
  CU(cudaHostGetDevicePointer((void**)&g.img_d, g.img_h, 0));
  if (layout_hash) *layout_hash = g.layout_hash;
  if (image_bytes) *image_bytes = g.L;
  return JITC_OK;
}

// ------------------------------------------------------------ phase words
jitc_status jitc_mark(jitc_ctx* c, uint32_t group, uint64_t version, int32_t phase, void* stream) {
  if (!c) return fail(JITC_EINVAL, "jitc_mark: null ctx");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_mark: group not registered");
  if (phase != JITC_PHASE_CLEAN && phase != JITC_PHASE_DIRTY) return fail(JITC_EINVAL, "jitc_mark: bad phase");
  if (version >> 63) return fail(JITC_EINVAL, "jitc_mark: version too large");
  uint64_t w = (version << 1) | (uint64_t)phase;
  int slot = it->second.slot;
  if (!stream) {
    __atomic_store_n(&c->phase_h[slot], w, __ATOMIC_RELEASE);
    return JITC_OK;
  }
  if (c->write_value64) {
    CUresult r = c->write_value64((CUstream)stream, (CUdeviceptr)(c->phase_d + slot), w, 0);
    if (r == CUDA_SUCCESS) return JITC_OK;
  }
  CU(launch_phase_write(c->phase_d + slot, w, (cudaStream_t)stream));
  return JITC_OK;
}

jitc_status jitc_phase(jitc_ctx* c, uint32_t group, uint64_t* version, int32_t* phase) {
  if (!c || !version || !phase) return fail(JITC_EINVAL, "jitc_phase: null argument");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_phase: group not registered");
  uint64_t w = __atomic_load_n(&c->phase_h[it->second.slot], __ATOMIC_ACQUIRE);
  *version = w >> 1;
  *phase = (int32_t)(w & 1);
  return JITC_OK;
}

// ------------------------------------------------------------ communicator
jitc_status jitc_get_unique_id(void* id128) {
  if (!id128) return fail(JITC_EINVAL, "jitc_get_unique_id: null");
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  NC(ncclGetUniqueId(reinterpret_cast<ncclUniqueId*>(id128)));
  return JITC_OK;
}

jitc_status jitc_comm_init(jitc_ctx* c, const void* id128, int32_t nranks, int32_t comm_rank, const int32_t* job_ranks) {
  if (!c || !id128 || nranks <= 0 || comm_rank < 0 || comm_rank >= nranks)
    return fail(JITC_EINVAL, "jitc_comm_init: bad argument");
  CU(cudaSetDevice(c->device));
  if (c->comm) {
    ncclCommDestroy(c->comm);
    c->comm = nullptr;
  }
  ncclUniqueId id;
  memcpy(&id, id128, sizeof id);
  NC(ncclCommInitRank(&c->comm, nranks, id, comm_rank));
  c->comm_n = nranks;
  c->comm_rank = comm_rank;
  c->comm_job.resize(nranks);
  for (int i = 0; i < nranks; ++i) c->comm_job[i] = job_ranks ? job_ranks[i] : i;
  if (c->comm_job[comm_rank] != c->cfg.rank)
    return fail(JITC_EINVAL, "jitc_comm_init: job_ranks[comm_rank] != cfg.rank");
  return JITC_OK;
}

jitc_status jitc_comm_shrink(jitc_ctx* c, const int32_t* failed, int32_t n_failed) {
  if (!c || !c->comm) return fail(JITC_ESTATE, "jitc_comm_shrink: no communicator");
  if (n_failed < 0 || (n_failed && !failed)) return fail(JITC_EINVAL, "jitc_comm_shrink: bad list");
  CU(cudaSetDevice(c->device));
  std::vector<int> excl;
  for (int i = 0; i < n_failed; ++i) {
    int r = comm_rank_of(c, failed[i]);
    if (r < 0) return fail(JITC_EINVAL, "jitc_comm_shrink: rank not in communicator");
    if (r == c->comm_rank) return fail(JITC_EINVAL, "jitc_comm_shrink: cannot exclude self");
    excl.push_back(r);
  }
  std::sort(excl.begin(), excl.end());
  ncclComm_t nc = nullptr;
  NC(ncclCommShrink(c->comm, excl.data(), (int)excl.size(), &nc, nullptr, NCCL_SHRINK_ABORT));
  ncclCommAbort(c->comm);
  c->comm = nc;
  std::vector<int32_t> job;
  for (int i = 0; i < c->comm_n; ++i)
    if (!std::binary_search(excl.begin(), excl.end(), i)) job.push_back(c->comm_job[i]);
  c->comm_job = job;
  c->comm_n = (int)job.size();
  c->comm_rank = comm_rank_of(c, c->cfg.rank);
  return JITC_OK;
}

jitc_status jitc_comm_destroy(jitc_ctx* c) {
  if (!c) return fail(JITC_EINVAL, "jitc_comm_destroy: null ctx");
  if (c->comm) ncclCommDestroy(c->comm);
  c->comm = nullptr;
  c->comm_n = 0;
  c->comm_rank = -1;
  c->comm_job.clear();
  return JITC_OK;
}

// ------------------------------------------------------------ fingerprint (K1)
static jitc_status fingerprint_group(jitc_ctx* c, GroupState& g) {
  uint64_t w = __atomic_load_n(&c->phase_h[g.slot], __ATOMIC_ACQUIRE);
  g.fp_version = w >> 1;
  g.fp_phase = (int)(w & 1);
  if (g.n_c) {
    CU(cudaMemsetAsync(g.d_dig, 0, g.n_c * 8, c->s_comp));
    jitc_status st = run_segments(c, g, kDigest, one_range(0, (uint32_t)g.segs.size(), nullptr, 0), g.d_dig, g.L);
    if (st) return st;
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
  }
  CU(cudaStreamSynchronize(c->s_comp));
  g.fp.assign(c->h_dig, c->h_dig + g.n_c);
  g.fp_root = root_of(g.layout_hash, g.fp.data(), g.n_c);
  g.has_fp = true;
  return JITC_OK;
}

static RecordHdr record_of(const jitc_ctx* c, const GroupState& g) {
  RecordHdr h{};
  h.magic = kMagicRecord;
  h.fmt = 1;
  h.policy = (uint8_t)g.policy;
  h.phase = (uint8_t)g.fp_phase;
  h.rank = c->cfg.rank;
  h.group = g.id;
  h.version = g.fp_version;
  h.layout_hash = g.layout_hash;
  h.n_c = g.n_c;
  h.chunk_bytes = g.C;
  h.root = g.fp_root;
  h.image_bytes = g.L;
  return h;
}

jitc_status jitc_fingerprint(jitc_ctx* c, uint32_t group, void* blob, size_t cap, size_t* len) {
  if (!c || !len) return fail(JITC_EINVAL, "jitc_fingerprint: null argument");
  CU(cudaSetDevice(c->device));
  std::vector<GroupState*> sel;
  for (auto& kv : c->groups)
    if (kv.second.held && (group == JITC_ALL_GROUPS || kv.first == group)) sel.push_back(&kv.second);
  if (sel.empty()) return fail(JITC_EINVAL, "jitc_fingerprint: group not registered");
  size_t need = sizeof(BlobHdr);
  for (auto& kv : c->groups) need += sizeof(TopoHdr) + align_up(4 * kv.second.members.size(), 8);
  for (auto* g : sel) need += sizeof(RecordHdr) + 8 * g->n_c;
  *len = need;
  if (cap == 0) return JITC_OK;
  if (cap < need || !blob) return fail(JITC_EINVAL, "jitc_fingerprint: blob buffer too small");
  CallTimer t(c);
  for (auto* g : sel) {
    jitc_status st = fingerprint_group(c, *g);
    if (st) return st;
  }
  harvest(c);
  std::vector<std::pair<RecordHdr, const uint64_t*>> recs;
  for (auto* g : sel) recs.push_back({record_of(c, *g), g->fp.data()});
  std::vector<uint8_t> b = encode_blob(c->cfg.rank, topology(c), recs);
  if (b.size() != need) return fail(JITC_EINVAL, "jitc_fingerprint: internal size mismatch");
  memcpy(blob, b.data(), b.size());
  return JITC_OK;
}

// ------------------------------------------------------------ record exchange (C1)
jitc_status jitc_exchange_records(jitc_ctx* c, const void* mine, size_t len, void* all, size_t cap, size_t* all_len) {
  if (!c || !mine || !all_len || len < sizeof(BlobHdr)) return fail(JITC_EINVAL, "jitc_exchange_records: bad argument");
  if (!c->comm) {
    *all_len = len;
    if (cap == 0) return JITC_OK;
    if (cap < len || !all) return fail(JITC_EINVAL, "jitc_exchange_records: buffer too small");
    memcpy(all, mine, len);
    return JITC_OK;
  }
  CU(cudaSetDevice(c->device));
  const int n = c->comm_n;
  // 1. sizes
  uint64_t* dsz = reinterpret_cast<uint64_t*>(c->staging);
  c->h_small[0] = len;
  CU(cudaMemcpyAsync(dsz + c->comm_rank, c->h_small, 8, cudaMemcpyHostToDevice, c->s_comp));
  NC(ncclAllGather(dsz + c->comm_rank, dsz, 1, ncclUint64, c->comm, c->s_comp));
  std::vector<uint64_t> sizes(n);
  CU(cudaMemcpyAsync(sizes.data(), dsz, 8ull * n, cudaMemcpyDeviceToHost, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  uint64_t maxlen = 0, total = 0;
  for (uint64_t s : sizes) maxlen = std::max(maxlen, s), total += s;
  maxlen = align_up(maxlen, 256);
  *all_len = (size_t)(n * maxlen);   // capacity needed (the compacted result is `total` <= this)
  if (cap == 0) return JITC_OK;
  if (cap < n * maxlen || !all) return fail(JITC_EINVAL, "jitc_exchange_records: buffer too small");
  if (256 + n * maxlen > c->staging_bytes) return fail(JITC_ENOMEM, "jitc_exchange_records: blobs exceed staging");
  // 2. padded blobs, in place
  uint8_t* recv = c->staging + 256;
  CU(cudaMemcpyAsync(recv + c->comm_rank * maxlen, mine, len, cudaMemcpyHostToDevice, c->s_comp));
  NC(ncclAllGather(recv + c->comm_rank * maxlen, recv, maxlen, ncclUint8, c->comm, c->s_comp));
  CU(cudaMemcpyAsync(all, recv, n * maxlen, cudaMemcpyDeviceToHost, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  uint8_t* a = static_cast<uint8_t*>(all);
  uint64_t pos = 0;
  for (int r = 0; r < n; ++r) {
    memmove(a + pos, a + r * maxlen, sizes[r]);
    pos += sizes[r];
  }
  *all_len = (size_t)total;
  return JITC_OK;
}

// ------------------------------------------------------------ capture (K2 + D2H)
static jitc_status capture_group(jitc_ctx* c, GroupState& g, const GroupSelection& gs, uint64_t v_star,
                                 jitc_stats* stats) {
  auto it = std::find(gs.writers.begin(), gs.writers.end(), c->cfg.rank);
  if (it == gs.writers.end()) return JITC_OK;  // not a writer
  uint64_t s = (uint64_t)(it - gs.writers.begin()), k = gs.writers.size();
  if (!g.has_fp) return fail(JITC_ESTATE, "jitc_capture: group " + std::to_string(g.id) + " not fingerprinted");
  if (gs.layout_hash != g.layout_hash || gs.n_c != g.n_c || gs.image_bytes != g.L)
    return fail(JITC_ELAYOUT, "jitc_capture: selection layout differs from the registered one");
  if (g.fp_version != v_star || g.fp_root != gs.root || g.fp_phase != JITC_PHASE_CLEAN)
    return fail(JITC_ESTATE, "jitc_capture: this rank's fingerprint is not the selected candidate");
  uint64_t c0, c1;
  shard_range(g.n_c, k, s, &c0, &c1);
  uint64_t b0 = std::min(c0 * g.C, g.L), b1 = std::min(c1 * g.C, g.L);
  // the lowest writer invalidates the previous commit before any byte changes
  if (s == 0 && g.img_shm) unlink(gpath(c, g.id, ".commit").c_str());
  g.commit_priv.clear();
  if (b1 > b0) {
    CU(cudaMemsetAsync(g.d_dig2 + c0, 0, (c1 - c0) * 8, c->s_comp));
    const bool zc = (c->cfg.flags & JITC_F_ZERO_COPY_D2H) != 0;
    if (zc) {
      uint32_t lo, hi;
      seg_span(g, b0, b1, &lo, &hi);
      jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, g.img_d, 0), g.d_dig2, b1 - b0);
      if (st) return st;
      if (stats) stats->rounds += 1;
    } else {
      const uint64_t R = c->slot_bytes;
      const int nslots = (int)std::min<uint64_t>(jitc_ctx::kSlots, c->staging_bytes / R);
      uint32_t j = 0;
      for (uint64_t a = b0; a < b1; a += R, ++j) {
        uint64_t b = std::min(a + R, b1);
        int sl = (int)(j % nslots);
        uint8_t* slot = c->staging + sl * R;
        if (j >= (uint32_t)nslots) CU(cudaStreamWaitEvent(c->s_comp, c->ev_free[sl], 0));
        uint32_t lo, hi;
        seg_span(g, a, b, &lo, &hi);
        jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, slot, a), g.d_dig2, b - a);
        if (st) return st;
        CU(cudaEventRecord(c->ev_ready[sl], c->s_comp));
        CU(cudaStreamWaitEvent(c->s_copy, c->ev_ready[sl], 0));
        CU(cudaMemcpyAsync(g.img_h + a, slot, b - a, cudaMemcpyDeviceToHost, c->s_copy));
        CU(cudaEventRecord(c->ev_free[sl], c->s_copy));
      }
      if (stats) stats->rounds += j;
      CU(cudaEventRecord(c->ev_join, c->s_copy));
      CU(cudaStreamWaitEvent(c->s_comp, c->ev_join, 0));
      if (stats) stats->d2h_bytes += b1 - b0;
    }
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2 + c0, (c1 - c0) * 8, cudaMemcpyDeviceToHost, c->s_comp));
  }
  CU(cudaStreamSynchronize(c->s_comp));
  for (uint64_t ch = c0; ch < c1; ++ch)
    if (c->h_dig[ch - c0] != g.fp[ch])
      return fail(JITC_EUNSTABLE, "jitc_capture: group " + std::to_string(g.id) + " chunk " + std::to_string(ch) +
                                      " changed between fingerprint and capture");
  g.captured = true;
  g.cap_v = v_star;
  if (stats) stats->image_bytes += b1 - b0;
  return JITC_OK;
}

jitc_status jitc_capture(jitc_ctx* c, const void* selection, size_t sel_len, uint32_t group, jitc_stats* stats) {
  if (!c) return fail(JITC_EINVAL, "jitc_capture: null ctx");
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
    return fail(JITC_EINVAL, "jitc_capture: " + why);
  if (sel.status != JITC_OK) return fail(sel.status, "jitc_capture: selection status is not OK");
  CU(cudaSetDevice(c->device));
  if (stats) memset(stats, 0, sizeof *stats), stats->first_bad_chunk = -1;
  CallTimer t(c);
  CU(cudaEventRecord(c->ev_t0, c->s_comp));
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held || (group != JITC_ALL_GROUPS && g.id != group)) continue;
    const GroupSelection* gs = sel.find(g.id);
    if (!gs) return fail(JITC_ELAYOUT, "jitc_capture: group missing from selection");
    jitc_status st = capture_group(c, g, *gs, sel.v_star, stats);
    if (st) return st;
  }
  CU(cudaEventRecord(c->ev_t1, c->s_comp));
  CU(cudaEventSynchronize(c->ev_t1));
  finish_stats(c, t, stats, true);
  return JITC_OK;
}

// ------------------------------------------------------------ commit (manifest, then commit record)
static std::vector<uint8_t> build_manifest(const GroupState& g, const GroupSelection& gs, uint64_t v_star) {
  std::vector<uint8_t> b;
  ManifestHdr h{};
  h.magic = kMagicManifest;
  h.fmt = 1;
  h.group = g.id;
  h.n_tensors = (uint32_t)g.t.size();
  h.v_star = v_star;
  h.layout_hash = g.layout_hash;
  h.chunk_bytes = g.C;
  h.n_c = g.n_c;
  h.image_bytes = g.L;
  h.k = (uint32_t)gs.writers.size();
  auto put = [&](const void* p, size_t n) { b.insert(b.end(), (const uint8_t*)p, (const uint8_t*)p + n); };
  auto pad = [&]() { while (b.size() % 8) b.push_back(0); };
  put(&h, sizeof h);
  put(gs.writers.data(), 4 * gs.writers.size());
  pad();
  for (size_t i = 0; i < g.t.size(); ++i) {
    uint16_t ln = (uint16_t)g.names[i].size();
    put(&ln, 2);
    put(g.names[i].data(), ln);
    uint32_t dt = g.t[i].dtype;
    uint64_t nb = g.t[i].nbytes, off = g.off[i];
    put(&dt, 4);
    put(&nb, 8);
    put(&off, 8);
  }
  pad();
  put(g.fp.data(), 8 * g.n_c);
  put(&g.fp_root, 8);
  for (size_t s = 0; s < gs.writers.size(); ++s) {
    ShardEnt e{};
    e.writer = gs.writers[s];
    shard_range(g.n_c, gs.writers.size(), s, &e.c0, &e.c1);
    put(&e, sizeof e);
  }
  uint64_t tr = manifest_trailer(b.data(), b.size());
  put(&tr, 8);
  return b;
}

static jitc_status commit_impl(jitc_ctx* c, const void* selection, size_t sel_len, bool collective) {
  if (!c) return fail(JITC_EINVAL, "jitc_commit: null ctx");
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
    return fail(JITC_EINVAL, "jitc_commit: " + why);
  if (sel.status != JITC_OK) return fail(sel.status, "jitc_commit: selection status is not OK");
  CU(cudaSetDevice(c->device));
  jitc_status st = collective ? barrier(c) : JITC_OK;  // every writer's capture has returned
  if (st) return st;
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held) continue;
    const GroupSelection* gs = sel.find(g.id);
    if (!gs || gs->writers.empty()) continue;
    bool writer = std::find(gs->writers.begin(), gs->writers.end(), c->cfg.rank) != gs->writers.end();
    if (!writer) continue;
    if (!g.captured || g.cap_v != sel.v_star) return fail(JITC_ESTATE, "jitc_commit: group not captured at v*");
    std::vector<uint8_t> man = build_manifest(g, *gs, sel.v_star);
    CommitRec cr{};
    cr.magic = kMagicCommit;
    cr.group = g.id;
    cr.v_star = sel.v_star;
    memcpy(&cr.trailer, man.data() + man.size() - 8, 8);
    cr.manifest_bytes = man.size();
    g.man_d = g.fp;
    g.man_root = g.fp_root;
    g.has_man = true;
    g.man_priv = man;
    g.commit_priv.assign((uint8_t*)&cr, (uint8_t*)&cr + sizeof cr);
    if (g.img_shm && gs->writers[0] == c->cfg.rank) {
      if (!write_file_atomic(gpath(c, g.id, ".manifest"), man.data(), man.size()))
        return fail(JITC_EIO, "jitc_commit: writing manifest: " + std::string(strerror(errno)));
      if (!write_file_atomic(gpath(c, g.id, ".commit"), (const uint8_t*)&cr, sizeof cr))
        return fail(JITC_EIO, "jitc_commit: writing commit record: " + std::string(strerror(errno)));
    }
  }
  return collective ? barrier(c) : JITC_OK;  // nobody restores before every commit record exists
}

jitc_status jitc_commit(jitc_ctx* c, const void* selection, size_t sel_len) {
  return commit_impl(c, selection, sel_len, true);
}

// ------------------------------------------------------------ restore
struct ManifestView {
  ManifestHdr h;
  std::vector<int32_t> writers;
  std::vector<uint64_t> d;
  uint64_t root = 0;
};

static jitc_status load_manifest(jitc_ctx* c, GroupState& g, ManifestView* mv) {
  std::vector<uint8_t> man, com;
  if (g.img_shm) {
    if (!read_file(gpath(c, g.id, ".commit"), &com) || !read_file(gpath(c, g.id, ".manifest"), &man))
      return fail(JITC_EINCOMPLETE, "jitc_restore: group " + std::to_string(g.id) + " has no committed checkpoint");
  } else {
    man = g.man_priv;
    com = g.commit_priv;
  }
  if (com.size() != sizeof(CommitRec) || man.size() < sizeof(ManifestHdr) + 16)
    return fail(JITC_EINCOMPLETE, "jitc_restore: missing or torn manifest / commit record");
  CommitRec cr;
  memcpy(&cr, com.data(), sizeof cr);
  uint64_t tr_stored;
  memcpy(&tr_stored, man.data() + man.size() - 8, 8);
  if (cr.magic != kMagicCommit || cr.manifest_bytes != man.size() || cr.trailer != tr_stored ||
      manifest_trailer(man.data(), man.size() - 8) != tr_stored || cr.group != g.id)
    return fail(JITC_EINCOMPLETE, "jitc_restore: commit record does not match the manifest");
  memcpy(&mv->h, man.data(), sizeof(ManifestHdr));
  const ManifestHdr& h = mv->h;
  if (h.magic != kMagicManifest || h.layout_hash != g.layout_hash || h.n_c != g.n_c || h.image_bytes != g.L ||
      h.chunk_bytes != g.C || h.v_star != cr.v_star)
    return fail(JITC_ELAYOUT, "jitc_restore: manifest layout differs from the registered tensors");
  size_t q = sizeof(ManifestHdr);
  mv->writers.resize(h.k);
  memcpy(mv->writers.data(), man.data() + q, 4ull * h.k);
  q = align_up(q + 4ull * h.k, 8);
  size_t t0 = q;
  for (uint32_t i = 0; i < h.n_tensors; ++i) {
    uint16_t ln;
    memcpy(&ln, man.data() + q, 2);
    q += 2 + ln + 20;
  }
  q = t0 + align_up(q - t0, 8);
  if (q + 8 * (h.n_c + 1) > man.size()) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  mv->d.resize(h.n_c);
  memcpy(mv->d.data(), man.data() + q, 8 * h.n_c);
  memcpy(&mv->root, man.data() + q + 8 * h.n_c, 8);
  if (root_of(h.layout_hash, mv->d.data(), h.n_c) != mv->root)
    return fail(JITC_EINCOMPLETE, "jitc_restore: manifest digests do not chain to its root");
  return JITC_OK;
}

static jitc_status compare_digests(jitc_ctx* c, GroupState& g, const std::vector<uint64_t>& want, jitc_stats* stats) {
  if (g.n_c) {
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
  }
  for (uint64_t ch = 0; ch < g.n_c; ++ch)
    if (c->h_dig[ch] != want[ch]) {
      if (stats) stats->first_bad_chunk = (int32_t)ch;
      return fail(JITC_ECORRUPT, "jitc_restore: group " + std::to_string(g.id) + " chunk " + std::to_string(ch) +
                                     " does not match the checkpoint digest");
    }
  return JITC_OK;
}

// Executes a restore plan (jitc_plan.cc) round by round: H2D on the copy
// stream; K2 packs, NCCL send/recv or all-gather and K3 unpacks on the
// compute stream; slot reuse ordered by the ready/free events.
static jitc_status execute_plan(jitc_ctx* c, GroupState& g, const std::vector<PlanOp>& ops, uint32_t S,
                                jitc_stats* stats) {
  if (S > (uint32_t)jitc_ctx::kSlots) return fail(JITC_EINVAL, "execute_plan: too many slots");
  bool used[jitc_ctx::kSlots] = {false};
  size_t i = 0;
  uint32_t rounds = 0;
  while (i < ops.size()) {
    if (ops[i].kind == kOpDigestSend || ops[i].kind == kOpDigestRecv) {
      ++i;
      continue;
    }
    const uint32_t j = ops[i].round;
    size_t e = i;
    while (e < ops.size() && ops[e].round == j && ops[e].kind != kOpDigestSend && ops[e].kind != kOpDigestRecv) ++e;
    const uint32_t sl = ops[i].slot;
    ++rounds;
    // 1. host -> device on the copy stream
    bool any_h2d = false;
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpH2D) continue;
      if (!any_h2d && used[sl]) CU(cudaStreamWaitEvent(c->s_copy, c->ev_free[sl], 0));
      any_h2d = true;
      CU(cudaMemcpyAsync(c->staging + op.off, g.img_h + op.a, op.bytes, cudaMemcpyHostToDevice, c->s_copy));
      if (stats) stats->h2d_bytes += op.bytes;
    }
    if (any_h2d) {
      CU(cudaEventRecord(c->ev_ready[sl], c->s_copy));
      CU(cudaStreamWaitEvent(c->s_comp, c->ev_ready[sl], 0));
    }
    // 2. K2 packs (PEER writers)
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpPack) continue;
      uint32_t lo, hi;
      seg_span(g, op.a, op.b, &lo, &hi);
      jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, c->staging + op.off, op.a), g.d_dig2, op.b - op.a);
      if (st) return st;
    }
    // 3. NCCL: point-to-point (PEER) and all-gather (HOST, n > 1)
    bool p2p = false;
    for (size_t q = i; q < e; ++q) p2p |= ops[q].kind == kOpSend || ops[q].kind == kOpRecv;
    if (p2p) {
      NC(ncclGroupStart());
      for (size_t q = i; q < e; ++q) {
        const PlanOp& op = ops[q];
        if (op.kind == kOpSend) NC(ncclSend(c->staging + op.off, op.bytes, ncclUint8, op.peer, c->comm, c->s_comp));
        if (op.kind == kOpRecv) NC(ncclRecv(c->staging + op.off, op.bytes, ncclUint8, op.peer, c->comm, c->s_comp));
        if (stats) stats->p2p_bytes += op.bytes;
      }
      NC(ncclGroupEnd());
    }
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpAllGather) continue;
      uint8_t* base = c->staging + op.off;
      NC(ncclAllGather(base + (uint64_t)c->comm_rank * op.bytes, base, op.bytes, ncclUint8, c->comm, c->s_comp));
      if (stats) stats->p2p_bytes += (uint64_t)(c->comm_n - 1) * op.bytes;
    }
    // 4. K3 unpack + verify of every block of the round (<= kMaxRanges per launch)
    LaunchRanges lr{};
    uint64_t bytes = 0;
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpUnpack) continue;
      uint32_t lo, hi;
      seg_span(g, op.a, op.b, &lo, &hi);
      add_range(lr, lo, hi, c->staging + op.off, op.a);
      bytes += op.b - op.a;
      if (lr.n == kMaxRanges) {
        jitc_status st = run_segments(c, g, kUnpack, lr, g.d_dig2, bytes);
        if (st) return st;
        lr = LaunchRanges{};
        bytes = 0;
      }
    }
    if (lr.n) {
      jitc_status st = run_segments(c, g, kUnpack, lr, g.d_dig2, bytes);
      if (st) return st;
    }
    CU(cudaEventRecord(c->ev_free[sl], c->s_comp));
    used[sl] = true;
    i = e;
  }
  if (stats) stats->rounds += rounds;
  return JITC_OK;
}

static jitc_status make_plan(jitc_ctx* c, const PlanInput& in, std::vector<PlanOp>* ops, uint32_t* S) {
  uint64_t R;
  std::string why;
  if (!build_restore_plan(in, ops, &R, S, &why)) return fail(JITC_ENOMEM, "jitc_restore: " + why);
  return JITC_OK;
}

// HOST mode: this rank (or, with a communicator, every comm rank) loads a
// 1/n slice of the committed image H2D; slices are all-gathered over NVLink
// round by round and every round is unpacked+verified by K3.
static jitc_status restore_host(jitc_ctx* c, GroupState& g, jitc_stats* stats) {
  ManifestView mv;
  jitc_status st = load_manifest(c, g, &mv);
  if (st) return st;
  if (g.n_c) CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
  const int n = c->comm ? c->comm_n : 1;
  if (n > 1 && !g.img_shm)
    return fail(JITC_EINVAL, "jitc_restore: HOST mode across ranks needs a shared image_dir (use PEER mode)");
  if (n == 1 && (c->cfg.flags & JITC_F_ZERO_COPY_H2D)) {
    st = run_segments(c, g, kUnpack, one_range(0, (uint32_t)g.segs.size(), g.img_d, 0), g.d_dig2, g.L);
    if (st) return st;
    if (stats) stats->rounds += 1, stats->h2d_bytes += g.L;
  } else {
    PlanInput in;
    in.mode = JITC_RESTORE_HOST;
    in.n_c = g.n_c;
    in.chunk_bytes = g.C;
    in.image_bytes = g.L;
    in.n = n;
    in.me = c->comm ? c->comm_rank : 0;
    in.staging_bytes = c->staging_bytes;
    in.slot_bytes = c->slot_bytes;
    if (c->comm) {
      for (int32_t m : g.members) {
        int r = comm_rank_of(c, m);
        if (r >= 0) in.participants.push_back(r);
      }
      std::sort(in.participants.begin(), in.participants.end());
    } else {
      in.participants = {0};
    }
    std::vector<PlanOp> ops;
    uint32_t S = 0;
    st = make_plan(c, in, &ops, &S);
    if (st) return st;
    st = execute_plan(c, g, ops, S, stats);
    if (st) return st;
  }
  st = compare_digests(c, g, mv.d, stats);
  if (st) return st;
  g.man_d = mv.d;
  g.man_root = mv.root;
  g.has_man = true;
  if (stats) stats->image_bytes += g.L;
  return JITC_OK;
}

// PEER mode: the selection's writers pack their O5 ranges from live HBM (K2)
// and send them over NVLink to every member that is not a writer; receivers
// unpack+verify (K3) against the writers' digests (broadcast first).
static jitc_status restore_peer(jitc_ctx* c, GroupState& g, const GroupSelection& gs, jitc_stats* stats) {
  if (!c->comm) return fail(JITC_ESTATE, "jitc_restore: PEER mode needs a communicator");
  if (gs.writers.empty()) return JITC_OK;  // dropped OPTIONAL group
  if (gs.layout_hash != g.layout_hash || gs.n_c != g.n_c || gs.image_bytes != g.L)
    return fail(JITC_ELAYOUT, "jitc_restore: selection layout differs from the registered one");
  PlanInput in;
  in.mode = JITC_RESTORE_PEER;
  in.n_c = g.n_c;
  in.chunk_bytes = g.C;
  in.image_bytes = g.L;
  in.n = c->comm_n;
  in.me = c->comm_rank;
  in.staging_bytes = c->staging_bytes;
  in.slot_bytes = c->slot_bytes;
  for (int32_t w : gs.writers) {
    int r = comm_rank_of(c, w);
    if (r < 0) return fail(JITC_EINVAL, "jitc_restore: a writer is not in the communicator");
    in.writers.push_back(r);
  }
  for (int32_t m : gs.members) {
    if (std::find(gs.writers.begin(), gs.writers.end(), m) != gs.writers.end()) continue;
    int r = comm_rank_of(c, m);
    if (r >= 0) in.dests.push_back(r);
  }
  const int my_s = (int)(std::find(in.writers.begin(), in.writers.end(), in.me) - in.writers.begin());
  const bool is_writer = my_s < (int)in.writers.size();
  const bool is_dst = std::find(in.dests.begin(), in.dests.end(), in.me) != in.dests.end();
  std::vector<PlanOp> ops;
  uint32_t S = 0;
  jitc_status st = make_plan(c, in, &ops, &S);
  if (st) return st;
  if (!is_writer && !is_dst) return JITC_OK;
  // 1. the lowest writer sends the selected class's digests to every destination
  uint64_t* d_expect = g.d_dig;
  if (is_writer && (!g.has_fp || g.fp_root != gs.root))
    return fail(JITC_ESTATE, "jitc_restore: writer fingerprint differs from the selected class");
  if (is_writer && my_s == 0 && g.n_c)
    CU(cudaMemcpyAsync(d_expect, g.fp.data(), g.n_c * 8, cudaMemcpyHostToDevice, c->s_comp));
  bool any = false;
  for (const PlanOp& op : ops) any |= op.kind == kOpDigestSend || op.kind == kOpDigestRecv;
  if (any && g.n_c) {
    NC(ncclGroupStart());
    for (const PlanOp& op : ops) {
      if (op.kind == kOpDigestSend) NC(ncclSend(d_expect, g.n_c, ncclUint64, op.peer, c->comm, c->s_comp));
      if (op.kind == kOpDigestRecv) NC(ncclRecv(d_expect, g.n_c, ncclUint64, op.peer, c->comm, c->s_comp));
    }
    NC(ncclGroupEnd());
  }
  std::vector<uint64_t> want(g.n_c);
  if (is_dst) {
    if (g.n_c) CU(cudaMemcpyAsync(want.data(), d_expect, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
    if (root_of(g.layout_hash, want.data(), g.n_c) != gs.root)
      return fail(JITC_ECORRUPT, "jitc_restore: received digests do not chain to the selected root");
  } else {
    want = g.fp;
  }
  if (g.n_c) CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
  // 2. data rounds
  st = execute_plan(c, g, ops, S, stats);
  if (st) return st;
  CU(cudaStreamSynchronize(c->s_comp));
  if (is_dst) {
    st = compare_digests(c, g, want, stats);
    if (st) return st;
    g.man_d = want;
    g.man_root = gs.root;
    g.has_man = true;
    if (stats) stats->image_bytes += g.L;
  } else if (g.n_c) {  // the writer's re-digest of its own range must still match
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
    uint64_t c0, c1;
    shard_range(g.n_c, in.writers.size(), my_s, &c0, &c1);
    for (uint64_t ch = c0; ch < c1; ++ch)
      if (c->h_dig[ch] != want[ch]) return fail(JITC_EUNSTABLE, "jitc_restore: writer state changed");
  }
  return JITC_OK;
}

jitc_status jitc_restore(jitc_ctx* c, uint32_t group, int32_t mode, const void* selection, size_t sel_len,
                         jitc_stats* stats) {
  if (!c) return fail(JITC_EINVAL, "jitc_restore: null ctx");
  if (mode != JITC_RESTORE_HOST && mode != JITC_RESTORE_PEER) return fail(JITC_EINVAL, "jitc_restore: bad mode");
  Selection sel;
  bool have_sel = false;
  if (selection) {
    std::string why;
    if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
      return fail(JITC_EINVAL, "jitc_restore: " + why);
    if (sel.status != JITC_OK) return fail(sel.status, "jitc_restore: selection status is not OK");
    have_sel = true;
  } else if (mode == JITC_RESTORE_PEER) {
    return fail(JITC_EINVAL, "jitc_restore: PEER mode needs the selection");
  }
  CU(cudaSetDevice(c->device));
  if (stats) memset(stats, 0, sizeof *stats), stats->first_bad_chunk = -1;
  CallTimer t(c);
  CU(cudaEventRecord(c->ev_t0, c->s_comp));
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held || (group != JITC_ALL_GROUPS && g.id != group)) continue;
    const GroupSelection* gs = have_sel ? sel.find(g.id) : nullptr;
    if (have_sel && !gs) return fail(JITC_ELAYOUT, "jitc_restore: group missing from selection");
    if (gs && gs->writers.empty()) continue;  // dropped OPTIONAL group: nothing to restore
    jitc_status st = mode == JITC_RESTORE_HOST ? restore_host(c, g, stats) : restore_peer(c, g, *gs, stats);
    if (st) {
      harvest(c);
      return st;
    }
  }
  CU(cudaEventRecord(c->ev_t1, c->s_comp));
  CU(cudaEventSynchronize(c->ev_t1));
  finish_stats(c, t, stats, true);
  return JITC_OK;
}

// ------------------------------------------------------------ verify (A12)
jitc_status jitc_verify(jitc_ctx* c, uint32_t group, const void* expected, size_t len, uint64_t* first_bad) {
  if (!c) return fail(JITC_EINVAL, "jitc_verify: null ctx");
  if (first_bad) *first_bad = UINT64_MAX;
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_verify: group not registered");
  GroupState& g = it->second;
  std::vector<uint64_t> want;
  if (expected) {
    std::vector<BlobView> bv;
    std::string why;
    if (!parse_blobs(static_cast<const uint8_t*>(expected), len, &bv, &why)) return fail(JITC_EINVAL, "jitc_verify: " + why);
    const RecordView* rv = nullptr;
    for (auto& b : bv)
      for (auto& r : b.recs)
        if (r.h.group == group && !rv) rv = &r;
    if (!rv) return fail(JITC_EINVAL, "jitc_verify: expected blob has no record of the group");
    if (rv->h.layout_hash != g.layout_hash || rv->h.n_c != g.n_c) return fail(JITC_ELAYOUT, "jitc_verify: layout differs");
    want.assign(rv->d, rv->d + rv->h.n_c);
  } else {
    if (!g.has_man) return fail(JITC_ESTATE, "jitc_verify: no manifest (restore or commit first)");
    want = g.man_d;
  }
  CU(cudaSetDevice(c->device));
  CallTimer t(c);
  if (g.n_c) {
    CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
    jitc_status st = run_segments(c, g, kDigest, one_range(0, (uint32_t)g.segs.size(), nullptr, 0), g.d_dig2, g.L);
    if (st) return st;
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
  }
  CU(cudaStreamSynchronize(c->s_comp));
  harvest(c);
  for (uint64_t ch = 0; ch < g.n_c; ++ch)
    if (c->h_dig[ch] != want[ch]) {
      if (first_bad) *first_bad = ch;
      return fail(JITC_ECORRUPT, "jitc_verify: chunk " + std::to_string(ch) + " differs");
    }
  return JITC_OK;
}

// ------------------------------------------------------------ durable tier (NEXT-4)
// PAPER.md:341, :356 §6.3: JIT and low-frequency periodic checkpoints share
// code and file format; a catastrophic multi-node failure needs a persistent
// copy.  jitc_persist streams a committed host image to a directory on disk
// with parallel O_DIRECT writes (64 MiB pieces), then writes the manifest and,
// LAST, the commit record; jitc_stage_in reads such a copy back
// into the host image (checking the commit record and the layout) so that
// jitc_restore's K3 verification covers it end to end.
static bool rw_parallel(int fd, uint8_t* buf, uint64_t n, bool write, int threads) {
  const uint64_t piece = 64ull << 20;
  std::vector<std::thread> th;
  std::vector<int> ok(threads, 1);
  for (int t = 0; t < threads; ++t)
    th.emplace_back([&, t] {
      for (uint64_t off = (uint64_t)t * piece; off < n; off += (uint64_t)threads * piece) {
        uint64_t len = std::min(piece, n - off), done = 0;
        while (done < len) {
          ssize_t r = write ? pwrite(fd, buf + off + done, len - done, (off_t)(off + done))
                            : pread(fd, buf + off + done, len - done, (off_t)(off + done));
          if (r <= 0) {
            if (r < 0 && errno == EINTR) continue;
            ok[t] = 0;
            return;
          }
          done += (uint64_t)r;
        }
      }
    });
  for (auto& x : th) x.join();
  for (int v : ok)
    if (!v) return false;
  return true;
}

static int open_maybe_direct(const std::string& path, int flags) {
  int fd = open(path.c_str(), flags | O_DIRECT, 0600);
  if (fd < 0 && errno == EINVAL) fd = open(path.c_str(), flags, 0600);  // e.g. tmpfs has no O_DIRECT
  return fd;
}

static void fsync_dir(const std::string& dir) {
  int fd = open(dir.c_str(), O_RDONLY | O_DIRECTORY);
  if (fd >= 0) {
    fsync(fd);
    close(fd);
  }
}

jitc_status jitc_persist(jitc_ctx* c, uint32_t group, const char* dir, jitc_stats* stats) {
  if (!c || !dir) return fail(JITC_EINVAL, "jitc_persist: null argument");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_persist: group not registered");
  GroupState& g = it->second;
  CallTimer t(c);
  std::vector<uint8_t> man, com;
  if (g.img_shm) {
    if (!read_file(gpath(c, g.id, ".commit"), &com) || !read_file(gpath(c, g.id, ".manifest"), &man))
      return fail(JITC_EINCOMPLETE, "jitc_persist: group has no committed checkpoint");
  } else {
    man = g.man_priv;
    com = g.commit_priv;
  }
  if (com.size() != sizeof(CommitRec) || man.size() < 16) return fail(JITC_EINCOMPLETE, "jitc_persist: not committed");
  std::string d(dir);
  mkdir(d.c_str(), 0700);
  std::string base = d + "/g" + std::to_string(g.id);
  unlink((base + ".commit").c_str());  // an older durable copy stops being valid first
  int fd = open_maybe_direct(base + ".img.tmp", O_WRONLY | O_CREAT | O_TRUNC);
  if (fd < 0) return fail(JITC_EIO, "jitc_persist: open " + base + ".img.tmp: " + strerror(errno));
  bool ok = rw_parallel(fd, g.img_h, g.img_bytes, true, 8) && fdatasync(fd) == 0;
  close(fd);
  if (!ok || rename((base + ".img.tmp").c_str(), (base + ".img").c_str()) != 0)
    return fail(JITC_EIO, "jitc_persist: writing image: " + std::string(strerror(errno)));
  if (!write_file_atomic(base + ".manifest", man.data(), man.size()) ||
      !write_file_atomic(base + ".commit", com.data(), com.size()))
    return fail(JITC_EIO, "jitc_persist: writing manifest / commit record: " + std::string(strerror(errno)));
  fsync_dir(d);
  if (stats) {
    memset(stats, 0, sizeof *stats);
    stats->first_bad_chunk = -1;
    stats->image_bytes = g.img_bytes;
    stats->ms_host = now_ms() - t.t0;
  }
  return JITC_OK;
}

jitc_status jitc_stage_in(jitc_ctx* c, uint32_t group, const char* dir, jitc_stats* stats) {
  if (!c || !dir) return fail(JITC_EINVAL, "jitc_stage_in: null argument");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_stage_in: group not registered");
  GroupState& g = it->second;
  CallTimer t(c);
  std::string base = std::string(dir) + "/g" + std::to_string(g.id);
  std::vector<uint8_t> man, com;
  if (!read_file(base + ".commit", &com) || !read_file(base + ".manifest", &man))
    return fail(JITC_EINCOMPLETE, "jitc_stage_in: no committed durable copy in " + std::string(dir));
  CommitRec cr;
  if (com.size() != sizeof cr || man.size() < sizeof(ManifestHdr) + 16)
    return fail(JITC_EINCOMPLETE, "jitc_stage_in: torn manifest / commit record");
  memcpy(&cr, com.data(), sizeof cr);
  uint64_t tr;
  memcpy(&tr, man.data() + man.size() - 8, 8);
  if (cr.magic != kMagicCommit || cr.manifest_bytes != man.size() || cr.trailer != tr ||
      manifest_trailer(man.data(), man.size() - 8) != tr)
    return fail(JITC_EINCOMPLETE, "jitc_stage_in: commit record does not match the manifest");
  ManifestHdr h;
  memcpy(&h, man.data(), sizeof h);
  if (h.layout_hash != g.layout_hash || h.image_bytes != g.L || h.n_c != g.n_c)
    return fail(JITC_ELAYOUT, "jitc_stage_in: durable copy has a different layout");
  if (g.img_shm) unlink(gpath(c, g.id, ".commit").c_str());  // the host image is about to change
  g.commit_priv.clear();
  int fd = open_maybe_direct(base + ".img", O_RDONLY);
  if (fd < 0) return fail(JITC_EIO, "jitc_stage_in: open " + base + ".img: " + strerror(errno));
  bool ok = rw_parallel(fd, g.img_h, g.img_bytes, false, 8);
  close(fd);
  if (!ok) return fail(JITC_EIO, "jitc_stage_in: reading image: " + std::string(strerror(errno)));
  g.man_priv = man;
  g.commit_priv = com;
  if (g.img_shm && (!write_file_atomic(gpath(c, g.id, ".manifest"), man.data(), man.size()) ||
                    !write_file_atomic(gpath(c, g.id, ".commit"), com.data(), com.size())))
    return fail(JITC_EIO, "jitc_stage_in: installing manifest / commit record");
  if (stats) {
    memset(stats, 0, sizeof *stats);
    stats->first_bad_chunk = -1;
    stats->image_bytes = g.img_bytes;
    stats->ms_host = now_ms() - t.t0;
  }
  return JITC_OK;
}

// ------------------------------------------------------------ watchdog (NEXT-1)
// PAPER.md:124-126 §3.1: events recorded after collectives are put on a
// watch-list; a watchdog thread polls them with cudaEventQuery and treats
// one that stays incomplete past a timeout as a hang of the collective.
// PAPER.md:132-134 §3.2: the checkpoint is then taken on a side stream by the
// watchdog thread itself -- here entirely in C++ (no Python callback, so the
// GIL cannot block it) on the library's non-blocking streams.
static jitc_status local_capture(jitc_ctx* c, jitc_stats* st) {
  size_t len = 0;
  jitc_status r = jitc_fingerprint(c, JITC_ALL_GROUPS, nullptr, 0, &len);
  if (r) return r;
  std::vector<uint8_t> blob(len);
  r = jitc_fingerprint(c, JITC_ALL_GROUPS, blob.data(), blob.size(), &len);
  if (r) return r;
  int32_t me = c->cfg.rank;
  size_t sl = 0;
  jitc_select_consistent_replica(blob.data(), len, &me, 1, nullptr, 0, &sl);
  std::vector<uint8_t> sel(sl);
  r = jitc_select_consistent_replica(blob.data(), len, &me, 1, sel.data(), sel.size(), &sl);
  if (r) return r;
  r = jitc_capture(c, sel.data(), sl, JITC_ALL_GROUPS, st);
  if (r) return r;
  return commit_impl(c, sel.data(), sl, false);
}

static void watchdog_loop(jitc_ctx* c) {
  cudaSetDevice(c->device);
  const double t0 = now_ms();
  for (;;) {
    std::unique_lock<std::mutex> lk(c->wmu);
    if (!c->wrun) return;
    double now = now_ms();
    bool hang = false;
    for (size_t i = 0; i < c->watches.size();) {
      cudaError_t q = cudaEventQuery(c->watches[i].ev);
      if (q == cudaSuccess) {
        c->watches.erase(c->watches.begin() + i);
        continue;
      }
      if (q != cudaErrorNotReady) cudaGetLastError();
      if (now - c->watches[i].t_added >= c->timeout_ms) {
        hang = true;
        c->fired_tag = c->watches[i].tag;
        c->waited_ms = now - c->watches[i].t_added;
        break;
      }
      ++i;
    }
    if (hang) {
      c->fired = true;
      c->detect_ms = now - t0;
      lk.unlock();
      double ta = now_ms();
      if (c->action == JITC_ON_HANG_LOCAL_CAPTURE) {
        jitc_stats st{};
        jitc_status r = local_capture(c, &st);
        lk.lock();
        c->action_status = r;
        c->action_stats = st;
        lk.unlock();
      }
      if (c->hang_fn) c->hang_fn(c->hang_user, c->fired_tag, c->waited_ms);
      lk.lock();
      c->action_ms = now_ms() - ta;
      c->action_done = true;
      c->wrun = false;
      c->wcv.notify_all();
      return;
    }
    c->wcv.wait_for(lk, std::chrono::microseconds(200));
  }
}

static void stop_thread(jitc_ctx* c) {
  {
    std::lock_guard<std::mutex> lk(c->wmu);
    c->wrun = false;
    c->wcv.notify_all();
  }
  if (c->wthread.joinable()) c->wthread.join();
}

jitc_status jitc_capture_local(jitc_ctx* c, jitc_stats* stats) {
  if (!c) return fail(JITC_EINVAL, "jitc_capture_local: null ctx");
  jitc_stats st{};
  st.first_bad_chunk = -1;
  jitc_status r = local_capture(c, &st);
  if (stats) *stats = st;
  return r;
}

jitc_status jitc_watch_event(jitc_ctx* c, void* event, uint64_t tag) {
  if (!c || !event) return fail(JITC_EINVAL, "jitc_watch_event: null argument");
  std::lock_guard<std::mutex> lk(c->wmu);
  c->watches.push_back({(cudaEvent_t)event, tag, now_ms()});
  return JITC_OK;
}

jitc_status jitc_watchdog_start(jitc_ctx* c, uint32_t timeout_ms, int32_t action, jitc_hang_fn fn, void* user) {
  if (!c) return fail(JITC_EINVAL, "jitc_watchdog_start: null ctx");
  if (action != JITC_ON_HANG_NOTIFY && action != JITC_ON_HANG_LOCAL_CAPTURE)
    return fail(JITC_EINVAL, "jitc_watchdog_start: bad action");
  stop_thread(c);  // a previous watchdog; the watch-list is kept
  std::lock_guard<std::mutex> lk(c->wmu);
  c->timeout_ms = timeout_ms;
  c->action = action;
  c->hang_fn = fn;
  c->hang_user = user;
  c->fired = c->action_done = false;
  c->action_status = JITC_OK;
  c->action_stats = jitc_stats{};
  c->action_stats.first_bad_chunk = -1;
  c->wrun = true;
  c->wthread = std::thread(watchdog_loop, c);
  return JITC_OK;
}

jitc_status jitc_watchdog_wait(jitc_ctx* c, uint32_t max_ms, int32_t* fired, uint64_t* tag, double* waited_ms,
                               double* action_ms, jitc_stats* action_stats) {
  if (!c || !fired) return fail(JITC_EINVAL, "jitc_watchdog_wait: null argument");
  std::unique_lock<std::mutex> lk(c->wmu);
  c->wcv.wait_for(lk, std::chrono::milliseconds(max_ms), [c] { return c->action_done; });
  *fired = c->action_done ? 1 : 0;
  if (tag) *tag = c->fired_tag;
  if (waited_ms) *waited_ms = c->waited_ms;
  if (action_ms) *action_ms = c->action_ms;
  if (action_stats) *action_stats = c->action_stats;
  jitc_status st = c->action_done ? c->action_status : JITC_OK;
  if (st) set_error("jitc_watchdog_wait: the on-hang capture failed with status " + std::to_string(st));
  return st;
}

jitc_status jitc_watchdog_stop(jitc_ctx* c) {
  if (!c) return fail(JITC_EINVAL, "jitc_watchdog_stop: null ctx");
  stop_thread(c);
  std::lock_guard<std::mutex> lk(c->wmu);
  c->watches.clear();
  return JITC_OK;
}

// ------------------------------------------------------------ counters
jitc_status jitc_kernel_counters(jitc_ctx* c, int32_t kind, jitc_kernel_counter* out) {
  if (!c || !out || kind < 1 || kind > 3) return fail(JITC_EINVAL, "jitc_kernel_counters: bad argument");
  *out = c->kc[kind];
  return JITC_OK;
}

jitc_status jitc_reset_counters(jitc_ctx* c) {
  if (!c) return fail(JITC_EINVAL, "jitc_reset_counters: null ctx");
  for (auto& k : c->kc) k = jitc_kernel_counter{};
  return JITC_OK;
}

}  // extern "C"
