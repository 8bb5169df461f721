// Internal definitions shared by the libjitc.so context sources
// (jitc_ctx.cc, jitc_capture.cc, jitc_restore.cc, jitc_durable.cc,
// jitc_watchdog.cc): the context and group state, and small helpers.
#pragma once

#include <cuda.h>
#include <errno.h>
#include <fcntl.h>
#include <nccl.h>
#include <stdio.h>
#include <string.h>
#include <sys/file.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <sys/syscall.h>
#include <ctype.h>
#include <sys/types.h>
#include <unistd.h>

#include <algorithm>
#include <functional>
#include <chrono>
#include <atomic>
#include <condition_variable>
#include <mutex>
#include <thread>
#include <map>
#include <memory>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "jitc_internal.h"


namespace jitc {

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
  std::vector<uint32_t> seg_tensor;  // tensor index of every segment
  Seg* d_segs = nullptr;
  uint64_t* d_remote = nullptr;      // K5: per-segment peer source address
  std::vector<uint64_t> h_remote;
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
  std::vector<uint8_t> man_aux;  // the user's CPU state carried by the manifest
  // host image
  uint8_t* img_h = nullptr;
  uint8_t* img_d = nullptr;  // device alias of the mapped host image
  size_t img_bytes = 0;
  bool img_shm = false;
  // a shared image is pinned as separate registrations of img_reg_piece bytes
  // each (0: one registration); a host<->device copy must not cross one
  uint64_t img_reg_piece = 0;
  int img_numa_slices = 0;  // slices given a NUMA policy when this rank created the image
  std::vector<uint8_t*> img_regs;
  std::string img_path;
  std::vector<uint8_t> man_priv, commit_priv;  // private-memory manifest / commit
};

typedef CUresult (*PFN_writeValue64)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);

// ------------------------------------------------------------- IPC transport
// Intra-node alternative to NCCL (jitc_ipc.cc): ranks share a control block
// in a /dev/shm file and map each other's staging buffers with CUDA IPC.
// Progress counters are written by the GPU in stream order
// (cuStreamWriteValue64 into the mapped control block) and polled by the
// peers' host threads; K3 reads a peer's block straight from its staging
// (peer memory over NVLink), so the exchange is fused into the unpack.
constexpr int kIpcMaxRanks = 64;
// Default copy-engine piece: 64 MiB pieces D2H at 55.6 GB/s vs 53.7 for one 2 GiB
// copy per round (C2 capture 448 vs 464 ms, same box; profiles/r01_copy_piece.txt).
constexpr uint64_t kDefaultCopyPiece = 64ull << 20;
constexpr int kIpcMaxGroups = 64;
struct IpcCtl {
  uint64_t arrive[kIpcMaxRanks];                  // barrier generations
  uint64_t posted[kIpcMaxRanks][kIpcMaxGroups];   // rounds whose outgoing block is ready
  uint64_t consumed[kIpcMaxRanks][kIpcMaxGroups]; // rounds whose incoming blocks were read
  cudaIpcMemHandle_t staging[kIpcMaxRanks];
  uint64_t staging_off[kIpcMaxRanks];
  uint64_t published[kIpcMaxRanks];
  uint64_t heartbeat[kIpcMaxRanks];  // CLOCK_MONOTONIC microseconds, refreshed every 10 ms while alive
  // capture fan-out rounds: (call generation << 24) | (round + 1)
  uint64_t cap_posted[kIpcMaxRanks][kIpcMaxGroups];
  uint64_t cap_consumed[kIpcMaxRanks][kIpcMaxGroups];
  // status agreement (jitc::agree): (generation << 16) | -status, two slots by
  // generation parity -- a rank can be at most one barrier generation ahead
  uint64_t agree[2][kIpcMaxRanks];
};
struct IpcComm {
  std::string dir;
  IpcCtl* ctl = nullptr;      // host mapping of dir/ctl
  uint8_t* ctl_dev = nullptr; // device alias (cudaHostRegister mapped)
  size_t ctl_bytes = 0;
  std::vector<int> slot;               // comm rank -> index into the IpcCtl arrays (stable across shrink)
  std::vector<uint8_t*> peer_staging;  // by comm rank (own entry = ctx staging)
  std::vector<void*> opened;
  uint64_t barrier_gen = 0, exchange_gen = 0, cap_gen = 0, agree_gen = 0;
  // restore calls per group slot.  Every participant of a group's restore
  // advances it once per call, before anything can fail, so a call that
  // aborts part-way (JITC_EPEER, a timeout) leaves every survivor on the same
  // generation; the round counters of call `gen` are (gen << 24) | (round + 1),
  // so stale counter values of an aborted call never satisfy a later wait.
  std::map<uint32_t, uint64_t> restore_gen;
  std::thread hb_thread;                    // heartbeat writer (failure localisation, NEXT-1)
  std::atomic<bool> hb_run{false};
  double dead_ms = 2000.0;                  // a peer whose heartbeat is older is dead (JITC_PEER_DEAD_MS)
};

// Liveness table for the NCCL transport (NEXT-1 failure localisation; the
// IPC transport keeps its heartbeats in IpcCtl): one CLOCK_MONOTONIC
// heartbeat per JOB rank in a small file on /dev/shm shared by the ranks of
// one box, refreshed every 10 ms by a thread of each process
// (jitc_liveness_init).
constexpr int kLiveMaxRanks = 1024;
struct Liveness {
  std::string path;
  uint64_t* hb = nullptr;  // kLiveMaxRanks heartbeats, indexed by job rank
  size_t bytes = 0;
  std::thread th;
  std::atomic<bool> run{false};
};

}  // namespace jitc

using namespace jitc;

struct jitc_ctx {
  jitc_config cfg{};
  std::string image_dir;
  int device = 0;
  cudaStream_t s_comp = nullptr, s_copy = nullptr;
  bool own_streams = false;
  uint8_t* staging = nullptr;
  uint64_t staging_bytes = 0, slot_bytes = 0;
  // copy-engine transfers (D2H / H2D) are issued in pieces of at most this
  // many bytes (env JITC_COPY_PIECE_MB; 0 = one copy per round)
  uint64_t copy_piece = 0;
  bool own_staging = false;
  static constexpr int kSlots = 8;
  cudaEvent_t ev_ready[kSlots]{}, ev_free[kSlots]{};
  cudaEvent_t ev_t0 = nullptr, ev_t1 = nullptr, ev_join = nullptr;
  std::vector<cudaEvent_t> kev;  // kernel timing pairs
  unsigned long long* d_span = nullptr;  // per timed launch: {~first CTA start, last CTA end} (%globaltimer)
  std::vector<unsigned long long> h_span;
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
  // parents of jitc_comm_shrink, aborted but not yet freed: freeing device
  // memory synchronises the device, and another communicator's collective
  // (the framework's all-reduce) may still be hung on the dead rank
  std::vector<ncclComm_t> retired_comms;
  int comm_n = 0, comm_rank = -1;
  std::vector<int32_t> comm_job;  // comm rank -> job rank
  std::unique_ptr<IpcComm> ipc;   // IPC transport (instead of `comm`)
  std::unique_ptr<Liveness> live; // heartbeats for the NCCL transport (jitc_liveness_init)
  bool comm_broken = false;       // an NCCL collective of `comm` waits on a dead peer (nccl_sync)
  std::vector<uint8_t> aux;       // user CPU state for the next commit (jitc_set_aux)
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
  std::vector<int32_t> fired_failed;  // job ranks the collective action found dead (guarded by wmu)
  std::string action_error;           // jitc_last_error text of a failed action (guarded by wmu)
  // test hook (JITC_DEBUG_FP_PAUSE_US, read at create): pause between the end
  // of K1 and the second phase-word read of jitc_fingerprint (seqlock test)
  uint32_t debug_fp_pause_us = 0;
  // test hook (JITC_DEBUG_EXIT_AFTER_ROUND=j, read at create): with the IPC
  // transport, the process exits right after posting restore round j - 1, so
  // that its peers' restore aborts part-way (tests/test_gpu_writer_death.py)
  uint32_t debug_exit_after_round = 0;
  // timeline (jitc_timeline_start / _read): two timing events per span
  struct TlRec {
    int32_t kind, stream;
    uint32_t group, round;
    uint64_t bytes;
    size_t e0, e1;
  };
  bool tl_on = false;
  std::vector<cudaEvent_t> tl_ev;
  std::vector<TlRec> tl;
  size_t tl_ev_used = 0;
  cudaEvent_t tl_base = nullptr;
  uint32_t tl_group = 0, tl_round = 0;  // attribution of the spans being recorded
  // counters
  jitc_kernel_counter kc[5]{};
  uint64_t launches_in_call = 0;
  double kernel_ms_in_call = 0;
};

// ----------------------------------------------------------------- helpers
namespace jitc {

inline jitc_status fail(jitc_status st, const std::string& msg) {
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

inline double now_ms() {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now().time_since_epoch()).count();
}

struct CallTimer {
  jitc_ctx* c;
  double t0;
  explicit CallTimer(jitc_ctx* ctx) : c(ctx), t0(now_ms()) {
    c->launches_in_call = 0;
    c->kernel_ms_in_call = 0;
    c->kev_used = 0;
    if (c->d_span) cudaMemsetAsync(c->d_span, 0, c->kev.size() * sizeof(unsigned long long), c->s_comp);
  }
};

// NVTX range for Nsight timelines (header-only NVTX3; a no-op without a tool attached)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

// Timeline spans (jitc_timeline_start): tl_open records the start event on
// stream s and returns its index (or SIZE_MAX when off / full); tl_close
// records the end event and the span.
inline size_t tl_open(jitc_ctx* c, cudaStream_t s) {
  if (!c->tl_on || c->tl_ev_used + 2 > c->tl_ev.size()) return SIZE_MAX;
  if (cudaEventRecord(c->tl_ev[c->tl_ev_used], s) != cudaSuccess) return SIZE_MAX;
  return c->tl_ev_used++;
}
inline void tl_close(jitc_ctx* c, size_t e0, cudaStream_t s, int kind, uint64_t bytes) {
  if (e0 == SIZE_MAX || c->tl_ev_used + 1 > c->tl_ev.size()) return;
  if (cudaEventRecord(c->tl_ev[c->tl_ev_used], s) != cudaSuccess) return;
  c->tl.push_back({kind, s == c->s_copy ? 1 : 0, c->tl_group, c->tl_round, bytes, e0, c->tl_ev_used++});
}

// Kernel launch with optional event bracketing (JITC_F_TIME_KERNELS).
inline jitc_status run_segments(jitc_ctx* c, GroupState& g, int mode, const LaunchRanges& r, uint64_t* dig,
                         uint64_t bytes, const uint64_t* remote = nullptr) {
  bool timed = (c->cfg.flags & JITC_F_TIME_KERNELS) && c->kev_used + 2 <= c->kev.size();
  const size_t tl0 = tl_open(c, c->s_comp);
  if (timed) CU(cudaEventRecord(c->kev[c->kev_used], c->s_comp));
  CU(launch_segments(mode, g.d_segs, r, dig, c->grid, c->d_work, c->s_comp, remote,
                     timed && c->d_span ? c->d_span + c->kev_used : nullptr));
  if (timed) {
    CU(cudaEventRecord(c->kev[c->kev_used + 1], c->s_comp));
    c->kev_kind[c->kev_used / 2] = mode;
    c->kev_bytes[c->kev_used / 2] = bytes;
    c->kev_used += 2;
  }
  tl_close(c, tl0, c->s_comp, mode, bytes);
  c->launches_in_call++;
  c->kc[mode].launches++;
  c->kc[mode].bytes += bytes;
  return JITC_OK;
}

// After the call's work has completed: harvest kernel timings into counters.
inline void harvest(jitc_ctx* c) {
  bool spans = c->d_span && c->kev_used &&
               cudaMemcpyAsync(c->h_span.data(), c->d_span, c->kev_used * sizeof(unsigned long long),
                               cudaMemcpyDeviceToHost, c->s_comp) == cudaSuccess &&
               cudaStreamSynchronize(c->s_comp) == cudaSuccess;
  for (size_t i = 0; i + 1 < c->kev_used; i += 2) {
    float ms = 0;
    if (cudaEventElapsedTime(&ms, c->kev[i], c->kev[i + 1]) == cudaSuccess) {
      c->kc[c->kev_kind[i / 2]].ms += ms;
      c->kernel_ms_in_call += ms;
    }
    if (spans && c->h_span[i + 1]) {
      const unsigned long long t0 = ~c->h_span[i], t1 = c->h_span[i + 1];
      if (t1 > t0) c->kc[c->kev_kind[i / 2]].span_ms += (t1 - t0) * 1e-6;
    }
  }
  c->kev_used = 0;
}

inline void finish_stats(jitc_ctx* c, const CallTimer& t, jitc_stats* st, bool device_span) {
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

// A copy between image bytes [img_off, img_off + n) of group g and device
// memory `dev`, issued in pieces of at most c->copy_piece bytes that never
// cross a registration boundary of the pinned image (cudaMemcpy refuses a
// host range that spans two registrations).
inline cudaError_t copy_image(jitc_ctx* c, const GroupState& g, uint64_t img_off, void* dev, uint64_t n,
                              cudaMemcpyKind kind, cudaStream_t s) {
  const size_t tl0 = tl_open(c, s);
  const uint64_t P = c->copy_piece ? c->copy_piece : n;
  const uint64_t R = g.img_reg_piece;
  uint64_t o = 0;
  while (o < n) {
    uint64_t len = std::min(P, n - o);
    if (R) len = std::min(len, R - (img_off + o) % R);
    uint8_t* h = g.img_h + img_off + o;
    uint8_t* d = static_cast<uint8_t*>(dev) + o;
    cudaError_t e = kind == cudaMemcpyDeviceToHost ? cudaMemcpyAsync(h, d, len, kind, s)
                                                   : cudaMemcpyAsync(d, h, len, kind, s);
    if (e != cudaSuccess) return e;
    o += len;
  }
  tl_close(c, tl0, s, kind == cudaMemcpyDeviceToHost ? 10 : 11, n);
  return cudaSuccess;
}

// Segments whose image offset lies in [a, b) (segments never straddle a chunk
// boundary and rounds are chunk-aligned, so this is exact).
inline void seg_span(const GroupState& g, uint64_t a, uint64_t b, uint32_t* lo, uint32_t* hi) {
  auto cmp = [](const Seg& s, uint64_t v) { return s.img_off < v; };
  *lo = (uint32_t)(std::lower_bound(g.segs.begin(), g.segs.end(), a, cmp) - g.segs.begin());
  *hi = (uint32_t)(std::lower_bound(g.segs.begin(), g.segs.end(), b, cmp) - g.segs.begin());
}

inline LaunchRanges one_range(uint32_t lo, uint32_t hi, const void* base, uint64_t base_off) {
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

inline void add_range(LaunchRanges& r, uint32_t lo, uint32_t hi, const void* base, uint64_t base_off) {
  r.seg_begin[r.n] = lo;
  r.seg_end[r.n] = hi;
  r.base[r.n] = (uint64_t)base;
  r.base_off[r.n] = base_off;
  r.prefix[r.n + 1] = r.prefix[r.n] + (hi - lo);
  r.n++;
}

inline jitc_status ensure_h_dig(jitc_ctx* c, size_t n) {
  if (n <= c->h_dig_n) return JITC_OK;
  if (c->h_dig) cudaFreeHost(c->h_dig);
  c->h_dig = nullptr;
  c->h_dig_n = 0;
  CU(cudaHostAlloc(&c->h_dig, std::max<size_t>(n, 1) * 8, cudaHostAllocDefault));
  c->h_dig_n = n;
  return JITC_OK;
}

// Unpins and unmaps a shared image, or frees a private one.
inline void release_image(GroupState& g) {
  if (g.img_h) {
    if (g.img_shm) {
      for (uint8_t* r : g.img_regs) cudaHostUnregister(r);
      munmap(g.img_h, g.img_bytes);
    } else {
      cudaFreeHost(g.img_h);
    }
  }
  g.img_regs.clear();
  g.img_reg_piece = 0;
  g.img_h = g.img_d = nullptr;
}

inline void free_group(GroupState& g) {
  if (g.d_segs) cudaFree(g.d_segs);
  if (g.d_dig) cudaFree(g.d_dig);
  if (g.d_dig2) cudaFree(g.d_dig2);
  if (g.d_remote) cudaFree(g.d_remote);
  g.d_remote = nullptr;
  release_image(g);
  g.d_segs = nullptr;
  g.d_dig = g.d_dig2 = nullptr;
}

inline std::string gpath(const jitc_ctx* c, uint32_t g, const char* ext) {
  return c->image_dir + "/g" + std::to_string(g) + ext;
}

inline std::vector<TopoEntry> topology(const jitc_ctx* c) {
  std::vector<TopoEntry> t;
  for (auto& kv : c->groups) t.push_back(TopoEntry{kv.first, kv.second.policy, kv.second.members});
  return t;
}

inline int comm_rank_of(const jitc_ctx* c, int32_t job) {
  for (int i = 0; i < c->comm_n; ++i)
    if (c->comm_job[i] == job) return i;
  return -1;
}

// Writes `path` via a temp file + rename.  The temp name is unique per process
// and call, so ranks that commit the same group at once (every rank's local
// capture) never write into each other's temp file; the last
// rename wins with a complete file.
inline bool write_file_atomic(const std::string& path, const uint8_t* p, size_t n) {
  static std::atomic<uint64_t> seq{0};
  std::string tmp = path + ".tmp." + std::to_string((long)getpid()) + "." + std::to_string(seq++);
  FILE* f = fopen(tmp.c_str(), "wb");
  if (!f) return false;
  bool ok = fwrite(p, 1, n, f) == n;
  ok = (fflush(f) == 0) && ok;
  ok = (fsync(fileno(f)) == 0) && ok;
  fclose(f);
  return ok && rename(tmp.c_str(), path.c_str()) == 0;
}

// A group the selection dropped (an OPTIONAL group with no candidate at v*,
// reading R1) keeps no checkpoint: its commit record (and manifest) from an
// earlier failure would otherwise stay valid at an older version and a later
// HOST restore without a selection would load it.  Every member that holds the
// group removes them (idempotent) at capture and again at commit.
inline void drop_commit(jitc_ctx* c, GroupState& g) {
  if (g.img_shm) {
    unlink(gpath(c, g.id, ".commit").c_str());
    unlink(gpath(c, g.id, ".manifest").c_str());
  }
  g.commit_priv.clear();
  g.man_priv.clear();
  g.captured = false;
}

inline bool read_file(const std::string& path, std::vector<uint8_t>* out) {
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

}  // namespace jitc
namespace jitc {
// IPC transport (jitc_ipc.cc)
jitc_status ipc_barrier(jitc_ctx* c);
jitc_status ipc_exchange(jitc_ctx* c, const void* mine, size_t len, void* all, size_t cap, size_t* all_len);
jitc_status ipc_gather(jitc_ctx* c, const void* mine, size_t len, std::vector<std::vector<uint8_t>>* parts);
jitc_status ipc_post(jitc_ctx* c, uint64_t* counter, uint64_t value, cudaStream_t s);
jitc_status ipc_wait(const uint64_t* counter, uint64_t value, const char* what);
// the same, failing with JITC_EPEER if comm rank `peer`'s heartbeat goes stale meanwhile
jitc_status ipc_wait_peer(const IpcComm& ic, int peer, const uint64_t* counter, uint64_t value, const char* what);
double peer_dead_ms();
bool ipc_peer_dead(const IpcComm& ic, int peer);  // comm rank's heartbeat older than ic.dead_ms
// job ranks of the communicator whose heartbeat is older than stale_ms (dead processes)
std::vector<int32_t> ipc_stale_ranks(jitc_ctx* c, double stale_ms);
// the same for whichever table this ctx has (IPC control block or liveness file)
std::vector<int32_t> stale_ranks(jitc_ctx* c, double stale_ms);
void liveness_destroy(jitc_ctx* c);
void ipc_destroy(jitc_ctx* c);
uint32_t group_slot(const jitc_ctx* c, uint32_t group);

inline bool has_comm(const jitc_ctx* c) { return c->comm || c->ipc; }

// Waits for the NCCL work enqueued on s_comp.  With a liveness table
// (jitc_liveness_init) the wait polls: a communicator member whose heartbeat
// goes stale cannot complete the collective, so the wait fails with
// JITC_EPEER and the caller shrinks (reading R9); an asynchronous NCCL error
// fails it with JITC_ENCCL.  Without a table: a plain stream synchronize.
jitc_status nccl_sync(jitc_ctx* c);

// Every comm rank contributes its local status; all return the same one: the
// first failing rank's code (lowest comm rank), JITC_OK if none failed.  A
// collective call whose ranks can fail independently (jitc_commit) ends with
// this instead of a plain barrier, so a failed rank neither leaves its peers
// blocked in the next collective nor lets them report success.
jitc_status agree(jitc_ctx* c, jitc_status mine);
// All-gather of one byte string per comm rank (any length, 0 included), in
// comm-rank order.  Collective; without a communicator returns {mine}.
jitc_status gather_bytes(jitc_ctx* c, const void* mine, size_t len, std::vector<std::vector<uint8_t>>* parts);

inline jitc_status barrier(jitc_ctx* c) {
  if (c->ipc) return ipc_barrier(c);
  if (!c->comm) return JITC_OK;
  NC(ncclAllReduce(c->d_small, c->d_small + 1, 1, ncclUint64, ncclSum, c->comm, c->s_comp));
  return nccl_sync(c);
}

}  // namespace jitc

namespace jitc {
// defined in jitc_capture.cc
jitc_status commit_impl(jitc_ctx* c, const void* selection, size_t sel_len, bool collective);
jitc_status local_capture(jitc_ctx* c, jitc_stats* st);
// defined in jitc_ctx.cc
jitc_status fingerprint_group(jitc_ctx* c, GroupState& g);
// defined in jitc_restore.cc: K2/K3/K5 digests of the group vs `want` (ECORRUPT + first bad chunk)
jitc_status compare_digests(jitc_ctx* c, GroupState& g, const std::vector<uint64_t>& want, jitc_stats* stats);
}  // namespace jitc
