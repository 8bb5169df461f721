// Intra-node IPC transport: the library communicator without NCCL.
//
// The ranks of one box share a control block (IpcCtl) in a /dev/shm file and
// map each other's staging buffers through CUDA IPC.  Every signal is a
// monotonically increasing counter:
//   posted[r][g]   -- rank r's outgoing block of its restore round is ready,
//   consumed[r][g] -- rank r has finished reading every block of a round,
//   arrive[r]      -- barrier generation,
// written by the GPU in stream order (cuStreamWriteValue64 into the
// cudaHostRegister-mapped block, after the kernels / copies that produce or
// consume the data) or by the host (barriers), and polled by the peers' host
// threads before they enqueue dependent work.  A receiver's K3 reads the
// sender's block straight out of the sender's staging buffer -- NVLink peer
// loads on a multi-GPU node -- so the exchange and the unpack+verify are one
// kernel.  The communicator's directory must be fresh for every communicator
// (it plays the role of an NCCL unique id).
#include <sched.h>

#include "jitc_ctx.h"

using namespace jitc;

namespace {

typedef CUresult (*PFN_getAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr);

PFN_getAddressRange range_fn() {
  static PFN_getAddressRange fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (PFN_getAddressRange)p;
  }
  return fn;
}

inline uint64_t load_acq(const uint64_t* p) { return __atomic_load_n(p, __ATOMIC_ACQUIRE); }
inline void store_rel(uint64_t* p, uint64_t v) { __atomic_store_n(p, v, __ATOMIC_RELEASE); }

constexpr double kIpcTimeoutMs = 600000.0;

uint64_t mono_us() {
  return (uint64_t)std::chrono::duration_cast<std::chrono::microseconds>(
             std::chrono::steady_clock::now().time_since_epoch()).count();
}

}  // namespace

namespace jitc {

uint32_t group_slot(const jitc_ctx* c, uint32_t group) {
  uint32_t i = 0;
  for (auto& kv : c->groups) {
    if (kv.first == group) return i;
    ++i;
  }
  return i;
}

jitc_status ipc_wait(const uint64_t* counter, uint64_t value, const char* what) {
  const double t0 = now_ms();
  uint32_t spins = 0;
  while (load_acq(counter) < value) {
    if (++spins > 1000) sched_yield();
    if ((spins & 0xFFFF) == 0 && now_ms() - t0 > kIpcTimeoutMs)
      return fail(JITC_ESTATE, std::string("IPC transport: timed out waiting for ") + what);
  }
  return JITC_OK;
}

double peer_dead_ms() {
  const char* e = getenv("JITC_PEER_DEAD_MS");
  double v = e ? atof(e) : 0.0;
  return v > 0 ? v : 2000.0;
}

jitc_status nccl_sync(jitc_ctx* c) {
  if (!c->live || !c->comm) {
    CU(cudaStreamSynchronize(c->s_comp));
    return JITC_OK;
  }
  const double dead_ms = peer_dead_ms();
  for (uint32_t it = 1;; ++it) {
    cudaError_t e = cudaStreamQuery(c->s_comp);
    if (e == cudaSuccess) return JITC_OK;
    if (e != cudaErrorNotReady) return fail(JITC_ECUDA, std::string("nccl_sync: ") + cudaGetErrorString(e));
    if ((it & 31) == 0) {
      std::vector<int32_t> d = stale_ranks(c, dead_ms);
      if (!d.empty()) {
        c->comm_broken = true;
        return fail(JITC_EPEER, "NCCL collective waits on a dead peer (job rank " + std::to_string(d[0]) +
                                    ", heartbeat stale); shrink and retry");
      }
      ncclResult_t ae = ncclSuccess;
      if (ncclCommGetAsyncError(c->comm, &ae) == ncclSuccess && ae != ncclSuccess && ae != ncclInProgress) {
        c->comm_broken = true;
        return fail(JITC_ENCCL, std::string("NCCL asynchronous error: ") + ncclGetErrorString(ae));
      }
    }
    std::this_thread::sleep_for(std::chrono::microseconds(50));
  }
}

bool ipc_peer_dead(const IpcComm& ic, int peer) {
  const uint64_t hb = load_acq(&ic.ctl->heartbeat[ic.slot[peer]]);
  return hb && mono_us() > hb + (uint64_t)(ic.dead_ms * 1000.0);
}

// Waits on a counter that comm rank `peer` advances; a peer whose heartbeat
// (refreshed every 10 ms by its heartbeat thread) is older than ic.dead_ms is
// dead: the wait fails with JITC_EPEER instead of spinning until the 10-minute
// timeout (reading R9: a writer that dies during the capture).
jitc_status ipc_wait_peer(const IpcComm& ic, int peer, const uint64_t* counter, uint64_t value, const char* what) {
  const double t0 = now_ms();
  uint32_t spins = 0;
  while (load_acq(counter) < value) {
    if (++spins > 1000) sched_yield();
    if ((spins & 0x3FF) == 0) {
      if (ipc_peer_dead(ic, peer))
        return fail(JITC_EPEER, std::string("IPC transport: comm rank ") + std::to_string(peer) +
                                    " died (heartbeat stale) while waiting for " + what);
      if (now_ms() - t0 > kIpcTimeoutMs)
        return fail(JITC_ESTATE, std::string("IPC transport: timed out waiting for ") + what);
    }
  }
  return JITC_OK;
}

jitc_status ipc_post(jitc_ctx* c, uint64_t* counter, uint64_t value, cudaStream_t s) {
  uint64_t* dev = reinterpret_cast<uint64_t*>(c->ipc->ctl_dev + ((uint8_t*)counter - (uint8_t*)c->ipc->ctl));
  if (c->write_value64 && c->write_value64((CUstream)s, (CUdeviceptr)dev, value, 0) == CUDA_SUCCESS) return JITC_OK;
  CU(launch_phase_write(dev, value, s));
  return JITC_OK;
}

jitc_status ipc_barrier(jitc_ctx* c) {
  IpcComm& ic = *c->ipc;
  const uint64_t gen = ++ic.barrier_gen;
  store_rel(&ic.ctl->arrive[ic.slot[c->comm_rank]], gen);
  for (int q = 0; q < c->comm_n; ++q) {
    jitc_status st = ipc_wait_peer(ic, q, &ic.ctl->arrive[ic.slot[q]], gen, "a barrier");
    if (st) return st;
  }
  return JITC_OK;
}

// (failed ? (~comm_rank << 32) | -status : 0): the max over ranks is the
// failing rank with the lowest comm rank, its status in the low word
static uint64_t agree_word(const jitc_ctx* c, jitc_status st) {
  return st ? ((uint64_t)(0xFFFFFFFFu - (uint32_t)c->comm_rank) << 32) | (uint32_t)(-st) : 0;
}

jitc_status agree(jitc_ctx* c, jitc_status mine) {
  const std::string mine_err = mine ? get_error() : std::string();
  uint64_t worst = agree_word(c, mine);
  if (c->ipc) {
    IpcComm& ic = *c->ipc;
    const uint64_t gen = ++ic.agree_gen;
    uint64_t* row = ic.ctl->agree[gen & 1];
    // (generation << 40) | (failed ? 1 << 16 | -status : 0); the reader knows the rank
    const uint64_t w = mine ? (1ull << 16) | (uint16_t)(-mine) : 0;
    store_rel(&row[ic.slot[c->comm_rank]], (gen << 40) | w);
    for (int q = 0; q < c->comm_n; ++q) {
      const uint64_t* p = &row[ic.slot[q]];
      jitc_status st = ipc_wait_peer(ic, q, p, gen << 40, "a status agreement");
      if (st) return st;
      const uint64_t v = load_acq(p) & ((1ull << 40) - 1);
      if (v) {
        const uint64_t full = ((0xFFFFFFFFull - (uint64_t)q) << 32) | (v & 0xFFFF);
        worst = std::max(worst, full);
      }
    }
  } else if (c->comm) {
    c->h_small[2] = worst;
    CU(cudaMemcpyAsync(c->d_small + 4, c->h_small + 2, 8, cudaMemcpyHostToDevice, c->s_comp));
    NC(ncclAllReduce(c->d_small + 4, c->d_small + 5, 1, ncclUint64, ncclMax, c->comm, c->s_comp));
    if (jitc_status st = nccl_sync(c)) return st;
    CU(cudaMemcpyAsync(c->h_small + 3, c->d_small + 5, 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
    worst = c->h_small[3];
  }
  if (!worst) return JITC_OK;
  const int who = (int)(0xFFFFFFFFu - (uint32_t)(worst >> 32));
  const jitc_status code = -(jitc_status)(worst & 0xFFFF);
  if (who == c->comm_rank) return fail(mine, mine_err);
  if (mine) return fail(mine, mine_err);
  return fail(code, "comm rank " + std::to_string(who) + " (job rank " +
                        std::to_string(who >= 0 && who < (int)c->comm_job.size() ? c->comm_job[who] : -1) +
                        ") failed with status " + std::to_string(code));
}

jitc_status ipc_gather(jitc_ctx* c, const void* mine, size_t len, std::vector<std::vector<uint8_t>>* parts) {
  IpcComm& ic = *c->ipc;
  // every gather (and each call of the two-call exchange size query) runs the
  // whole protocol, so the generations stay in step on every rank
  const uint64_t gen = ++ic.exchange_gen;
  std::string me = ic.dir + "/blob." + std::to_string(gen) + "." + std::to_string(ic.slot[c->comm_rank]);
  if (!write_file_atomic(me, static_cast<const uint8_t*>(mine), len)) return fail(JITC_EIO, "IPC gather: writing " + me);
  jitc_status st = ipc_barrier(c);
  if (st) return st;
  parts->assign(c->comm_n, {});
  for (int q = 0; q < c->comm_n; ++q) {
    std::string p = ic.dir + "/blob." + std::to_string(gen) + "." + std::to_string(ic.slot[q]);
    if (!read_file(p, &(*parts)[q])) return fail(JITC_EIO, "IPC gather: reading " + p);
  }
  st = ipc_barrier(c);  // every rank has read every blob
  if (st) return st;
  unlink(me.c_str());
  return JITC_OK;
}

jitc_status ipc_exchange(jitc_ctx* c, const void* mine, size_t len, void* all, size_t cap, size_t* all_len) {
  std::vector<std::vector<uint8_t>> parts;
  jitc_status st = ipc_gather(c, mine, len, &parts);
  if (st) return st;
  std::vector<uint8_t> out;
  for (auto& b : parts) out.insert(out.end(), b.begin(), b.end());
  *all_len = out.size();
  if (cap == 0) return JITC_OK;
  if (cap < out.size() || !all) return fail(JITC_EINVAL, "jitc_exchange_records: buffer too small");
  memcpy(all, out.data(), out.size());
  return JITC_OK;
}

std::vector<int32_t> ipc_stale_ranks(jitc_ctx* c, double stale_ms) {
  std::vector<int32_t> out;
  if (!c->ipc) return out;
  const uint64_t now = mono_us();
  for (int q = 0; q < c->comm_n; ++q) {
    if (q == c->comm_rank) continue;
    uint64_t hb = load_acq(&c->ipc->ctl->heartbeat[c->ipc->slot[q]]);
    if (hb == 0 || now > hb + (uint64_t)(stale_ms * 1000.0)) out.push_back(c->comm_job[q]);
  }
  return out;
}

std::vector<int32_t> stale_ranks(jitc_ctx* c, double stale_ms) {
  if (c->ipc) return ipc_stale_ranks(c, stale_ms);
  std::vector<int32_t> out;
  if (!c->live) return out;
  const uint64_t now = mono_us();
  for (int q = 0; q < c->comm_n; ++q) {
    const int32_t j = c->comm_job[q];
    if (q == c->comm_rank) continue;
    uint64_t hb = (j >= 0 && j < kLiveMaxRanks) ? load_acq(&c->live->hb[j]) : 0;
    if (hb == 0 || now > hb + (uint64_t)(stale_ms * 1000.0)) out.push_back(j);
  }
  return out;
}

void liveness_destroy(jitc_ctx* c) {
  if (!c->live) return;
  c->live->run = false;
  if (c->live->th.joinable()) c->live->th.join();
  if (c->live->hb) munmap(c->live->hb, c->live->bytes);
  c->live.reset();
}

void ipc_destroy(jitc_ctx* c) {
  if (!c->ipc) return;
  IpcComm& ic = *c->ipc;
  ic.hb_run = false;
  if (ic.hb_thread.joinable()) ic.hb_thread.join();
  for (void* p : ic.opened) cudaIpcCloseMemHandle(p);
  if (ic.ctl) {
    cudaHostUnregister(ic.ctl);
    munmap(ic.ctl, ic.ctl_bytes);
  }
  c->ipc.reset();
}

}  // namespace jitc

extern "C" jitc_status jitc_comm_init_ipc(jitc_ctx* c, const char* comm_dir, int32_t nranks, int32_t comm_rank,
                                          const int32_t* job_ranks) {
  if (!c || !comm_dir || nranks <= 0 || nranks > kIpcMaxRanks || comm_rank < 0 || comm_rank >= nranks)
    return fail(JITC_EINVAL, "jitc_comm_init_ipc: bad argument");
  if (c->groups.size() > (size_t)kIpcMaxGroups) return fail(JITC_EINVAL, "jitc_comm_init_ipc: too many groups");
  CU(cudaSetDevice(c->device));
  if (c->comm) {  // retired, not freed: see jitc_ctx::retired_comms
    c->retired_comms.push_back(c->comm);
    c->comm = nullptr;
  }
  ipc_destroy(c);
  PFN_getAddressRange range = range_fn();
  if (!range) return fail(JITC_ECUDA, "jitc_comm_init_ipc: cuMemGetAddressRange unavailable");
  std::unique_ptr<IpcComm> ic(new IpcComm());
  ic->dir = comm_dir;
  ic->dead_ms = peer_dead_ms();
  mkdir(ic->dir.c_str(), 0700);
  std::string path = ic->dir + "/ctl";
  ic->ctl_bytes = align_up(sizeof(IpcCtl), 4096);
  int fd = open(path.c_str(), O_RDWR | O_CREAT, 0600);
  if (fd < 0) return fail(JITC_EIO, "jitc_comm_init_ipc: open " + path + ": " + strerror(errno));
  flock(fd, LOCK_EX);
  struct stat sb;
  if (fstat(fd, &sb) == 0 && (uint64_t)sb.st_size < ic->ctl_bytes && ftruncate(fd, (off_t)ic->ctl_bytes) != 0) {
    flock(fd, LOCK_UN);
    close(fd);
    return fail(JITC_EIO, "jitc_comm_init_ipc: sizing " + path);
  }
  void* p = mmap(nullptr, ic->ctl_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  cudaError_t e = p == MAP_FAILED ? cudaErrorMemoryAllocation
                                  : cudaHostRegister(p, ic->ctl_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
  flock(fd, LOCK_UN);
  close(fd);
  if (p == MAP_FAILED) return fail(JITC_EIO, "jitc_comm_init_ipc: mmap " + path);
  if (e != cudaSuccess) {
    munmap(p, ic->ctl_bytes);
    return fail(JITC_ECUDA, std::string("jitc_comm_init_ipc: cudaHostRegister: ") + cudaGetErrorString(e));
  }
  ic->ctl = static_cast<IpcCtl*>(p);
  CU(cudaHostGetDevicePointer((void**)&ic->ctl_dev, p, 0));
  // publish this rank's staging
  CUdeviceptr base = 0;
  size_t size = 0;
  if (range(&base, &size, (CUdeviceptr)c->staging) != CUDA_SUCCESS)
    return fail(JITC_ECUDA, "jitc_comm_init_ipc: staging is not device memory");
  cudaIpcMemHandle_t h;
  e = cudaIpcGetMemHandle(&h, (void*)base);
  if (e != cudaSuccess)
    return fail(JITC_ECUDA, std::string("jitc_comm_init_ipc: cudaIpcGetMemHandle(staging): ") + cudaGetErrorString(e));
  ic->ctl->staging[comm_rank] = h;
  ic->ctl->staging_off[comm_rank] = (uint64_t)c->staging - (uint64_t)base;
  store_rel(&ic->ctl->published[comm_rank], 1);
  ic->slot.resize(nranks);
  for (int i = 0; i < nranks; ++i) ic->slot[i] = i;
  ic->peer_staging.assign(nranks, nullptr);
  ic->peer_staging[comm_rank] = c->staging;
  c->comm_n = nranks;
  c->comm_rank = comm_rank;
  c->comm_job.resize(nranks);
  for (int i = 0; i < nranks; ++i) c->comm_job[i] = job_ranks ? job_ranks[i] : i;
  if (c->comm_job[comm_rank] != c->cfg.rank) return fail(JITC_EINVAL, "jitc_comm_init_ipc: job_ranks[comm_rank] != cfg.rank");
  for (int q = 0; q < nranks; ++q) {
    if (q == comm_rank) continue;
    jitc_status st = ipc_wait(&ic->ctl->published[q], 1, "a peer to publish its staging");
    if (st) return st;
    void* m = nullptr;
    e = cudaIpcOpenMemHandle(&m, ic->ctl->staging[q], cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess)
      return fail(JITC_ECUDA, std::string("jitc_comm_init_ipc: cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
    ic->opened.push_back(m);
    ic->peer_staging[q] = static_cast<uint8_t*>(m) + ic->ctl->staging_off[q];
  }
  // heartbeat: lets the survivors of a hang tell a dead peer from a hung one
  store_rel(&ic->ctl->heartbeat[comm_rank], mono_us());
  ic->hb_run = true;
  IpcCtl* ctl = ic->ctl;
  IpcComm* icp = ic.get();
  ic->hb_thread = std::thread([ctl, icp, comm_rank] {
    while (icp->hb_run) {
      store_rel(&ctl->heartbeat[comm_rank], mono_us());
      std::this_thread::sleep_for(std::chrono::milliseconds(10));
    }
  });
  c->ipc = std::move(ic);
  return ipc_barrier(c);
}

// Liveness table for the NCCL transport (see include/jitc.h).
extern "C" jitc_status jitc_liveness_init(jitc_ctx* c, const char* dir) {
  if (!c || !dir) return fail(JITC_EINVAL, "jitc_liveness_init: null argument");
  if (c->cfg.rank < 0 || c->cfg.rank >= kLiveMaxRanks)
    return fail(JITC_EINVAL, "jitc_liveness_init: job rank out of range [0, " + std::to_string(kLiveMaxRanks) + ")");
  liveness_destroy(c);
  std::unique_ptr<Liveness> lv(new Liveness());
  mkdir(dir, 0700);
  lv->path = std::string(dir) + "/liveness";
  lv->bytes = align_up(sizeof(uint64_t) * kLiveMaxRanks, 4096);
  int fd = open(lv->path.c_str(), O_RDWR | O_CREAT, 0600);
  if (fd < 0) return fail(JITC_EIO, "jitc_liveness_init: open " + lv->path + ": " + strerror(errno));
  flock(fd, LOCK_EX);
  struct stat sb;
  bool ok = fstat(fd, &sb) == 0 && ((uint64_t)sb.st_size >= lv->bytes || ftruncate(fd, (off_t)lv->bytes) == 0);
  void* p = ok ? mmap(nullptr, lv->bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0) : MAP_FAILED;
  flock(fd, LOCK_UN);
  close(fd);
  if (p == MAP_FAILED) return fail(JITC_EIO, "jitc_liveness_init: mapping " + lv->path);
  lv->hb = static_cast<uint64_t*>(p);
  const int32_t me = c->cfg.rank;
  store_rel(&lv->hb[me], mono_us());
  lv->run = true;
  Liveness* l = lv.get();
  lv->th = std::thread([l, me] {
    while (l->run) {
      store_rel(&l->hb[me], mono_us());
      std::this_thread::sleep_for(std::chrono::milliseconds(10));
    }
  });
  c->live = std::move(lv);
  return JITC_OK;
}

extern "C" jitc_status jitc_comm_dead(jitc_ctx* c, int32_t* ranks, int32_t cap, int32_t* n) {
  if (!c || !n || (cap > 0 && !ranks)) return fail(JITC_EINVAL, "jitc_comm_dead: bad argument");
  if (!has_comm(c)) return fail(JITC_ESTATE, "jitc_comm_dead: no communicator");
  if (!c->ipc && !c->live) return fail(JITC_ESTATE, "jitc_comm_dead: no heartbeats (IPC transport or jitc_liveness_init)");
  std::vector<int32_t> d = stale_ranks(c, c->ipc ? c->ipc->dead_ms : peer_dead_ms());
  *n = (int32_t)d.size();
  for (int32_t i = 0; i < *n && i < cap; ++i) ranks[i] = d[i];
  return JITC_OK;
}
