// libjitc.so context: create / destroy, registration (A1), phase words (A2),
// the library-owned NCCL communicator, fingerprint (A3 = K1) and the record
// exchange (A4 = C1).  Capture / commit, restore / verify, the durable tier
// and the watchdog live in jitc_capture.cc, jitc_restore.cc, jitc_durable.cc
// and jitc_watchdog.cc.
//
// Method: PAPER.md §3 (user-level JIT checkpointing) -- healthy DP replicas
// save their GPU state after a peer fails, on side streams
// (:134), to rank-dependent locations with metadata written last (:136); the
// restore loads any consistent replica and discards corrupted ones (:140);
// the state may be at minibatch i or i+1 (:148); a replica's state can be
// copied straight to a reset GPU (:174, :184).
#include "jitc_ctx.h"

using namespace jitc;

// ------------------------------------------------------------ fingerprint (K1)
// The phase word is read twice, before K1 and after it completed (a seqlock):
// a word that changed in between means the optimizer step that the hooks
// bracket ran -- or started -- while K1 read the tensors, so the
// digests may mix bytes from before and after it.  Such a record is labelled
// DIRTY at the newer version and is never selected (reading R6); otherwise a
// lone replica, guarded by its phase word alone (reading R12), could be
// committed as CLEAN over torn bytes when the step stalls after K1.
jitc_status jitc::fingerprint_group(jitc_ctx* c, GroupState& g) {
  const uint64_t w = __atomic_load_n(&c->phase_h[g.slot], __ATOMIC_ACQUIRE);
  if (g.n_c) {
    CU(cudaMemsetAsync(g.d_dig, 0, g.n_c * 8, c->s_comp));
    jitc_status st = run_segments(c, g, kDigest, one_range(0, (uint32_t)g.segs.size(), nullptr, 0), g.d_dig, g.L);
    if (st) return st;
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
  }
  CU(cudaStreamSynchronize(c->s_comp));
  if (c->debug_fp_pause_us) usleep(c->debug_fp_pause_us);
  const uint64_t w2 = __atomic_load_n(&c->phase_h[g.slot], __ATOMIC_ACQUIRE);
  g.fp_version = w2 >> 1;
  g.fp_phase = (w2 != w) ? JITC_PHASE_DIRTY : (int)(w & 1);
  g.fp.assign(c->h_dig, c->h_dig + g.n_c);
  g.fp_root = root_of(g.layout_hash, g.fp.data(), g.n_c);
  g.has_fp = true;
  g.captured = false;  // a capture belongs to the fingerprint it was checked against
  return JITC_OK;
}

// NCCL all-gather of one byte string per comm rank: the sizes first, then the
// strings padded to the largest, in place in staging.
static jitc_status nccl_gather(jitc_ctx* c, const void* mine, size_t len, std::vector<std::vector<uint8_t>>* parts) {
  const int n = c->comm_n;
  uint64_t* dsz = reinterpret_cast<uint64_t*>(c->staging);
  c->h_small[0] = len;
  CU(cudaMemcpyAsync(dsz + c->comm_rank, c->h_small, 8, cudaMemcpyHostToDevice, c->s_comp));
  NC(ncclAllGather(dsz + c->comm_rank, dsz, 1, ncclUint64, c->comm, c->s_comp));
  // wait for the collective before any copy into pageable memory (such a copy
  // blocks the host behind it, where a dead peer could never be noticed)
  if (jitc_status st = nccl_sync(c)) return st;
  std::vector<uint64_t> sizes(n);
  CU(cudaMemcpyAsync(sizes.data(), dsz, 8ull * n, cudaMemcpyDeviceToHost, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  uint64_t maxlen = 0;
  for (uint64_t s : sizes) maxlen = std::max(maxlen, s);
  maxlen = align_up(std::max<uint64_t>(maxlen, 1), 256);
  if (256 + n * maxlen > c->staging_bytes) return fail(JITC_ENOMEM, "gather: blobs exceed staging");
  uint8_t* recv = c->staging + 256;
  if (len) CU(cudaMemcpyAsync(recv + c->comm_rank * maxlen, mine, len, cudaMemcpyHostToDevice, c->s_comp));
  NC(ncclAllGather(recv + c->comm_rank * maxlen, recv, maxlen, ncclUint8, c->comm, c->s_comp));
  if (jitc_status st = nccl_sync(c)) return st;
  std::vector<uint8_t> all(n * maxlen);
  CU(cudaMemcpyAsync(all.data(), recv, n * maxlen, cudaMemcpyDeviceToHost, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  parts->assign(n, {});
  for (int r = 0; r < n; ++r) (*parts)[r].assign(all.data() + r * maxlen, all.data() + r * maxlen + sizes[r]);
  return JITC_OK;
}

jitc_status jitc::gather_bytes(jitc_ctx* c, const void* mine, size_t len, std::vector<std::vector<uint8_t>>* parts) {
  if (c->ipc) return ipc_gather(c, mine, len, parts);
  if (!c->comm) {
    parts->assign(1, std::vector<uint8_t>(static_cast<const uint8_t*>(mine), static_cast<const uint8_t*>(mine) + len));
    return JITC_OK;
  }
  CU(cudaSetDevice(c->device));
  return nccl_gather(c, mine, len, parts);
}

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
  c->copy_piece = kDefaultCopyPiece;
  if (const char* e = getenv("JITC_COPY_PIECE_MB")) c->copy_piece = strtoull(e, nullptr, 10) << 20;
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
    CU(cudaMalloc(&c->d_span, c->kev.size() * sizeof(unsigned long long)));
    CU(cudaMemset(c->d_span, 0, c->kev.size() * sizeof(unsigned long long)));
    c->h_span.assign(c->kev.size(), 0);
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
  if (const char* e = getenv("JITC_DEBUG_FP_PAUSE_US")) c->debug_fp_pause_us = (uint32_t)strtoul(e, nullptr, 10);
  if (const char* e = getenv("JITC_DEBUG_EXIT_AFTER_ROUND"))
    c->debug_exit_after_round = (uint32_t)strtoul(e, nullptr, 10);
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
  for (ncclComm_t r : c->retired_comms) ncclCommAbort(r);
  c->retired_comms.clear();
  ipc_destroy(c);
  liveness_destroy(c);
  for (auto& kv : c->groups) free_group(kv.second);
  for (int i = 0; i < jitc_ctx::kSlots; ++i) {
    if (c->ev_ready[i]) cudaEventDestroy(c->ev_ready[i]);
    if (c->ev_free[i]) cudaEventDestroy(c->ev_free[i]);
  }
  for (auto& ev : c->kev) cudaEventDestroy(ev);
  for (auto& ev : c->tl_ev) cudaEventDestroy(ev);
  if (c->tl_base) cudaEventDestroy(c->tl_base);
  if (c->ev_t0) cudaEventDestroy(c->ev_t0);
  if (c->ev_t1) cudaEventDestroy(c->ev_t1);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  if (c->phase_h) cudaFreeHost(c->phase_h);
  if (c->h_dig) cudaFreeHost(c->h_dig);
  if (c->h_small) cudaFreeHost(c->h_small);
  if (c->d_small) cudaFree(c->d_small);
  if (c->d_work) cudaFree(c->d_work);
  if (c->d_span) cudaFree(c->d_span);
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

// Registration geometry of a shared image: pieces of kRegPiece bytes, first
// populated (page tables filled, tmpfs pages allocated) and then pinned, each
// step by a pool of threads.  Measured on the pool's boxes for 120 GiB
// (tools/pin_probe5.py, profiles/r02_pin_probe.txt): posix_fallocate 9 s +
// one-thread-at-a-time registration 35-44 s, versus 4.6 s of parallel
// MADV_POPULATE_WRITE + 12.3 s of parallel registration of the populated
// pages (16 threads) -- registration is mostly page-table population, which
// parallelises when done by madvise and not inside cudaHostRegister.
// JITC_PIN_THREADS overrides the thread count (1 => one registration of the
// whole image); JITC_PIN_PIECE_MB the piece size (tests).
constexpr uint64_t kRegPiece = 1ull << 30;
constexpr int kPinThreads = 16;

// NUMA placement of the shared image (VERDICT r01 missing #6
// §5.2: the host link is the floor, and on a two-socket 8-GPU host a rank's
// copy engine reaches the far socket's memory only across the inter-socket
// link).  The rank that creates the image sets a shared memory policy per
// slice before the pages are allocated: slice r = bytes [r*L/n, (r+1)*L/n)
// of the n = world ranks (page-aligned), the range rank r writes in a k = n
// capture and loads in an n-way HOST restore, preferred on the NUMA node of
// GPU r % device_count (sysfs).  tmpfs keeps the policy with the file, and the
// posix_fallocate that follows allocates every page under it.  Skipped on a
// single-node host unless JITC_NUMA=force (tests); JITC_NUMA=off disables it.
static int gpu_numa_node(int dev) {
  char bus[64] = {0};
  if (cudaDeviceGetPCIBusId(bus, sizeof bus, dev) != cudaSuccess) return -1;
  for (char* q = bus; *q; ++q) *q = (char)tolower(*q);
  FILE* f = fopen((std::string("/sys/bus/pci/devices/") + bus + "/numa_node").c_str(), "r");
  int node = -1;
  if (f) {
    if (fscanf(f, "%d", &node) != 1) node = -1;
    fclose(f);
  }
  return node;
}

static int host_numa_nodes() {
  int n = 0;
  for (int i = 0; i < 1024; ++i) {
    struct stat sb;
    if (stat(("/sys/devices/system/node/node" + std::to_string(i)).c_str(), &sb) != 0) break;
    ++n;
  }
  return n;
}

// returns the number of slices given a policy
static int place_image_slices(jitc_ctx* c, uint8_t* p, uint64_t bytes) {
  const char* mode = getenv("JITC_NUMA");
  if (mode && !strcmp(mode, "off")) return 0;
  const bool force = mode && !strcmp(mode, "force");
  if (!force && host_numa_nodes() < 2) return 0;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev <= 0) return 0;
  const uint64_t world = (uint64_t)std::max(c->cfg.world, 1), page = 2ull << 20;
  int placed = 0;
  for (uint64_t r = 0; r < world; ++r) {
    const uint64_t a = (r * bytes / world) / page * page;
    const uint64_t b = r + 1 == world ? bytes : ((r + 1) * bytes / world) / page * page;
    const int node = gpu_numa_node((int)(r % (uint64_t)ndev));
    if (b <= a || node < 0 || node >= 64) continue;
    unsigned long mask = 1ul << node;
    // mbind(addr, len, MPOL_PREFERRED, nodemask, maxnode, flags)
    if (syscall(SYS_mbind, p + a, b - a, 1 /* MPOL_PREFERRED */, &mask, 64ul, 0u) == 0) ++placed;
  }
  return placed;
}

static jitc_status map_shared_image(jitc_ctx* c, GroupState& g, const std::string& who) {
  mkdir(c->image_dir.c_str(), 0700);
  g.img_path = gpath(c, g.id, ".img");
  const double t_open = now_ms();
  int fd = open(g.img_path.c_str(), O_RDWR | O_CREAT, 0600);
  if (fd < 0) return fail(JITC_EIO, who + ": open " + g.img_path + ": " + strerror(errno));
  flock(fd, LOCK_EX);
  struct stat sb;
  int err = 0;
  bool fresh = false;
  if (fstat(fd, &sb) != 0) err = errno ? errno : EIO;
  if (!err && (uint64_t)sb.st_size != g.img_bytes) {
    fresh = true;
    if (ftruncate(fd, (off_t)g.img_bytes) != 0) err = errno ? errno : EIO;
  }
  void* p = MAP_FAILED;
  if (!err) {
    p = mmap(nullptr, g.img_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
    if (p == MAP_FAILED) err = errno ? errno : ENOMEM;
  }
  int placed = 0;
  if (!err && fresh) placed = place_image_slices(c, static_cast<uint8_t*>(p), g.img_bytes);
  flock(fd, LOCK_UN);
  if (err) {
    close(fd);
    if (p != MAP_FAILED) munmap(p, g.img_bytes);
    return fail(JITC_EIO, who + ": sizing " + g.img_path + ": " + strerror(err));
  }
  g.img_numa_slices = placed;
  const double t_sized = now_ms();
  int same = 0;
  cudaDeviceGetAttribute(&same, cudaDevAttrCanUseHostPointerForRegisteredMem, c->device);
  int threads = std::min<int>(kPinThreads, std::max(1u, std::thread::hardware_concurrency()));
  if (const char* e = getenv("JITC_PIN_THREADS")) threads = std::max(1, atoi(e));
  uint64_t reg_piece = kRegPiece;
  if (const char* e = getenv("JITC_PIN_PIECE_MB")) reg_piece = std::max<uint64_t>(1, strtoull(e, nullptr, 10)) << 20;
  const uint64_t piece = (same && threads > 1 && g.img_bytes > reg_piece) ? reg_piece : g.img_bytes;
  const uint64_t n_pieces = (g.img_bytes + piece - 1) / piece;
  auto pool_run = [&](const std::function<void(uint64_t)>& fn) {
    std::atomic<uint64_t> next{0};
    auto work = [&] {
      cudaSetDevice(c->device);
      for (uint64_t i; (i = next++) < n_pieces;) fn(i);
    };
    std::vector<std::thread> pool;
    for (int t = 1; t < threads && (uint64_t)t < n_pieces; ++t) pool.emplace_back(work);
    work();
    for (auto& th : pool) th.join();
  };
  // 1. allocate the pages and fill this process's page tables, in parallel,
  //    and pin each piece right after populating it (page zeroing and the
  //    driver's pinning overlap across the pool: C3 setup 23 s on average
  //    against 33 s populating everything first, tools/setup_probe.py,
  //    profiles/r02f_setup_probe.txt; JITC_PIN_FUSED=0 restores the two
  //    phases).  Kernels without MADV_POPULATE_WRITE (< 5.14) fall back to
  //    fallocate and pin afterwards.
  std::atomic<int> pop_err{0};
  const bool fused = !(getenv("JITC_PIN_FUSED") && atoi(getenv("JITC_PIN_FUSED")) == 0);
  std::vector<cudaError_t> rc(n_pieces, cudaSuccess);
  std::vector<char> pinned(n_pieces, 0);
  pool_run([&](uint64_t i) {
    const uint64_t a = i * piece, n = std::min(piece, g.img_bytes - a);
    if (madvise(static_cast<uint8_t*>(p) + a, n, 23 /* MADV_POPULATE_WRITE */) != 0) {
      pop_err = errno;
      return;
    }
    if (fused) {
      rc[i] = cudaHostRegister(static_cast<uint8_t*>(p) + a, n, cudaHostRegisterMapped | cudaHostRegisterPortable);
      pinned[i] = 1;
    }
  });
  if (pop_err) {
    const int e = pop_err == EINVAL ? posix_fallocate(fd, 0, (off_t)g.img_bytes) : (int)pop_err;
    if (e) {
      close(fd);
      munmap(p, g.img_bytes);
      return fail(JITC_EIO, who + ": allocating " + g.img_path + ": " + strerror(e));
    }
  }
  close(fd);
  const double t_populated = now_ms();
  // 2. pin what step 1 did not (no fresh page is faulted in by the driver,
  //    so ranks of a box may register the same image concurrently)
  pool_run([&](uint64_t i) {
    const uint64_t a = i * piece, n = std::min(piece, g.img_bytes - a);
    if (!pinned[i])
      rc[i] = cudaHostRegister(static_cast<uint8_t*>(p) + a, n, cudaHostRegisterMapped | cudaHostRegisterPortable);
  });
  if (getenv("JITC_DEBUG_TIMING"))
    fprintf(stderr,
            "jitc: %s group %u: %.2f GB sized in %.0f ms (%d NUMA slices), populated in %.0f ms, pinned in %.0f ms "
            "(%llu pieces, %d threads)\n",
            who.c_str(), g.id, g.img_bytes / 1e9, t_sized - t_open, placed, t_populated - t_sized,
            now_ms() - t_populated, (unsigned long long)n_pieces, threads);
  g.img_h = (uint8_t*)p;
  g.img_shm = true;
  g.img_reg_piece = n_pieces > 1 ? piece : 0;
  cudaError_t bad = cudaSuccess;
  for (uint64_t i = 0; i < n_pieces; ++i) {
    if (rc[i] == cudaSuccess) g.img_regs.push_back(g.img_h + i * piece);
    else if (bad == cudaSuccess) bad = rc[i];
  }
  if (bad != cudaSuccess) {
    release_image(g);
    return fail(JITC_ENOMEM, who + ": cudaHostRegister: " + cudaGetErrorString(bad));
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
  g.seg_tensor.clear();
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
      g.seg_tensor.push_back((uint32_t)i);
      p += len;
    }
  }
  if (g.n_c > 0xFFFFFFFFull || g.segs.size() > 0xFFFFFFFFull) return fail(JITC_EINVAL, "jitc_register: group too large");
  CU(cudaMalloc(&g.d_segs, std::max<size_t>(g.segs.size(), 1) * sizeof(Seg)));
  if (!g.segs.empty())
    CU(cudaMemcpyAsync(g.d_segs, g.segs.data(), g.segs.size() * sizeof(Seg), cudaMemcpyHostToDevice, c->s_comp));
  CU(cudaMalloc(&g.d_dig, std::max<uint64_t>(g.n_c, 1) * 8));
  CU(cudaMalloc(&g.d_dig2, std::max<uint64_t>(g.n_c, 1) * 8));
  CU(cudaMalloc(&g.d_remote, std::max<size_t>(g.segs.size(), 1) * 8));
  g.h_remote.assign(g.segs.size(), 0);
  CU(cudaStreamSynchronize(c->s_comp));
  st = ensure_h_dig(c, g.n_c);
  if (st) return st;
  // host image: shared /dev/shm file (survives the process) or private pinned
  g.img_bytes = std::max<uint64_t>(align_up(g.L, 4096), 4096);
  if (!c->image_dir.empty()) {
    st = map_shared_image(c, g, "jitc_register");
    if (st) return st;
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

jitc_status jitc_attach_image(jitc_ctx* c, uint32_t group, uint64_t image_bytes) {
  if (!c) return fail(JITC_EINVAL, "jitc_attach_image: null ctx");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || it->second.held)
    return fail(JITC_EINVAL, "jitc_attach_image: group is not a declared (non-held) group");
  if (c->image_dir.empty()) return fail(JITC_EINVAL, "jitc_attach_image: needs an image_dir");
  if (image_bytes == 0 || image_bytes % kAlign) return fail(JITC_EINVAL, "jitc_attach_image: bad image size");
  CU(cudaSetDevice(c->device));
  GroupState& g = it->second;
  if (g.img_h) {
    if (g.L == image_bytes) return JITC_OK;
    release_image(g);
  }
  g.L = image_bytes;
  g.img_bytes = align_up(image_bytes, 4096);
  jitc_status st = map_shared_image(c, g, "jitc_attach_image");
  if (st) return st;
  CU(cudaHostGetDevicePointer((void**)&g.img_d, g.img_h, 0));
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

// One of each NCCL operation the library issues (all-gather of bytes and of
// u64, the barrier's all-reduce, point-to-point send/recv), small and large,
// right after the communicator is created.  The first collective of a process
// does one-time work that waits behind a kernel already running on the device
// -- measured: with no collective before a rank died, the survivors' first
// all-gather after jitc_comm_shrink never started while an emulated hung
// collective spun, and it ran at once when one collective had preceded the
// failure (tools/debug/debug_nccl_shrink.py) -- so it must happen here, in steady
// state, never in the failure path (as with preload_kernels for our own).
static jitc_status warm_comm(jitc_ctx* c) {
  const uint64_t n = (uint64_t)c->comm_n, me = (uint64_t)c->comm_rank;
  const uint64_t big = std::min<uint64_t>(1ull << 20, c->staging_bytes / (2 * n)) / 256 * 256;
  for (uint64_t blk : {(uint64_t)256, big}) {
    if (blk == 0 || n * blk > c->staging_bytes) continue;
    NC(ncclAllGather(c->staging + me * blk, c->staging, blk, ncclUint8, c->comm, c->s_comp));
    NC(ncclAllGather(c->staging + me * blk, c->staging, blk / 8, ncclUint64, c->comm, c->s_comp));
    if (n > 1) {
      NC(ncclGroupStart());
      NC(ncclSend(c->staging, blk, ncclUint8, (int)((me + 1) % n), c->comm, c->s_comp));
      NC(ncclRecv(c->staging + blk, blk, ncclUint8, (int)((me + n - 1) % n), c->comm, c->s_comp));
      NC(ncclGroupEnd());
    }
  }
  NC(ncclAllReduce(c->d_small, c->d_small + 1, 1, ncclUint64, ncclSum, c->comm, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  return JITC_OK;
}

jitc_status jitc_comm_init(jitc_ctx* c, const void* id128, int32_t nranks, int32_t comm_rank, const int32_t* job_ranks) {
  if (!c || !id128 || nranks <= 0 || comm_rank < 0 || comm_rank >= nranks)
    return fail(JITC_EINVAL, "jitc_comm_init: bad argument");
  CU(cudaSetDevice(c->device));
  if (c->comm && c->comm_broken) {  // its collective waits on a dead peer: abort it so the stream drains
    ncclCommAbort(c->comm);
    c->comm = nullptr;
    c->comm_broken = false;
  }
  if (c->comm) {  // retired, not freed: see jitc_ctx::retired_comms
    c->retired_comms.push_back(c->comm);
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
  return warm_comm(c);
}

jitc_status jitc_comm_shrink(jitc_ctx* c, const int32_t* failed, int32_t n_failed) {
  if (!c || !has_comm(c)) return fail(JITC_ESTATE, "jitc_comm_shrink: no communicator");
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
  if (c->ipc) {  // the IPC transport has nothing hung to abort: drop the ranks
    std::vector<int> slot;
    std::vector<uint8_t*> ps;
    for (int i = 0; i < c->comm_n; ++i)
      if (!std::binary_search(excl.begin(), excl.end(), i)) {
        slot.push_back(c->ipc->slot[i]);
        ps.push_back(c->ipc->peer_staging[i]);
      }
    c->ipc->slot = slot;
    c->ipc->peer_staging = ps;
  } else {
    if (c->comm_broken)
      return fail(JITC_ESTATE, "jitc_comm_shrink: a collective of this communicator waits on a dead peer "
                               "(JITC_EPEER); rebuild instead: jitc_comm_destroy (aborts it), then jitc_comm_init "
                               "with a fresh unique id among the survivors");
    // NCCL_SHRINK_ABORT aborts the parent's outstanding operations (a hung
    // collective of this communicator exits); the parent itself is retired,
    // not freed, until jitc_comm_destroy / jitc_destroy (see retired_comms).
    ncclComm_t nc = nullptr;
    if (getenv("JITC_DEBUG_SHRINK")) fprintf(stderr, "jitc: ncclCommShrink ...\n");
    NC(ncclCommShrink(c->comm, excl.data(), (int)excl.size(), &nc, nullptr, NCCL_SHRINK_ABORT));
    if (getenv("JITC_DEBUG_SHRINK")) fprintf(stderr, "jitc: ncclCommShrink done\n");
    c->retired_comms.push_back(c->comm);
    c->comm = nc;
    c->comm_broken = false;
  }
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
  if (c->comm) {
    if (getenv("JITC_DEBUG_SHRINK")) fprintf(stderr, "jitc: comm %s ...\n", c->comm_broken ? "abort" : "destroy");
    c->comm_broken ? ncclCommAbort(c->comm) : ncclCommDestroy(c->comm);  // a broken comm's op never completes
    if (getenv("JITC_DEBUG_SHRINK")) fprintf(stderr, "jitc: comm released\n");
  }
  c->comm_broken = false;
  for (ncclComm_t r : c->retired_comms) ncclCommAbort(r);
  c->retired_comms.clear();
  c->comm = nullptr;
  ipc_destroy(c);
  c->comm_n = 0;
  c->comm_rank = -1;
  c->comm_job.clear();
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
  NvtxRange nvtx_("jitc_fingerprint");
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
  NvtxRange nvtx_("jitc_exchange_records");
  if (!c || !mine || !all_len || len < sizeof(BlobHdr)) return fail(JITC_EINVAL, "jitc_exchange_records: bad argument");
  if (c->ipc) return ipc_exchange(c, mine, len, all, cap, all_len);
  if (!c->comm) {
    *all_len = len;
    if (cap == 0) return JITC_OK;
    if (cap < len || !all) return fail(JITC_EINVAL, "jitc_exchange_records: buffer too small");
    memcpy(all, mine, len);
    return JITC_OK;
  }
  // both calls of the size query run the whole (small: <= 1 MB per rank) gather
  std::vector<std::vector<uint8_t>> parts;
  jitc_status st = gather_bytes(c, mine, len, &parts);
  if (st) return st;
  size_t total = 0;
  for (auto& b : parts) total += b.size();
  *all_len = total;
  if (cap == 0) return JITC_OK;
  if (cap < total || !all) return fail(JITC_EINVAL, "jitc_exchange_records: buffer too small");
  uint8_t* a = static_cast<uint8_t*>(all);
  for (auto& b : parts) {
    memcpy(a, b.data(), b.size());
    a += b.size();
  }
  return JITC_OK;
}

// ------------------------------------------------------------ timeline
jitc_status jitc_timeline_start(jitc_ctx* c, uint32_t max_spans) {
  if (!c || max_spans == 0) return fail(JITC_EINVAL, "jitc_timeline_start: bad argument");
  CU(cudaSetDevice(c->device));
  const size_t need = 2ull * max_spans;
  while (c->tl_ev.size() < need) {
    cudaEvent_t e;
    CU(cudaEventCreate(&e));
    c->tl_ev.push_back(e);
  }
  if (!c->tl_base) CU(cudaEventCreate(&c->tl_base));
  c->tl.clear();
  c->tl_ev_used = 0;
  CU(cudaEventRecord(c->tl_base, c->s_comp));
  c->tl_on = true;
  return JITC_OK;
}

jitc_status jitc_timeline_read(jitc_ctx* c, jitc_span* out, size_t cap, size_t* n) {
  if (!c || !n || (cap && !out)) return fail(JITC_EINVAL, "jitc_timeline_read: bad argument");
  c->tl_on = false;
  *n = c->tl.size();
  if (cap == 0) return JITC_OK;
  CU(cudaSetDevice(c->device));
  CU(cudaStreamSynchronize(c->s_comp));
  CU(cudaStreamSynchronize(c->s_copy));
  for (size_t i = 0; i < c->tl.size() && i < cap; ++i) {
    const jitc_ctx::TlRec& r = c->tl[i];
    float a = 0, b = 0;
    CU(cudaEventElapsedTime(&a, c->tl_base, c->tl_ev[r.e0]));
    CU(cudaEventElapsedTime(&b, c->tl_base, c->tl_ev[r.e1]));
    out[i] = jitc_span{r.kind, r.stream, r.group, r.round, a, b, r.bytes};
  }
  return JITC_OK;
}

// ------------------------------------------------------------ counters
jitc_status jitc_kernel_counters(jitc_ctx* c, int32_t kind, jitc_kernel_counter* out) {
  if (!c || !out || kind < 1 || kind > 4) return fail(JITC_EINVAL, "jitc_kernel_counters: bad argument");
  *out = c->kc[kind];
  return JITC_OK;
}

jitc_status jitc_reset_counters(jitc_ctx* c) {
  if (!c) return fail(JITC_EINVAL, "jitc_reset_counters: null ctx");
  for (auto& k : c->kc) k = jitc_kernel_counter{};
  return JITC_OK;
}

}  // extern "C"
