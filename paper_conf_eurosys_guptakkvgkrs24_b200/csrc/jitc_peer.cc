// F1 fusion: intra-node PEER restore by direct peer-memory
// reads.  A writer publishes CUDA IPC handles of the allocations holding its
// registered tensors plus its fingerprint digests (jitc_peer_export); the
// replacement maps them and one kernel (K5, seg_kernel<kPull>) reads every
// writer's live tensors over NVLink, scatters the bytes into its own tensors
// and re-digests them in the same pass -- the transfer and the verification
// are one kernel, with no staging buffer, no writer-side kernel and no NCCL.
// The B200 analogue of "copy the state from a data-parallel replica that is
// waiting at the all-reduce".
#include <cuda.h>

#include "jitc_ctx.h"

using namespace jitc;

namespace {

constexpr uint32_t kMagicPeer = 0x5854494Au;  // "JITX"

#pragma pack(push, 1)
struct PeerHdr {      // 56 B, then u64 d[n_c], PeerAlloc[n_alloc], PeerTensor[n_tensors]
  uint32_t magic;
  uint32_t group;
  int32_t rank;
  uint32_t n_alloc;
  uint64_t layout_hash;
  uint64_t n_c;
  uint64_t root;
  uint64_t version;
  uint32_t n_tensors;
  uint32_t phase;
};
struct PeerAlloc {    // 80 B
  cudaIpcMemHandle_t handle;
  uint64_t base;
  uint64_t size;
};
struct PeerTensor {   // 16 B
  uint32_t alloc;     // UINT32_MAX for a zero-byte tensor
  uint32_t pad;
  uint64_t offset;    // byte offset of the tensor inside its allocation
};
#pragma pack(pop)
static_assert(sizeof(PeerHdr) == 56 && sizeof(PeerAlloc) == 80 && sizeof(PeerTensor) == 16, "peer formats");

typedef CUresult (*PFN_getAddressRange)(CUdeviceptr*, size_t*, CUdeviceptr);

PFN_getAddressRange address_range_fn() {
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

std::string peer_path(const jitc_ctx* c, uint32_t g, int32_t rank) {
  return c->image_dir + "/g" + std::to_string(g) + ".peer." + std::to_string(rank);
}

}  // namespace

extern "C" {

jitc_status jitc_peer_export(jitc_ctx* c, uint32_t group) {
  if (!c) return fail(JITC_EINVAL, "jitc_peer_export: null ctx");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_peer_export: group not registered");
  GroupState& g = it->second;
  if (c->image_dir.empty()) return fail(JITC_EINVAL, "jitc_peer_export: needs an image_dir shared by the node's ranks");
  if (!g.has_fp) return fail(JITC_ESTATE, "jitc_peer_export: fingerprint the group first");
  PFN_getAddressRange range = address_range_fn();
  if (!range) return fail(JITC_ECUDA, "jitc_peer_export: cuMemGetAddressRange unavailable");
  CU(cudaSetDevice(c->device));
  std::vector<PeerAlloc> allocs;
  std::vector<PeerTensor> tens(g.t.size());
  for (size_t i = 0; i < g.t.size(); ++i) {
    tens[i] = PeerTensor{0xFFFFFFFFu, 0, 0};
    if (!g.t[i].nbytes) continue;
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)g.t[i].ptr) != CUDA_SUCCESS)
      return fail(JITC_ECUDA, "jitc_peer_export: tensor " + g.names[i] + " is not device memory");
    uint32_t a = 0;
    while (a < allocs.size() && allocs[a].base != (uint64_t)base) ++a;
    if (a == allocs.size()) {
      PeerAlloc pa{};
      cudaError_t e = cudaIpcGetMemHandle(&pa.handle, (void*)base);
      if (e != cudaSuccess)
        return fail(JITC_ECUDA, std::string("jitc_peer_export: cudaIpcGetMemHandle (VMM / expandable-segment "
                                            "allocations are not IPC-exportable): ") + cudaGetErrorString(e));
      pa.base = (uint64_t)base;
      pa.size = size;
      allocs.push_back(pa);
    }
    tens[i].alloc = a;
    tens[i].offset = (uint64_t)g.t[i].ptr - (uint64_t)base;
  }
  PeerHdr h{};
  h.magic = kMagicPeer;
  h.group = g.id;
  h.rank = c->cfg.rank;
  h.n_alloc = (uint32_t)allocs.size();
  h.layout_hash = g.layout_hash;
  h.n_c = g.n_c;
  h.root = g.fp_root;
  h.version = g.fp_version;
  h.n_tensors = (uint32_t)tens.size();
  h.phase = (uint32_t)g.fp_phase;
  std::vector<uint8_t> b(sizeof h + 8 * g.n_c + sizeof(PeerAlloc) * allocs.size() + sizeof(PeerTensor) * tens.size());
  uint8_t* p = b.data();
  memcpy(p, &h, sizeof h);
  p += sizeof h;
  if (g.n_c) memcpy(p, g.fp.data(), 8 * g.n_c);
  p += 8 * g.n_c;
  if (!allocs.empty()) memcpy(p, allocs.data(), sizeof(PeerAlloc) * allocs.size());
  p += sizeof(PeerAlloc) * allocs.size();
  if (!tens.empty()) memcpy(p, tens.data(), sizeof(PeerTensor) * tens.size());
  mkdir(c->image_dir.c_str(), 0700);
  if (!write_file_atomic(peer_path(c, g.id, c->cfg.rank), b.data(), b.size()))
    return fail(JITC_EIO, "jitc_peer_export: writing " + peer_path(c, g.id, c->cfg.rank));
  return JITC_OK;
}

jitc_status jitc_restore_pull(jitc_ctx* c, uint32_t group, const void* selection, size_t sel_len, jitc_stats* stats) {
  NvtxRange nvtx_("jitc_restore_pull");
  if (!c) return fail(JITC_EINVAL, "jitc_restore_pull: null ctx");
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
    return fail(JITC_EINVAL, "jitc_restore_pull: " + why);
  if (sel.status != JITC_OK) return fail(sel.status, "jitc_restore_pull: selection status is not OK");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held) return fail(JITC_EINVAL, "jitc_restore_pull: group not registered");
  GroupState& g = it->second;
  const GroupSelection* gs = sel.find(group);
  if (!gs) return fail(JITC_ELAYOUT, "jitc_restore_pull: group missing from selection");
  if (gs->layout_hash != g.layout_hash || gs->n_c != g.n_c || gs->image_bytes != g.L)
    return fail(JITC_ELAYOUT, "jitc_restore_pull: selection layout differs from the registered one");
  if (gs->writers.empty()) return JITC_OK;  // dropped OPTIONAL group
  if (std::find(gs->writers.begin(), gs->writers.end(), c->cfg.rank) != gs->writers.end())
    return JITC_OK;  // a writer already holds the selected state
  CU(cudaSetDevice(c->device));
  if (stats) memset(stats, 0, sizeof *stats), stats->first_bad_chunk = -1;
  CallTimer t(c);
  const uint64_t k = gs->writers.size();
  std::vector<void*> opened;
  auto close_all = [&]() {
    for (void* p : opened) cudaIpcCloseMemHandle(p);
    opened.clear();
  };
  std::vector<uint64_t> want;
  for (uint64_t s = 0; s < k; ++s) {
    std::vector<uint8_t> b;
    std::string path = peer_path(c, group, gs->writers[s]);
    if (!read_file(path, &b) || b.size() < sizeof(PeerHdr)) {
      close_all();
      return fail(JITC_EINCOMPLETE, "jitc_restore_pull: writer has not exported: " + path);
    }
    PeerHdr h;
    memcpy(&h, b.data(), sizeof h);
    size_t need = sizeof h + 8 * h.n_c + sizeof(PeerAlloc) * (size_t)h.n_alloc + sizeof(PeerTensor) * (size_t)h.n_tensors;
    if (h.magic != kMagicPeer || h.group != group || b.size() != need || h.n_tensors != g.t.size()) {
      close_all();
      return fail(JITC_EINCOMPLETE, "jitc_restore_pull: malformed export " + path);
    }
    if (h.layout_hash != g.layout_hash || h.n_c != g.n_c) {
      close_all();
      return fail(JITC_ELAYOUT, "jitc_restore_pull: writer layout differs");
    }
    const uint64_t* d = reinterpret_cast<const uint64_t*>(b.data() + sizeof h);
    if (h.root != gs->root || root_of(h.layout_hash, d, h.n_c) != h.root || h.version != sel.v_star ||
        h.phase != JITC_PHASE_CLEAN) {
      close_all();
      return fail(JITC_ESTATE, "jitc_restore_pull: writer " + std::to_string(gs->writers[s]) +
                                   " exported a state other than the selected class");
    }
    if (s == 0) want.assign(d, d + h.n_c);
    const PeerAlloc* pa = reinterpret_cast<const PeerAlloc*>(b.data() + sizeof h + 8 * h.n_c);
    const PeerTensor* pt = reinterpret_cast<const PeerTensor*>(pa + h.n_alloc);
    std::vector<uint64_t> mapped(h.n_alloc, 0);
    for (uint32_t a = 0; a < h.n_alloc; ++a) {
      void* p = nullptr;
      cudaError_t e = cudaIpcOpenMemHandle(&p, pa[a].handle, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) {
        close_all();
        return fail(JITC_ECUDA, std::string("jitc_restore_pull: cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
      }
      opened.push_back(p);
      mapped[a] = (uint64_t)p;
    }
    uint64_t c0, c1;
    shard_range(g.n_c, k, s, &c0, &c1);
    for (size_t i = 0; i < g.segs.size(); ++i) {
      const Seg& sg = g.segs[i];
      if (sg.chunk < c0 || sg.chunk >= c1) continue;
      const uint32_t ti = g.seg_tensor[i];
      if (pt[ti].alloc >= h.n_alloc) {
        close_all();
        return fail(JITC_EINCOMPLETE, "jitc_restore_pull: export lacks tensor " + g.names[ti]);
      }
      g.h_remote[i] = mapped[pt[ti].alloc] + pt[ti].offset + (sg.src - (uint64_t)g.t[ti].ptr);
    }
  }
  CU(cudaEventRecord(c->ev_t0, c->s_comp));
  if (!g.segs.empty())
    CU(cudaMemcpyAsync(g.d_remote, g.h_remote.data(), g.segs.size() * 8, cudaMemcpyHostToDevice, c->s_comp));
  if (g.n_c) CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
  jitc_status st = run_segments(c, g, kPull, one_range(0, (uint32_t)g.segs.size(), nullptr, 0), g.d_dig2, g.L,
                                g.d_remote);
  if (st) {
    cudaStreamSynchronize(c->s_comp);
    close_all();
    return st;
  }
  CU(cudaEventRecord(c->ev_t1, c->s_comp));
  st = compare_digests(c, g, want, stats);  // synchronises the stream
  close_all();
  finish_stats(c, t, stats, true);
  if (st) return st;
  g.man_d = want;
  g.man_root = gs->root;
  g.has_man = true;
  if (stats) {
    stats->image_bytes = g.L;
    stats->p2p_bytes = g.L;
    stats->rounds = 1;
  }
  return JITC_OK;
}

}  // extern "C"
