// libjitc.so capture path: A7 capture (K2 gather-pack + D2H, shard s of k),
// A8 commit (manifest, then the commit record LAST -- PAPER.md:136), and the
// local non-collective capture used by transient recovery and the watchdog
// (PAPER.md:105-108, :173).
#include "jitc_ctx.h"

using namespace jitc;

// ------------------------------------------------------------ capture (K2 + D2H)
// One pipeline over every group of the call: K2 packs round j of the writer's
// shard into staging slot j % S on the compute stream, the copy stream D2Hs
// it, and slot reuse is ordered by the ready/free events.  The round counter
// runs on across groups, so a group's first K2 overlaps the previous group's
// last D2H, and the call's first round is short (kFirstRound) so that the
// copy engine starts within ~0.1 ms instead of after a whole 8 GiB K2
// (pipeline fill).  Every group's re-digests are checked
// against its fingerprint once the pipeline has drained.
constexpr uint64_t kFirstRound = 512ull << 20;

struct CapturePlan {
  GroupState* g;
  uint64_t c0, c1;
};

// Validation and the enqueue of one group's rounds; *j is the call's round counter.
static jitc_status capture_enqueue(jitc_ctx* c, GroupState& g, const GroupSelection& gs, uint64_t v_star,
                                   jitc_stats* stats, uint32_t* j, std::vector<CapturePlan>* todo) {
  if (gs.writers.empty()) {  // dropped OPTIONAL group: no checkpoint of it may survive
    drop_commit(c, g);
    return JITC_OK;
  }
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
  // every writer invalidates the previous commit before it changes any image
  // byte (whichever writer starts first; unlink is idempotent)
  if (g.img_shm) unlink(gpath(c, g.id, ".commit").c_str());
  g.commit_priv.clear();
  g.captured = false;
  todo->push_back({&g, c0, c1});
  if (b1 <= b0) return JITC_OK;
  CU(cudaMemsetAsync(g.d_dig2 + c0, 0, (c1 - c0) * 8, c->s_comp));
  if (c->cfg.flags & JITC_F_ZERO_COPY_D2H) {
    uint32_t lo, hi;
    seg_span(g, b0, b1, &lo, &hi);
    jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, g.img_d, 0), g.d_dig2, b1 - b0);
    if (st) return st;
    if (stats) stats->rounds += 1, stats->d2h_bytes += b1 - b0;
    return JITC_OK;
  }
  const uint64_t R = c->slot_bytes;
  const int nslots = (int)std::min<uint64_t>(jitc_ctx::kSlots, c->staging_bytes / R);
  const uint64_t first = std::max<uint64_t>(g.C, std::min<uint64_t>(R, kFirstRound / g.C * g.C));
  for (uint64_t a = b0; a < b1; ++*j) {
    const uint64_t b = std::min(a + (*j == 0 ? first : R), b1);
    const int sl = (int)(*j % nslots);
    uint8_t* slot = c->staging + sl * R;
    if (*j >= (uint32_t)nslots) CU(cudaStreamWaitEvent(c->s_comp, c->ev_free[sl], 0));
    c->tl_group = g.id, c->tl_round = *j;
    uint32_t lo, hi;
    seg_span(g, a, b, &lo, &hi);
    jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, slot, a), g.d_dig2, b - a);
    if (st) return st;
    CU(cudaEventRecord(c->ev_ready[sl], c->s_comp));
    CU(cudaStreamWaitEvent(c->s_copy, c->ev_ready[sl], 0));
    CU(copy_image(c, g, a, slot, b - a, cudaMemcpyDeviceToHost, c->s_copy));
    CU(cudaEventRecord(c->ev_free[sl], c->s_copy));
    if (stats) stats->rounds += 1;
    a = b;
  }
  if (stats) stats->d2h_bytes += b1 - b0;
  return JITC_OK;
}

// After the pipeline drained: the re-digests of the writer's range must equal
// its fingerprint (else the state changed between K1 and K2: EUNSTABLE).
static jitc_status capture_check(jitc_ctx* c, const CapturePlan& p, uint64_t v_star, jitc_stats* stats) {
  GroupState& g = *p.g;
  if (p.c1 > p.c0) {
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2 + p.c0, (p.c1 - p.c0) * 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
  }
  for (uint64_t ch = p.c0; ch < p.c1; ++ch)
    if (c->h_dig[ch - p.c0] != g.fp[ch])
      return fail(JITC_EUNSTABLE, "jitc_capture: group " + std::to_string(g.id) + " chunk " + std::to_string(ch) +
                                      " changed between fingerprint and capture");
  g.captured = true;
  g.cap_v = v_star;
  if (stats) stats->image_bytes += std::min(p.c1 * g.C, g.L) - std::min(p.c0 * g.C, g.L);
  return JITC_OK;
}

jitc_status jitc_capture(jitc_ctx* c, const void* selection, size_t sel_len, uint32_t group, jitc_stats* stats) {
  NvtxRange nvtx_("jitc_capture");
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
  std::vector<CapturePlan> todo;
  uint32_t j = 0;
  jitc_status st = JITC_OK;
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held || (group != JITC_ALL_GROUPS && g.id != group)) continue;
    const GroupSelection* gs = sel.find(g.id);
    if (!gs) {
      st = fail(JITC_ELAYOUT, "jitc_capture: group missing from selection");
      break;
    }
    st = capture_enqueue(c, g, *gs, sel.v_star, stats, &j, &todo);
    if (st) break;
  }
  // drain the pipeline (also on an error: no copy may still read staging or
  // write the image after the call returns)
  CU(cudaEventRecord(c->ev_join, c->s_copy));
  CU(cudaStreamWaitEvent(c->s_comp, c->ev_join, 0));
  CU(cudaStreamSynchronize(c->s_comp));
  if (st) {
    harvest(c);
    return st;
  }
  for (const CapturePlan& p : todo) {
    st = capture_check(c, p, sel.v_star, stats);
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

// ------------------------------------------------------------ capture with NVLink fan-out
// Executes build_capture_plan (jitc_plan.cc) for one group, round by round:
// the writer's K2 packs and the transfers on the compute stream, the D2H of
// every block this rank moves on the copy stream; slot reuse is ordered by
// the ready/free events.  NCCL: grouped send/recv per round.  IPC: a writer
// posts its round (stream-ordered counter write), a mover copies the block
// out of the writer's staging (peer-to-peer over NVLink) into its own and
// posts "consumed"; a writer refills a slot only after its readers consumed
// the round that last used it, and returns only after they read every round.
static jitc_status fanout_group(jitc_ctx* c, GroupState& g, const GroupSelection& gs, uint64_t v_star,
                                const int32_t* movers, int32_t n_movers, uint64_t gen, jitc_stats* stats) {
  PlanInput in;
  std::string why;
  if (!capture_plan_input(gs, movers, n_movers, c->comm_job.data(), c->comm_n, c->comm_rank, c->staging_bytes,
                          c->slot_bytes, &in, &why))
    return fail(JITC_EINVAL, "jitc_capture_fanout: " + why);
  std::vector<PlanOp> ops;
  uint64_t R = 0;
  uint32_t S = 0, J = 0;
  if (!build_capture_plan(in, &ops, &R, &S, &why, &J)) return fail(JITC_ENOMEM, "jitc_capture_fanout: " + why);
  if (S > (uint32_t)jitc_ctx::kSlots) return fail(JITC_EINVAL, "jitc_capture_fanout: too many slots");
  const int me = c->comm_rank;
  const auto wit = std::find(in.writers.begin(), in.writers.end(), me);
  const bool is_writer = wit != in.writers.end();
  const bool is_mover = std::find(in.movers.begin(), in.movers.end(), me) != in.movers.end();
  if (!is_writer && !is_mover) return JITC_OK;
  uint64_t c0 = 0, c1 = 0;
  if (is_writer) {
    if (!g.held) return fail(JITC_ESTATE, "jitc_capture_fanout: writer does not hold the group");
    if (!g.has_fp) return fail(JITC_ESTATE, "jitc_capture_fanout: group " + std::to_string(g.id) + " not fingerprinted");
    if (gs.layout_hash != g.layout_hash || gs.n_c != g.n_c || gs.image_bytes != g.L)
      return fail(JITC_ELAYOUT, "jitc_capture_fanout: selection layout differs from the registered one");
    if (g.fp_version != v_star || g.fp_root != gs.root || g.fp_phase != JITC_PHASE_CLEAN)
      return fail(JITC_ESTATE, "jitc_capture_fanout: this rank's fingerprint is not the selected candidate");
    shard_range(g.n_c, in.writers.size(), (uint64_t)(wit - in.writers.begin()), &c0, &c1);
    if (g.img_shm) unlink(gpath(c, g.id, ".commit").c_str());  // invalidate before any image byte changes
    g.commit_priv.clear();
    if (c1 > c0) CU(cudaMemsetAsync(g.d_dig2 + c0, 0, (c1 - c0) * 8, c->s_comp));
  }
  bool moves = false;
  for (const PlanOp& op : ops) moves |= op.kind == kOpD2H;
  if (moves && (!g.img_h || !g.img_shm || g.L != gs.image_bytes))
    return fail(JITC_EINVAL, "jitc_capture_fanout: mover has no host image of group " + std::to_string(g.id) +
                                 " (jitc_attach_image)");
  IpcComm* ic = c->ipc.get();
  const uint32_t gsl = ic ? group_slot(c, g.id) : 0;
  const int my_slot = ic ? ic->slot[me] : 0;
  std::vector<int> readers;  // movers that receive from me (IPC slot reuse)
  for (const PlanOp& op : ops)
    if (op.kind == kOpSend && std::find(readers.begin(), readers.end(), op.peer) == readers.end())
      readers.push_back(op.peer);
  bool used[jitc_ctx::kSlots] = {false};
  size_t i = 0;
  uint32_t rounds = 0;
  for (uint32_t j = 0; j < J; ++j) {
    size_t e = i;
    while (e < ops.size() && ops[e].round == j) ++e;
    const uint32_t sl = j % S;
    const uint64_t seq = (gen << 24) | (j + 1);
    c->tl_group = g.id, c->tl_round = j;
    if (e > i) ++rounds;
    if (e > i && used[sl]) CU(cudaStreamWaitEvent(c->s_comp, c->ev_free[sl], 0));
    bool packs = false;
    for (size_t q = i; q < e; ++q) packs |= ops[q].kind == kOpPack;
    // IPC: my readers must have consumed the round that last used this slot
    if (ic && packs && j >= S)
      for (int r : readers) {
        jitc_status st = ipc_wait_peer(*ic, r, &ic->ctl->cap_consumed[ic->slot[r]][gsl], seq - S, "a mover to consume a round");
        if (st) return st;
      }
    // 1. K2: pack my block (re-digest into d_dig2)
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpPack) continue;
      uint32_t lo, hi;
      seg_span(g, op.a, op.b, &lo, &hi);
      jitc_status st = run_segments(c, g, kPack, one_range(lo, hi, c->staging + op.off, op.a), g.d_dig2, op.b - op.a);
      if (st) return st;
    }
    // 2. NVLink: writer -> mover
    if (ic) {
      if (is_writer) {
        jitc_status st = ipc_post(c, &ic->ctl->cap_posted[my_slot][gsl], seq, c->s_comp);
        if (st) return st;
      }
      bool recv = false;
      for (size_t q = i; q < e; ++q) {
        const PlanOp& op = ops[q];
        if (op.kind != kOpRecv) continue;
        recv = true;
        jitc_status st = ipc_wait_peer(*ic, op.peer, &ic->ctl->cap_posted[ic->slot[op.peer]][gsl], seq, "a writer to post a round");
        if (st) return st;
        const size_t tl0 = tl_open(c, c->s_comp);
        CU(cudaMemcpyAsync(c->staging + op.off, ic->peer_staging[op.peer] + op.off, op.bytes, cudaMemcpyDefault,
                           c->s_comp));
        tl_close(c, tl0, c->s_comp, 12, op.bytes);
        if (stats) stats->p2p_bytes += op.bytes;
      }
      if (recv || is_mover) {
        jitc_status st = ipc_post(c, &ic->ctl->cap_consumed[my_slot][gsl], seq, c->s_comp);
        if (st) return st;
      }
    } else {
      bool p2p = false;
      for (size_t q = i; q < e; ++q) p2p |= ops[q].kind == kOpSend || ops[q].kind == kOpRecv;
      if (p2p) {
        NC(ncclGroupStart());
        for (size_t q = i; q < e; ++q) {
          const PlanOp& op = ops[q];
          if (op.kind == kOpSend) NC(ncclSend(c->staging + op.off, op.bytes, ncclUint8, op.peer, c->comm, c->s_comp));
          if (op.kind == kOpRecv) NC(ncclRecv(c->staging + op.off, op.bytes, ncclUint8, op.peer, c->comm, c->s_comp));
          if (stats && (op.kind == kOpSend || op.kind == kOpRecv)) stats->p2p_bytes += op.bytes;
        }
        NC(ncclGroupEnd());
      }
    }
    // 3. D2H of every block of my lane on the copy stream
    if (e > i) {
      CU(cudaEventRecord(c->ev_ready[sl], c->s_comp));
      CU(cudaStreamWaitEvent(c->s_copy, c->ev_ready[sl], 0));
      for (size_t q = i; q < e; ++q) {
        const PlanOp& op = ops[q];
        if (op.kind != kOpD2H) continue;
        CU(copy_image(c, g, op.a, c->staging + op.off, op.bytes, cudaMemcpyDeviceToHost, c->s_copy));
        if (stats) stats->d2h_bytes += op.bytes;
      }
      CU(cudaEventRecord(c->ev_free[sl], c->s_copy));
      used[sl] = true;
    }
    i = e;
  }
  CU(cudaEventRecord(c->ev_join, c->s_copy));
  CU(cudaStreamWaitEvent(c->s_comp, c->ev_join, 0));
  if (is_writer && c1 > c0) CU(cudaMemcpyAsync(c->h_dig, g.d_dig2 + c0, (c1 - c0) * 8, cudaMemcpyDeviceToHost, c->s_comp));
  CU(cudaStreamSynchronize(c->s_comp));
  // IPC: my staging may be reused once this call returns -- wait for my readers
  if (ic && !readers.empty())
    for (int r : readers) {
      jitc_status st = ipc_wait_peer(*ic, r, &ic->ctl->cap_consumed[ic->slot[r]][gsl], (gen << 24) | J, "a mover to finish");
      if (st) return st;
    }
  if (stats) stats->rounds += rounds;
  if (!is_writer) return JITC_OK;
  for (uint64_t ch = c0; ch < c1; ++ch)
    if (c->h_dig[ch - c0] != g.fp[ch])
      return fail(JITC_EUNSTABLE, "jitc_capture_fanout: group " + std::to_string(g.id) + " chunk " +
                                      std::to_string(ch) + " changed between fingerprint and capture");
  g.captured = true;
  g.cap_v = v_star;
  if (stats) stats->image_bytes += std::min(c1 * g.C, g.L) - std::min(c0 * g.C, g.L);
  return JITC_OK;
}

jitc_status jitc_capture_fanout(jitc_ctx* c, const void* selection, size_t sel_len, uint32_t group,
                                const int32_t* movers, int32_t n_movers, jitc_stats* stats) {
  NvtxRange nvtx_("jitc_capture_fanout");
  if (!c || n_movers <= 0 || !movers) return fail(JITC_EINVAL, "jitc_capture_fanout: bad argument");
  if (!has_comm(c)) return fail(JITC_ESTATE, "jitc_capture_fanout: needs a communicator");
  if (c->image_dir.empty()) return fail(JITC_EINVAL, "jitc_capture_fanout: needs a shared image_dir");
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
    return fail(JITC_EINVAL, "jitc_capture_fanout: " + why);
  if (sel.status != JITC_OK) return fail(sel.status, "jitc_capture_fanout: selection status is not OK");
  CU(cudaSetDevice(c->device));
  if (stats) memset(stats, 0, sizeof *stats), stats->first_bad_chunk = -1;
  CallTimer t(c);
  // every comm rank advances the generation once per call (collective)
  const uint64_t gen = c->ipc ? ++c->ipc->cap_gen : 0;
  CU(cudaEventRecord(c->ev_t0, c->s_comp));
  for (const GroupSelection& gs : sel.groups) {  // increasing group id on every rank
    if (group != JITC_ALL_GROUPS && gs.group != group) continue;
    auto it = c->groups.find(gs.group);
    if (it == c->groups.end()) return fail(JITC_ELAYOUT, "jitc_capture_fanout: group unknown to this rank");
    if (gs.writers.empty()) {  // dropped OPTIONAL group
      if (it->second.held) drop_commit(c, it->second);
      continue;
    }
    jitc_status st = fanout_group(c, it->second, gs, sel.v_star, movers, n_movers, gen, stats);
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

// ------------------------------------------------------------ commit (manifest, then commit record)
static std::vector<uint8_t> build_manifest(const GroupState& g, const GroupSelection& gs, uint64_t v_star,
                                           const std::vector<uint8_t>& aux) {
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
  // the user's CPU state (iteration, RNG, data position: PAPER.md:132), opaque
  uint64_t aux_len = aux.size();
  put(&aux_len, 8);
  if (aux_len) put(aux.data(), aux_len);
  pad();
  uint64_t tr = manifest_trailer(b.data(), b.size());
  put(&tr, 8);
  return b;
}

// The local part of jitc_commit: manifest + commit record of every group this
// rank is the lowest writer of; dropped groups lose any older checkpoint.
// Every group this rank writes must be captured at v* before any manifest or
// commit record is written anywhere (the ranks agree on it first), so a
// multi-group commit is all or nothing.
static jitc_status commit_check(jitc_ctx* c, const Selection& sel) {
  for (auto& kv : c->groups) {
    const GroupState& g = kv.second;
    const GroupSelection* gs = g.held ? sel.find(g.id) : nullptr;
    if (!gs || gs->writers.empty()) continue;
    if (std::find(gs->writers.begin(), gs->writers.end(), c->cfg.rank) == gs->writers.end()) continue;
    if (!g.captured || g.cap_v != sel.v_star)
      return fail(JITC_ESTATE, "jitc_commit: group " + std::to_string(g.id) + " not captured at v*");
  }
  return JITC_OK;
}

static jitc_status commit_groups(jitc_ctx* c, const Selection& sel) {
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held) continue;
    const GroupSelection* gs = sel.find(g.id);
    if (!gs) continue;
    if (gs->writers.empty()) {
      drop_commit(c, g);
      g.has_man = false;
      continue;
    }
    bool writer = std::find(gs->writers.begin(), gs->writers.end(), c->cfg.rank) != gs->writers.end();
    if (!writer) continue;
    if (!g.captured || g.cap_v != sel.v_star) return fail(JITC_ESTATE, "jitc_commit: group not captured at v*");
    std::vector<uint8_t> man = build_manifest(g, *gs, sel.v_star, c->aux);
    CommitRec cr{};
    cr.magic = kMagicCommit;
    cr.group = g.id;
    cr.v_star = sel.v_star;
    memcpy(&cr.trailer, man.data() + man.size() - 8, 8);
    cr.manifest_bytes = man.size();
    g.man_d = g.fp;
    g.man_root = g.fp_root;
    g.man_aux = c->aux;
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
  return JITC_OK;
}

jitc_status jitc::commit_impl(jitc_ctx* c, const void* selection, size_t sel_len, bool collective) {
  if (!c) return fail(JITC_EINVAL, "jitc_commit: null ctx");
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
    return fail(JITC_EINVAL, "jitc_commit: " + why);
  if (sel.status != JITC_OK) return fail(sel.status, "jitc_commit: selection status is not OK");
  CU(cudaSetDevice(c->device));
  jitc_status st = collective ? barrier(c) : JITC_OK;  // every writer's capture has returned
  if (st) return st;
  st = commit_check(c, sel);
  if (collective && has_comm(c)) st = agree(c, st);    // nobody writes unless every writer can
  if (st) return st;
  st = commit_groups(c, sel);
  // nobody restores before every commit record exists, and a rank that failed
  // here (ESTATE, EIO) makes every rank fail with it instead of leaving them in
  // a collective it never joins
  return collective && has_comm(c) ? agree(c, st) : st;
}

jitc_status jitc_commit(jitc_ctx* c, const void* selection, size_t sel_len) {
  NvtxRange nvtx_("jitc_commit");
  return commit_impl(c, selection, sel_len, true);
}

jitc_status jitc::local_capture(jitc_ctx* c, jitc_stats* st) {
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

extern "C" {

jitc_status jitc_capture_local(jitc_ctx* c, jitc_stats* stats) {
  if (!c) return fail(JITC_EINVAL, "jitc_capture_local: null ctx");
  jitc_stats st{};
  st.first_bad_chunk = -1;
  jitc_status r = local_capture(c, &st);
  if (stats) *stats = st;
  return r;
}

}  // extern "C"
