// libjitc.so restore path: A9-A11 (HOST: H2D slices + NVLink exchange + K3
// unpack+verify; PEER: K2 from the writers' live HBM over NVLink + K3) executed
// from an explicit round plan (jitc_plan.cc), and A12 verify.
#include "jitc_ctx.h"

using namespace jitc;

// ------------------------------------------------------------ restore
struct ManifestView {
  ManifestHdr h;
  std::vector<int32_t> writers;
  std::vector<uint64_t> d;
  uint64_t root = 0;
  std::vector<uint8_t> aux;
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
  if (4ull * h.k > man.size() - q) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  mv->writers.resize(h.k);
  if (h.k) memcpy(mv->writers.data(), man.data() + q, 4ull * h.k);
  q = align_up(q + 4ull * h.k, 8);
  size_t t0 = q;
  for (uint32_t i = 0; i < h.n_tensors; ++i) {
    uint16_t ln;
    if (q + 2 > man.size()) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
    memcpy(&ln, man.data() + q, 2);
    q += 2 + ln + 20;
    if (q > man.size()) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  }
  q = t0 + align_up(q - t0, 8);
  if (q + 8 * (h.n_c + 1) > man.size()) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  mv->d.resize(h.n_c);
  if (h.n_c) memcpy(mv->d.data(), man.data() + q, 8 * h.n_c);
  memcpy(&mv->root, man.data() + q + 8 * h.n_c, 8);
  if (root_of(h.layout_hash, mv->d.data(), h.n_c) != mv->root)
    return fail(JITC_EINCOMPLETE, "jitc_restore: manifest digests do not chain to its root");
  q += 8 * (h.n_c + 1) + sizeof(ShardEnt) * (uint64_t)h.k;   // skip d[], root and the shard table
  uint64_t aux_len = 0;
  if (q + 8 > man.size() - 8) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  memcpy(&aux_len, man.data() + q, 8);
  q += 8;
  if (aux_len > man.size() - 8 - q) return fail(JITC_EINCOMPLETE, "jitc_restore: manifest truncated");
  mv->aux.assign(man.data() + q, man.data() + q + aux_len);
  return JITC_OK;
}

jitc_status jitc::compare_digests(jitc_ctx* c, GroupState& g, const std::vector<uint64_t>& want, jitc_stats* stats) {
  if (g.n_c) {
    CU(cudaMemcpyAsync(c->h_dig, g.d_dig2, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
    if (jitc_status st = nccl_sync(c)) return st;  // NCCL rounds may wait on a dead peer
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
// stream; K2 packs, the exchange and K3 unpacks on the compute stream; slot
// reuse ordered by the ready/free events.  The exchange is NCCL (send/recv or
// in-place all-gather) or, with the IPC transport, nothing at all: K3 reads a
// peer's block straight from the peer's staging once the peer has posted it,
// and every rank posts / consumes every round (counters in shared memory)
// so that senders know when a slot may be refilled.
static jitc_status execute_plan(jitc_ctx* c, GroupState& g, const std::vector<PlanOp>& ops, uint32_t S, uint32_t J,
                                const std::vector<int>& readers, uint64_t gen, jitc_stats* stats) {
  if (S > (uint32_t)jitc_ctx::kSlots) return fail(JITC_EINVAL, "execute_plan: too many slots");
  if (J >= (1u << 24)) return fail(JITC_EINVAL, "execute_plan: too many rounds");
  IpcComm* ic = c->ipc.get();
  const uint32_t gs = ic ? group_slot(c, g.id) : 0;
  const uint64_t base_round = gen << 24;  // IPC counters of this call: (gen << 24) | (round + 1)
  const int my_slot = ic ? ic->slot[c->comm_rank] : 0;
  bool used[jitc_ctx::kSlots] = {false};
  size_t i = 0;
  uint32_t rounds = 0;
  for (uint32_t j = 0; j < J; ++j) {
    while (i < ops.size() && (ops[i].kind == kOpDigestSend || ops[i].kind == kOpDigestRecv)) ++i;
    size_t e = i;
    while (e < ops.size() && ops[e].round == j && ops[e].kind != kOpDigestSend && ops[e].kind != kOpDigestRecv) ++e;
    const uint32_t sl = j % (S ? S : 1);
    const uint64_t seq = base_round + j + 1;  // IPC: this round's counter value
    c->tl_group = g.id, c->tl_round = j;
    bool writes_slot = false;
    for (size_t q = i; q < e; ++q) writes_slot |= ops[q].kind == kOpH2D || ops[q].kind == kOpPack;
    if (e > i) ++rounds;
    // 0. IPC: the readers of my slot must have consumed the round that used it last
    if (ic && writes_slot && j >= S)
      for (int r : readers) {
        jitc_status st = ipc_wait_peer(*ic, r, &ic->ctl->consumed[ic->slot[r]][gs], seq - S, "a peer to consume a round");
        if (st) return st;
      }
    // 1. host -> device on the copy stream
    bool any_h2d = false;
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpH2D) continue;
      if (!any_h2d && used[sl]) CU(cudaStreamWaitEvent(c->s_copy, c->ev_free[sl], 0));
      any_h2d = true;
      CU(copy_image(c, g, op.a, c->staging + op.off, op.bytes, cudaMemcpyHostToDevice, c->s_copy));
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
    // 3. the exchange
    if (ic) {
      jitc_status st = ipc_post(c, &ic->ctl->posted[my_slot][gs], seq, c->s_comp);  // my block is ready
      if (st) return st;
      if (c->debug_exit_after_round && j + 1 >= c->debug_exit_after_round) {
        cudaStreamSynchronize(c->s_comp);
        cudaStreamSynchronize(c->s_copy);
        _exit(17);
      }
      for (size_t q = i; q < e; ++q) {
        const PlanOp& op = ops[q];
        if (op.kind != kOpUnpack || op.peer == c->comm_rank) continue;
        st = ipc_wait_peer(*ic, op.peer, &ic->ctl->posted[ic->slot[op.peer]][gs], seq, "a peer to post a round");
        if (st) return st;
        if (stats) stats->p2p_bytes += op.b - op.a;
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
      for (size_t q = i; q < e; ++q) {
        const PlanOp& op = ops[q];
        if (op.kind != kOpAllGather) continue;
        uint8_t* base = c->staging + op.off;
        NC(ncclAllGather(base + (uint64_t)c->comm_rank * op.bytes, base, op.bytes, ncclUint8, c->comm, c->s_comp));
        if (stats) stats->p2p_bytes += (uint64_t)(c->comm_n - 1) * op.bytes;
      }
    }
    // 4. K3 unpack + verify of every block of the round (<= kMaxRanges per launch);
    //    with IPC a peer's block is read in place from the peer's staging
    LaunchRanges lr{};
    uint64_t bytes = 0;
    for (size_t q = i; q < e; ++q) {
      const PlanOp& op = ops[q];
      if (op.kind != kOpUnpack) continue;
      uint32_t lo, hi;
      seg_span(g, op.a, op.b, &lo, &hi);
      const uint8_t* src = (ic && op.peer != c->comm_rank) ? ic->peer_staging[op.peer] + op.off : c->staging + op.off;
      add_range(lr, lo, hi, src, op.a);
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
    if (ic) {
      jitc_status st = ipc_post(c, &ic->ctl->consumed[my_slot][gs], seq, c->s_comp);  // done reading this round
      if (st) return st;
    }
    if (e > i) {
      CU(cudaEventRecord(c->ev_free[sl], c->s_comp));
      used[sl] = true;
    }
    i = e;
  }
  if (ic) {
    // my staging may be reused as soon as this call returns: wait for its readers
    for (int r : readers) {
      jitc_status st = ipc_wait_peer(*ic, r, &ic->ctl->consumed[ic->slot[r]][gs], base_round + J, "a peer to finish reading");
      if (st) return st;
    }
  }
  if (stats) stats->rounds += rounds;
  return JITC_OK;
}

static jitc_status make_plan(jitc_ctx* c, const PlanInput& in, std::vector<PlanOp>* ops, uint32_t* S, uint32_t* J) {
  uint64_t R;
  std::string why;
  if (!build_restore_plan(in, ops, &R, S, &why, J)) return fail(JITC_ENOMEM, "jitc_restore: " + why);
  return JITC_OK;
}

// HOST mode: this rank (or, with a communicator, every comm rank) loads a
// 1/n slice of the committed image H2D; slices are all-gathered over NVLink
// round by round and every round is unpacked+verified by K3.
static jitc_status restore_host(jitc_ctx* c, GroupState& g, const ManifestView& mv, uint64_t gen, jitc_stats* stats) {
  jitc_status st = JITC_OK;
  if (g.n_c) CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
  const int n = has_comm(c) ? c->comm_n : 1;
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
    in.me = has_comm(c) ? c->comm_rank : 0;
    in.staging_bytes = c->staging_bytes;
    in.slot_bytes = c->slot_bytes;
    if (has_comm(c)) {
      for (int32_t m : g.members) {
        int r = comm_rank_of(c, m);
        if (r >= 0) in.participants.push_back(r);
      }
      std::sort(in.participants.begin(), in.participants.end());
    } else {
      in.participants = {0};
    }
    std::vector<PlanOp> ops;
    uint32_t S = 0, J = 0;
    st = make_plan(c, in, &ops, &S, &J);
    if (st) return st;
    std::vector<int> readers;  // every other member reads my slice
    for (int r : in.participants)
      if (r != in.me) readers.push_back(r);
    if (std::find(in.participants.begin(), in.participants.end(), in.me) == in.participants.end()) readers.clear();
    st = execute_plan(c, g, ops, S, J, readers, gen, stats);
    if (st) return st;
  }
  st = compare_digests(c, g, mv.d, stats);
  if (st) return st;
  g.man_d = mv.d;
  g.man_root = mv.root;
  g.has_man = true;
  g.man_aux = mv.aux;
  if (stats) stats->image_bytes += g.L;
  return JITC_OK;
}

// PEER mode: the selection's writers pack their O5 ranges from live HBM (K2)
// and send them over NVLink to every member that is not a writer; receivers
// unpack+verify (K3) against the writers' digests (broadcast first).
static jitc_status restore_peer(jitc_ctx* c, GroupState& g, const GroupSelection& gs, uint64_t gen, jitc_stats* stats) {
  if (!has_comm(c)) return fail(JITC_ESTATE, "jitc_restore: PEER mode needs a communicator");
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
  uint32_t S = 0, J = 0;
  jitc_status st = make_plan(c, in, &ops, &S, &J);
  if (st) return st;
  if (!is_writer && !is_dst) return JITC_OK;
  if (in.dests.empty()) return JITC_OK;  // every member is a writer: nobody to rebuild (the plan is empty)
  // 1. the lowest writer sends the selected class's digests to every destination
  uint64_t* d_expect = g.d_dig;
  if (is_writer && (!g.has_fp || g.fp_root != gs.root))
    return fail(JITC_ESTATE, "jitc_restore: writer fingerprint differs from the selected class");
  if (is_writer && my_s == 0 && g.n_c)
    CU(cudaMemcpyAsync(d_expect, g.fp.data(), g.n_c * 8, cudaMemcpyHostToDevice, c->s_comp));
  bool any = false;
  for (const PlanOp& op : ops) any |= op.kind == kOpDigestSend || op.kind == kOpDigestRecv;
  if (c->ipc) {
    // IPC: the lowest writer leaves the digests in a file of the communicator
    // directory (per group and hand-off generation); receivers wait for it.
    const uint32_t gsl = group_slot(c, g.id);
    const std::string path = c->ipc->dir + "/dig." + std::to_string(gsl) + "." + std::to_string(gen);
    if (is_writer && my_s == 0 && !write_file_atomic(path, reinterpret_cast<const uint8_t*>(g.fp.data()), 8 * g.n_c))
      return fail(JITC_EIO, "jitc_restore: writing " + path);
    if (is_dst) {
      std::vector<uint8_t> b;
      const double t0 = now_ms();
      while (!read_file(path, &b) || b.size() != 8 * g.n_c) {
        if (ipc_peer_dead(*c->ipc, in.writers[0]))
          return fail(JITC_EPEER, "jitc_restore: the lowest writer died before handing over its digests");
        if (now_ms() - t0 > 600000.0) return fail(JITC_ESTATE, "jitc_restore: no digests from the writers");
        usleep(200);
      }
      if (g.n_c) CU(cudaMemcpyAsync(d_expect, b.data(), g.n_c * 8, cudaMemcpyHostToDevice, c->s_comp));
    }
  } else if (any && g.n_c) {
    NC(ncclGroupStart());
    for (const PlanOp& op : ops) {
      if (op.kind == kOpDigestSend) NC(ncclSend(d_expect, g.n_c, ncclUint64, op.peer, c->comm, c->s_comp));
      if (op.kind == kOpDigestRecv) NC(ncclRecv(d_expect, g.n_c, ncclUint64, op.peer, c->comm, c->s_comp));
    }
    NC(ncclGroupEnd());
  }
  std::vector<uint64_t> want(g.n_c);
  if (is_dst) {
    if (jitc_status st2 = nccl_sync(c)) return st2;  // the digest hand-off may wait on a dead writer
    if (g.n_c) CU(cudaMemcpyAsync(want.data(), d_expect, g.n_c * 8, cudaMemcpyDeviceToHost, c->s_comp));
    CU(cudaStreamSynchronize(c->s_comp));
    if (root_of(g.layout_hash, want.data(), g.n_c) != gs.root)
      return fail(JITC_ECORRUPT, "jitc_restore: received digests do not chain to the selected root");
  } else {
    want = g.fp;
  }
  if (g.n_c) CU(cudaMemsetAsync(g.d_dig2, 0, g.n_c * 8, c->s_comp));
  // 2. data rounds
  std::vector<int> readers;  // a writer's blocks are read by every destination
  if (is_writer) readers = in.dests;
  st = execute_plan(c, g, ops, S, J, readers, gen, stats);
  if (st) return st;
  st = nccl_sync(c);
  if (st) return st;
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

// PEER mode without a selection on some ranks (a fresh replacement took no
// part in the selection): every comm rank contributes the selection it holds
// (or nothing) and all adopt the one of the lowest comm rank that has one --
// the surviving writers computed it from the same all-gathered records, so
// every selection present must be byte-identical (the
// replacement gets the selection over the new communicator).  The writers'
// digests follow in restore_peer's hand-off.
static jitc_status share_selection(jitc_ctx* c, const void* selection, size_t sel_len, std::vector<uint8_t>* out) {
  std::vector<std::vector<uint8_t>> parts;
  jitc_status st = gather_bytes(c, selection, selection ? sel_len : 0, &parts);
  if (st) return st;
  out->clear();
  for (auto& p : parts) {
    if (p.empty()) continue;
    if (out->empty()) {
      *out = p;
    } else if (p != *out) {
      return fail(JITC_EINVAL, "jitc_restore: ranks passed different selections");
    }
  }
  if (out->empty()) return fail(JITC_EINVAL, "jitc_restore: PEER mode needs the selection on at least one rank");
  return JITC_OK;
}

jitc_status jitc_restore(jitc_ctx* c, uint32_t group, int32_t mode, const void* selection, size_t sel_len,
                         jitc_stats* stats) {
  NvtxRange nvtx_(mode == JITC_RESTORE_HOST ? "jitc_restore(HOST)" : "jitc_restore(PEER)");
  if (!c) return fail(JITC_EINVAL, "jitc_restore: null ctx");
  if (mode != JITC_RESTORE_HOST && mode != JITC_RESTORE_PEER) return fail(JITC_EINVAL, "jitc_restore: bad mode");
  CU(cudaSetDevice(c->device));
  if (stats) memset(stats, 0, sizeof *stats), stats->first_bad_chunk = -1;
  // the groups of this call; with the IPC transport each advances its restore
  // generation first, so every participant stays on the same generation even
  // if this call fails part-way on some rank
  std::vector<GroupState*> todo;
  std::map<uint32_t, uint64_t> gen;
  for (auto& kv : c->groups) {
    GroupState& g = kv.second;
    if (!g.held || (group != JITC_ALL_GROUPS && g.id != group)) continue;
    todo.push_back(&g);
    gen[g.id] = c->ipc ? ++c->ipc->restore_gen[group_slot(c, g.id)] : 0;
  }
  // 1. the selection (PEER: shared from the ranks that have it)
  Selection sel;
  bool have_sel = false;
  std::vector<uint8_t> shared;
  jitc_status st = JITC_OK;
  if (mode == JITC_RESTORE_PEER && has_comm(c)) {
    st = share_selection(c, selection, sel_len, &shared);
    if (!st) selection = shared.data(), sel_len = shared.size();
  } else if (mode == JITC_RESTORE_PEER && !selection) {
    st = fail(JITC_EINVAL, "jitc_restore: PEER mode needs the selection");
  }
  if (!st && selection) {
    std::string why;
    if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why))
      st = fail(JITC_EINVAL, "jitc_restore: " + why);
    else if (sel.status != JITC_OK)
      st = fail(sel.status, "jitc_restore: selection status is not OK");
    have_sel = !st;
  }
  // 2. what each group restores from.  HOST: its committed manifest, whose v*
  //    must be the selection's, or -- without a selection -- the one v* of the
  //    REQUIRED groups; an OPTIONAL group committed at another version is
  //    stale (its checkpoint predates a failure that dropped it) and is left
  //    out, as a dropped group is (reading R1).  PEER: the selection's entry.
  std::map<uint32_t, ManifestView> man;
  std::vector<GroupState*> run;
  uint32_t skipped = 0;
  if (!st) {
    for (GroupState* g : todo) {
      const GroupSelection* gs = have_sel ? sel.find(g->id) : nullptr;
      if (have_sel && !gs) {
        st = fail(JITC_ELAYOUT, "jitc_restore: group " + std::to_string(g->id) + " missing from selection");
        break;
      }
      if (gs && gs->writers.empty()) {  // dropped OPTIONAL group: nothing to restore
        ++skipped;
        continue;
      }
      if (mode == JITC_RESTORE_HOST) {
        st = load_manifest(c, *g, &man[g->id]);
        if (st == JITC_EINCOMPLETE && !have_sel && g->policy == JITC_OPTIONAL) {
          st = JITC_OK;  // no checkpoint of this OPTIONAL group: the last selection dropped it
          ++skipped;
          continue;
        }
        if (st) break;
        if (have_sel && man[g->id].h.v_star != sel.v_star) {
          st = fail(JITC_EINCOMPLETE, "jitc_restore: group " + std::to_string(g->id) + " is committed at version " +
                                          std::to_string(man[g->id].h.v_star) + ", the selection's v* is " +
                                          std::to_string(sel.v_star));
          break;
        }
      } else if (gs->layout_hash != g->layout_hash || gs->n_c != g->n_c || gs->image_bytes != g->L) {
        st = fail(JITC_ELAYOUT, "jitc_restore: selection layout differs from the registered one");
        break;
      }
      run.push_back(g);
    }
  }
  if (!st && mode == JITC_RESTORE_HOST && !have_sel) {
    std::vector<uint64_t> req;
    for (GroupState* g : run)
      if (g->policy == JITC_REQUIRED) req.push_back(man[g->id].h.v_star);
    std::sort(req.begin(), req.end());
    req.erase(std::unique(req.begin(), req.end()), req.end());
    if (req.size() > 1) {
      st = fail(JITC_EINCOMPLETE, "jitc_restore: REQUIRED groups are committed at different versions (" +
                                      std::to_string(req.front()) + " .. " + std::to_string(req.back()) + ")");
    } else if (req.size() == 1) {
      std::vector<GroupState*> keep;
      for (GroupState* g : run)
        if (g->policy == JITC_REQUIRED || man[g->id].h.v_star == req[0]) keep.push_back(g);
        else ++skipped;
      run.swap(keep);
    }
  }
  // every rank fails together before any data moves (restore is collective)
  if (has_comm(c)) st = agree(c, st);
  if (st) return st;
  CallTimer t(c);
  CU(cudaEventRecord(c->ev_t0, c->s_comp));
  for (GroupState* g : run) {
    st = mode == JITC_RESTORE_HOST ? restore_host(c, *g, man[g->id], gen[g->id], stats)
                                   : restore_peer(c, *g, *sel.find(g->id), gen[g->id], stats);
    if (st) {
      harvest(c);
      return st;
    }
  }
  CU(cudaEventRecord(c->ev_t1, c->s_comp));
  CU(cudaEventSynchronize(c->ev_t1));
  finish_stats(c, t, stats, true);
  if (stats) stats->groups_done = (uint32_t)run.size(), stats->groups_skipped = skipped;
  return JITC_OK;
}

// ------------------------------------------------------------ user CPU state
jitc_status jitc_set_aux(jitc_ctx* c, const void* data, size_t len) {
  if (!c || (len && !data)) return fail(JITC_EINVAL, "jitc_set_aux: bad argument");
  c->aux.assign(static_cast<const uint8_t*>(data), static_cast<const uint8_t*>(data) + len);
  return JITC_OK;
}

jitc_status jitc_get_aux(jitc_ctx* c, uint32_t group, void* out, size_t cap, size_t* len) {
  if (!c || !len) return fail(JITC_EINVAL, "jitc_get_aux: bad argument");
  auto it = c->groups.find(group);
  if (it == c->groups.end() || !it->second.held || !it->second.has_man)
    return fail(JITC_ESTATE, "jitc_get_aux: no restored / committed manifest for the group");
  const std::vector<uint8_t>& a = it->second.man_aux;
  *len = a.size();
  if (cap == 0) return JITC_OK;
  if (cap < a.size() || (!out && !a.empty())) return fail(JITC_EINVAL, "jitc_get_aux: buffer too small");
  if (!a.empty()) memcpy(out, a.data(), a.size());
  return JITC_OK;
}

// ------------------------------------------------------------ verify (A12)
jitc_status jitc_verify(jitc_ctx* c, uint32_t group, const void* expected, size_t len, uint64_t* first_bad) {
  NvtxRange nvtx_("jitc_verify");
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

