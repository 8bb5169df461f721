// Restore round schedule (pure host code).  jitc_restore executes exactly
// this list of operations; jitc_restore_plan exports it so the multi-rank
// logic can be checked without GPUs (tests/test_multirank_gloo.py).
//
// HOST (every rank restarts; reading R17): the n members of
// the group present in the communicator split the committed image by O5;
// member q loads chunk range O5(n_c, n, q) H2D; every round the members
// exchange R-byte blocks over NVLink -- one in-place NCCL all-gather when
// the group spans the whole communicator, else point-to-point sends/receives
// among the members only -- and K3 unpacks every member's block.
// PEER (only the replacement lost its state): the lowest writer
// sends the digests to every destination; writer s packs its O5(n_c, k, s)
// range from live HBM (K2) and sends it to every member that is not a
// writer; receivers unpack all k blocks (K3).
// Only a group's members take part in its transfers, and every rank handles
// its groups in increasing group id, so per-group point-to-point traffic
// cannot form a cycle between ranks (a canonical order, as with locks).
#include <string.h>

#include <algorithm>

#include "jitc_internal.h"

namespace jitc {

// Round boundaries [off[j], off[j+1]) within every participant's range of
// at most maxlen bytes: R-byte rounds, except that the last one is short
// (kLastRound, capped at R) so that the K3 left after the last transfer is
// short (pipeline drain).  Boundaries are chunk multiples (a
// range starts on a chunk and only the image's end is ragged), so no segment
// straddles two rounds.
constexpr uint64_t kLastRound = 512ull << 20;

static std::vector<uint64_t> round_offsets(uint64_t maxlen, uint64_t R, uint64_t C) {
  std::vector<uint64_t> off{0};
  const uint64_t last = std::max<uint64_t>(C, std::min<uint64_t>(R, kLastRound / C * C));
  const uint64_t body = maxlen > last ? (maxlen - last + C - 1) / C * C : 0;
  for (uint64_t x = 0; x < body; x = std::min(x + R, body)) off.push_back(std::min(x + R, body));
  if (body < maxlen) off.push_back(maxlen);
  return off;
}

static void o5_bytes(uint64_t n_c, uint64_t k, uint64_t s, uint64_t C, uint64_t L, uint64_t* a, uint64_t* b) {
  unsigned __int128 c0 = (unsigned __int128)s * n_c / k, c1 = (unsigned __int128)(s + 1) * n_c / k;
  *a = std::min<uint64_t>((uint64_t)c0 * C, L);
  *b = std::min<uint64_t>((uint64_t)c1 * C, L);
}

bool build_restore_plan(const PlanInput& in, std::vector<PlanOp>* ops, uint64_t* round_bytes, uint32_t* slots,
                        std::string* why, uint32_t* n_rounds) {
  ops->clear();
  *round_bytes = 0;
  *slots = 0;
  uint32_t dummy_rounds;
  if (!n_rounds) n_rounds = &dummy_rounds;
  *n_rounds = 0;
  const uint64_t C = in.chunk_bytes, L = in.image_bytes, n_c = in.n_c;
  if (C == 0 || in.n <= 0 || in.me < 0 || in.me >= in.n) {
    *why = "bad plan input";
    return false;
  }
  if (in.mode == JITC_RESTORE_HOST) {
    // participants: the group's members present in the communicator (every
    // rank restarts and holds its own tensors of the group)
    const std::vector<int32_t>& P = in.participants;
    const uint64_t n = P.size();
    const auto it = std::find(P.begin(), P.end(), in.me);
    if (n == 0 || it == P.end()) return true;  // not a member: nothing to do
    const uint64_t me = (uint64_t)(it - P.begin());
    const bool whole_comm = n == (uint64_t)in.n;  // NCCL all-gather over the whole comm, else p2p
    uint64_t R = std::min<uint64_t>(in.slot_bytes, in.staging_bytes / (2 * n)) / C * C;
    if (R == 0) {
      *why = "staging too small for the restore rounds (need >= 2 * n * C bytes)";
      return false;
    }
    uint64_t S = std::max<uint64_t>(2, std::min<uint64_t>(8, in.staging_bytes / (n * R)));
    *round_bytes = R;
    *slots = (uint32_t)S;
    std::vector<uint64_t> q0(n), q1(n);
    uint64_t maxlen = 0;
    for (uint64_t r = 0; r < n; ++r) {
      o5_bytes(n_c, n, r, C, L, &q0[r], &q1[r]);
      maxlen = std::max(maxlen, q1[r] - q0[r]);
    }
    // Round j covers bytes [off[j], off[j+1]) of every member's slice.  Block
    // q of round j sits at base + q * len_j in the slot (len_j = the round's
    // length, the all-gather's count).
    const std::vector<uint64_t> off = round_offsets(maxlen, R, C);
    const uint64_t J = off.size() - 1;
    *n_rounds = (uint32_t)J;
    for (uint64_t j = 0; j < J; ++j) {
      const uint32_t sl = (uint32_t)(j % S);
      const uint64_t base = sl * n * R, len = off[j + 1] - off[j];
      const uint32_t rj = (uint32_t)j;
      auto range = [&](uint64_t q, uint64_t* a, uint64_t* b) {
        *a = std::min(q1[q], q0[q] + off[j]);
        *b = std::min(q1[q], q0[q] + off[j + 1]);
      };
      uint64_t a, b;
      range(me, &a, &b);
      if (b > a) ops->push_back(PlanOp{rj, kOpH2D, (uint8_t)sl, 0, in.me, 0, a, b, base + me * len, b - a});
      if (n > 1 && whole_comm) {
        ops->push_back(PlanOp{rj, kOpAllGather, (uint8_t)sl, 0, -1, 0, 0, 0, base, len});
      } else if (n > 1) {
        for (uint64_t q = 0; q < n; ++q) {
          if (q == me) continue;
          if (b > a) ops->push_back(PlanOp{rj, kOpSend, (uint8_t)sl, 0, P[q], 0, a, b, base + me * len, b - a});
          uint64_t qa, qb;
          range(q, &qa, &qb);
          if (qb > qa) ops->push_back(PlanOp{rj, kOpRecv, (uint8_t)sl, 0, P[q], 0, qa, qb, base + q * len, qb - qa});
        }
      }
      for (uint64_t q = 0; q < n; ++q) {
        uint64_t qa, qb;
        range(q, &qa, &qb);
        if (qb > qa) ops->push_back(PlanOp{rj, kOpUnpack, (uint8_t)sl, 0, P[q], 0, qa, qb, base + q * len, qb - qa});
      }
    }
    return true;
  }
  if (in.mode != JITC_RESTORE_PEER) {
    *why = "bad mode";
    return false;
  }
  const uint64_t k = in.writers.size();
  if (k == 0) return true;  // dropped group: nothing moves
  for (int32_t w : in.writers)
    if (w < 0 || w >= in.n) {
      *why = "a writer is not in the communicator";
      return false;
    }
  uint64_t R = std::min<uint64_t>(in.slot_bytes, in.staging_bytes / (2 * k)) / C * C;
  if (R == 0) {
    *why = "staging too small for the PEER rounds (need >= 2 * k * C bytes)";
    return false;
  }
  const uint64_t S = 2;
  *round_bytes = R;
  *slots = (uint32_t)S;
  int my_s = -1;
  for (uint64_t s = 0; s < k; ++s)
    if (in.writers[s] == in.me) my_s = (int)s;
  const bool is_dst = std::find(in.dests.begin(), in.dests.end(), in.me) != in.dests.end();
  if (in.dests.empty() || (my_s < 0 && !is_dst)) return true;
  // the lowest writer sends the selected class's digests to every destination
  if (my_s == 0)
    for (int32_t d : in.dests) ops->push_back(PlanOp{0, kOpDigestSend, 0, 0, d, 0, 0, 0, 0, n_c * 8});
  if (is_dst) ops->push_back(PlanOp{0, kOpDigestRecv, 0, 0, in.writers[0], 0, 0, 0, 0, n_c * 8});
  std::vector<uint64_t> q0(k), q1(k);
  uint64_t maxlen = 0;
  for (uint64_t s = 0; s < k; ++s) {
    o5_bytes(n_c, k, s, C, L, &q0[s], &q1[s]);
    maxlen = std::max(maxlen, q1[s] - q0[s]);
  }
  // round j covers bytes [off[j], off[j+1]) of every writer's range
  const std::vector<uint64_t> roff = round_offsets(maxlen, R, C);
  const uint64_t J = roff.size() - 1;
  *n_rounds = (uint32_t)J;
  auto range = [&](uint64_t s, uint64_t j, uint64_t* a, uint64_t* b) {
    *a = std::min(q1[s], q0[s] + roff[j]);
    *b = std::min(q1[s], q0[s] + roff[j + 1]);
  };
  for (uint64_t j = 0; j < J; ++j) {
    const uint32_t sl = (uint32_t)(j % S);
    const uint64_t base = sl * k * R;   // block s of a round sits at base + s*R on every rank
    if (my_s >= 0) {
      uint64_t a, b;
      range((uint64_t)my_s, j, &a, &b);
      if (b <= a) continue;
      const uint64_t off = base + (uint64_t)my_s * R;
      ops->push_back(PlanOp{(uint32_t)j, kOpPack, (uint8_t)sl, 0, in.me, 0, a, b, off, b - a});
      for (int32_t d : in.dests) ops->push_back(PlanOp{(uint32_t)j, kOpSend, (uint8_t)sl, 0, d, 0, a, b, off, b - a});
    } else {
      for (uint64_t s = 0; s < k; ++s) {
        uint64_t a, b;
        range(s, j, &a, &b);
        if (b > a) ops->push_back(PlanOp{(uint32_t)j, kOpRecv, (uint8_t)sl, 0, in.writers[s], 0, a, b, base + s * R, b - a});
      }
      for (uint64_t s = 0; s < k; ++s) {
        uint64_t a, b;
        range(s, j, &a, &b);
        if (b > a) ops->push_back(PlanOp{(uint32_t)j, kOpUnpack, (uint8_t)sl, 0, in.writers[s], 0, a, b, base + s * R, b - a});
      }
    }
  }
  return true;
}

// Capture with NVLink fan-out.  The host
// link, not HBM, bounds capture, and a group with few writers (k = 1 for the
// TP partition that lost a replica, C5) would leave every other GPU's link
// idle.  The image is therefore D2H'd in m lanes, lane q = O5(n_c, m, q) by
// mover q, while writer s still packs (and re-digests) exactly its O5(n_c, k,
// s) shard: the piece shard s ∩ lane q is PACKed by s and, when s is not q,
// SENT over NVLink to q, which RECEIVEs and D2Hs it.  Each writer walks its
// shard in blocks of <= R bytes cut at lane boundaries; round j carries every
// writer's j-th block, at staging offset slot*k*R + s*R on both sides.  With
// m == k and movers == writers this is the plain sharded capture.
bool build_capture_plan(const PlanInput& in, std::vector<PlanOp>* ops, uint64_t* round_bytes, uint32_t* slots,
                        std::string* why, uint32_t* n_rounds) {
  ops->clear();
  *round_bytes = 0;
  *slots = 0;
  *n_rounds = 0;
  const uint64_t C = in.chunk_bytes, L = in.image_bytes, n_c = in.n_c;
  const uint64_t k = in.writers.size(), m = in.movers.size();
  if (C == 0 || in.n <= 0 || in.me < 0 || in.me >= in.n) {
    *why = "bad plan input";
    return false;
  }
  if (k == 0) return true;  // dropped group: nothing is captured
  if (m == 0) {
    *why = "no movers";
    return false;
  }
  for (int32_t w : in.writers)
    if (w < 0 || w >= in.n) {
      *why = "a writer is not in the communicator";
      return false;
    }
  for (size_t i = 0; i < m; ++i) {
    if (in.movers[i] < 0 || in.movers[i] >= in.n) {
      *why = "a mover is not in the communicator";
      return false;
    }
    for (size_t j = 0; j < i; ++j)
      if (in.movers[j] == in.movers[i]) {
        *why = "duplicate mover";
        return false;
      }
  }
  const uint64_t S = 2;
  const uint64_t R = std::min<uint64_t>(in.slot_bytes, in.staging_bytes / (S * k)) / C * C;
  if (R == 0) {
    *why = "staging too small for the capture rounds (need >= 2 * k * C bytes)";
    return false;
  }
  *round_bytes = R;
  *slots = (uint32_t)S;
  struct Block {
    uint64_t a, b;
    uint32_t q;
  };
  // Writer s cuts the part of its shard in each lane into <= R blocks and
  // visits the lanes round-robin (lane q's i-th block, then lane q+1's i-th
  // block, ...), so consecutive rounds go to different movers and every
  // mover's D2H runs at once.  Lane-major order (all of lane q's blocks,
  // then lane q+1's) would keep one or two movers busy at a time: a mover's
  // slot is reused two rounds later and its D2H takes far longer than the
  // K2 + NVLink transfer that feed it (tools/fanout_sim.py).
  std::vector<std::vector<Block>> blocks(k);
  uint64_t J = 0;
  for (uint64_t s = 0; s < k; ++s) {
    uint64_t a, b;
    o5_bytes(n_c, k, s, C, L, &a, &b);
    std::vector<std::vector<Block>> per_lane;
    size_t most = 0;
    for (uint64_t q = 0; q < m; ++q) {
      uint64_t la, lb;
      o5_bytes(n_c, m, q, C, L, &la, &lb);
      const uint64_t x = std::max(a, la), y = std::min(b, lb);
      if (x >= y) continue;
      per_lane.emplace_back();
      for (uint64_t u = x; u < y; u += R) per_lane.back().push_back(Block{u, std::min(u + R, y), (uint32_t)q});
      most = std::max(most, per_lane.back().size());
    }
    for (size_t i = 0; i < most; ++i)
      for (auto& lane : per_lane)
        if (i < lane.size()) blocks[s].push_back(lane[i]);
    J = std::max<uint64_t>(J, blocks[s].size());
  }
  *n_rounds = (uint32_t)J;
  for (uint64_t j = 0; j < J; ++j) {
    const uint32_t sl = (uint32_t)(j % S);
    const uint64_t base = sl * k * R;
    std::vector<PlanOp> pack, xfer, d2h;
    for (uint64_t s = 0; s < k; ++s) {
      if (j >= blocks[s].size()) continue;
      const Block& bl = blocks[s][j];
      const uint64_t off = base + s * R, n = bl.b - bl.a;
      const int32_t w = in.writers[s], q = in.movers[bl.q];
      if (w == in.me) {
        pack.push_back(PlanOp{(uint32_t)j, kOpPack, (uint8_t)sl, 0, in.me, 0, bl.a, bl.b, off, n});
        if (q != in.me) xfer.push_back(PlanOp{(uint32_t)j, kOpSend, (uint8_t)sl, 0, q, 0, bl.a, bl.b, off, n});
      } else if (q == in.me) {
        xfer.push_back(PlanOp{(uint32_t)j, kOpRecv, (uint8_t)sl, 0, w, 0, bl.a, bl.b, off, n});
      }
      if (q == in.me) d2h.push_back(PlanOp{(uint32_t)j, kOpD2H, (uint8_t)sl, 0, w, 0, bl.a, bl.b, off, n});
    }
    ops->insert(ops->end(), pack.begin(), pack.end());
    ops->insert(ops->end(), xfer.begin(), xfer.end());
    ops->insert(ops->end(), d2h.begin(), d2h.end());
  }
  return true;
}

// Plan input of a fan-out capture: writers from the selection (sorted by job
// rank), movers = the caller's job ranks sorted, both mapped to comm ranks.
bool capture_plan_input(const GroupSelection& gs, const int32_t* movers, int32_t n_movers,
                        const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank, uint64_t staging_bytes,
                        uint64_t slot_bytes, PlanInput* in, std::string* why) {
  auto comm_of = [&](int32_t job) {
    for (int i = 0; i < n; ++i)
      if (comm_job_ranks[i] == job) return i;
    return -1;
  };
  in->mode = 0;
  in->n_c = gs.n_c;
  in->chunk_bytes = gs.chunk_bytes;
  in->image_bytes = gs.image_bytes;
  in->n = n;
  in->me = comm_rank;
  in->staging_bytes = staging_bytes;
  in->slot_bytes = slot_bytes;
  in->writers.clear();
  in->movers.clear();
  for (int32_t w : gs.writers) {
    int r = comm_of(w);
    if (r < 0) {
      *why = "writer " + std::to_string(w) + " is not in the communicator";
      return false;
    }
    in->writers.push_back(r);
  }
  std::vector<int32_t> mv(movers, movers + n_movers);
  std::sort(mv.begin(), mv.end());
  for (int32_t q : mv) {
    int r = comm_of(q);
    if (r < 0) {
      *why = "mover " + std::to_string(q) + " is not in the communicator";
      return false;
    }
    in->movers.push_back(r);
  }
  return true;
}

}  // namespace jitc

using namespace jitc;

extern "C" jitc_status jitc_restore_plan(const void* selection, size_t sel_len, uint32_t group, int32_t mode,
                                         const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank,
                                         uint64_t staging_bytes, uint64_t slot_bytes, void* plan, size_t cap,
                                         size_t* len) {
  if (!selection || !comm_job_ranks || !len || n <= 0) {
    set_error("jitc_restore_plan: bad argument");
    return JITC_EINVAL;
  }
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why)) {
    set_error("jitc_restore_plan: " + why);
    return JITC_EINVAL;
  }
  const GroupSelection* gs = sel.find(group);
  if (!gs) {
    set_error("jitc_restore_plan: group not in selection");
    return JITC_EINVAL;
  }
  auto comm_of = [&](int32_t job) {
    for (int i = 0; i < n; ++i)
      if (comm_job_ranks[i] == job) return i;
    return -1;
  };
  PlanInput in;
  in.mode = mode;
  in.n_c = gs->n_c;
  in.chunk_bytes = gs->chunk_bytes;
  in.image_bytes = gs->image_bytes;
  in.n = n;
  in.me = comm_rank;
  in.staging_bytes = staging_bytes;
  in.slot_bytes = slot_bytes;
  for (int32_t w : gs->writers) in.writers.push_back(comm_of(w));
  for (int32_t m : gs->members) {
    int r = comm_of(m);
    if (r >= 0) in.participants.push_back(r);
  }
  std::sort(in.participants.begin(), in.participants.end());
  for (int32_t m : gs->members) {
    if (std::find(gs->writers.begin(), gs->writers.end(), m) != gs->writers.end()) continue;
    int r = comm_of(m);
    if (r >= 0) in.dests.push_back(r);
  }
  std::vector<PlanOp> ops;
  uint64_t R = 0;
  uint32_t S = 0, J = 0;
  // a dropped (OPTIONAL, no candidate) group has nothing to restore: empty plan
  if (!gs->writers.empty() && !build_restore_plan(in, &ops, &R, &S, &why, &J)) {
    set_error("jitc_restore_plan: " + why);
    return JITC_EINVAL;
  }
  PlanHdr h{};
  h.magic = kMagicPlan;
  h.n_ops = (uint32_t)ops.size();
  h.round_bytes = R;
  h.slots = S;
  h.n_rounds = J;
  *len = sizeof h + ops.size() * sizeof(PlanOp);
  if (cap == 0) return JITC_OK;
  if (cap < *len || !plan) {
    set_error("jitc_restore_plan: buffer too small");
    return JITC_EINVAL;
  }
  memcpy(plan, &h, sizeof h);
  if (!ops.empty()) memcpy(static_cast<uint8_t*>(plan) + sizeof h, ops.data(), ops.size() * sizeof(PlanOp));
  return JITC_OK;
}

extern "C" jitc_status jitc_capture_plan(const void* selection, size_t sel_len, uint32_t group, const int32_t* movers,
                                         int32_t n_movers, const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank,
                                         uint64_t staging_bytes, uint64_t slot_bytes, void* plan, size_t cap,
                                         size_t* len) {
  if (!selection || !comm_job_ranks || !len || n <= 0 || n_movers < 0 || (n_movers && !movers)) {
    set_error("jitc_capture_plan: bad argument");
    return JITC_EINVAL;
  }
  Selection sel;
  std::string why;
  if (!parse_selection(static_cast<const uint8_t*>(selection), sel_len, &sel, &why)) {
    set_error("jitc_capture_plan: " + why);
    return JITC_EINVAL;
  }
  const GroupSelection* gs = sel.find(group);
  if (!gs) {
    set_error("jitc_capture_plan: group not in selection");
    return JITC_EINVAL;
  }
  PlanInput in;
  if (!capture_plan_input(*gs, movers, n_movers, comm_job_ranks, n, comm_rank, staging_bytes, slot_bytes, &in, &why)) {
    set_error("jitc_capture_plan: " + why);
    return JITC_EINVAL;
  }
  std::vector<PlanOp> ops;
  uint64_t R = 0;
  uint32_t S = 0, J = 0;
  if (!build_capture_plan(in, &ops, &R, &S, &why, &J)) {
    set_error("jitc_capture_plan: " + why);
    return JITC_EINVAL;
  }
  PlanHdr h{};
  h.magic = kMagicPlan;
  h.n_ops = (uint32_t)ops.size();
  h.round_bytes = R;
  h.slots = S;
  h.n_rounds = J;
  *len = sizeof h + ops.size() * sizeof(PlanOp);
  if (cap == 0) return JITC_OK;
  if (cap < *len || !plan) {
    set_error("jitc_capture_plan: buffer too small");
    return JITC_EINVAL;
  }
  memcpy(plan, &h, sizeof h);
  if (!ops.empty()) memcpy(static_cast<uint8_t*>(plan) + sizeof h, ops.data(), ops.size() * sizeof(PlanOp));
  return JITC_OK;
}
