// Host-side formats and pure decision procedures of libjitc.so:
// record blobs (O4), the replica-consistency rule (O6), selection encoding,
// layout (O1) and shard rule (O5).  Formats: DESIGN.md §Formats.
#include <string.h>

#include <algorithm>
#include <map>
#include <set>

#include "jitc_internal.h"

namespace jitc {

static thread_local std::string g_err;
void set_error(const std::string& s) { g_err = s; }
const std::string& get_error() { return g_err; }

uint64_t fnv1a64(const char* s, size_t n) {
  uint64_t h = 0xcbf29ce484222325ull;
  for (size_t i = 0; i < n; ++i) {
    h ^= (uint8_t)s[i];
    h *= 0x100000001b3ull;
  }
  return h;
}

uint64_t root_of(uint64_t layout_hash, const uint64_t* d, uint64_t n_c) {
  uint64_t r = mix64(layout_hash ^ n_c);
  for (uint64_t c = 0; c < n_c; ++c) r = mix64(r ^ d[c]);
  return r;
}

uint64_t manifest_trailer(const uint8_t* p, size_t n) {
  uint64_t h = 0;
  size_t i = 0;
  for (; i + 8 <= n; i += 8) {
    uint64_t w;
    memcpy(&w, p + i, 8);
    h = mix64(h ^ w);
  }
  if (i < n) {
    uint64_t w = 0;
    memcpy(&w, p + i, n - i);
    h = mix64(h ^ w);
  }
  return h;
}

uint64_t topo_hash(const std::vector<TopoEntry>& topo) {
  std::vector<TopoEntry> t = topo;
  std::sort(t.begin(), t.end(), [](const TopoEntry& a, const TopoEntry& b) { return a.group < b.group; });
  uint64_t h = fold(0, t.size());
  for (auto& e : t) {
    h = fold(h, e.group);
    h = fold(h, (uint64_t)e.policy);
    h = fold(h, e.members.size());
    std::vector<int32_t> m = e.members;
    std::sort(m.begin(), m.end());
    for (int32_t r : m) h = fold(h, (uint64_t)(int64_t)r);
  }
  return h;
}

template <class T>
static void put(std::vector<uint8_t>& b, const T& v) {
  const uint8_t* p = reinterpret_cast<const uint8_t*>(&v);
  b.insert(b.end(), p, p + sizeof(T));
}
static void pad8(std::vector<uint8_t>& b) {
  while (b.size() % 8) b.push_back(0);
}

std::vector<uint8_t> encode_blob(int32_t rank, const std::vector<TopoEntry>& topo_in,
                                 const std::vector<std::pair<RecordHdr, const uint64_t*>>& recs) {
  std::vector<TopoEntry> topo = topo_in;
  std::sort(topo.begin(), topo.end(), [](const TopoEntry& a, const TopoEntry& b) { return a.group < b.group; });
  std::vector<uint8_t> b;
  BlobHdr h{};
  h.magic = kMagicBlob;
  h.fmt = 1;
  h.n_topo = (uint16_t)topo.size();
  h.rank = rank;
  h.n_recs = (uint32_t)recs.size();
  h.topo_hash = topo_hash(topo);
  put(b, h);
  for (auto& e : topo) {
    TopoHdr t{e.group, (uint8_t)e.policy, 0, (uint16_t)e.members.size()};
    put(b, t);
    std::vector<int32_t> m = e.members;
    std::sort(m.begin(), m.end());
    for (int32_t r : m) put(b, r);
    pad8(b);
  }
  for (auto& r : recs) {
    put(b, r.first);
    const uint8_t* d = reinterpret_cast<const uint8_t*>(r.second);
    b.insert(b.end(), d, d + 8 * r.first.n_c);
  }
  reinterpret_cast<BlobHdr*>(b.data())->blob_bytes = b.size();
  return b;
}

bool parse_blobs(const uint8_t* p, size_t len, std::vector<BlobView>* out, std::string* why) {
  size_t pos = 0;
  while (pos < len) {
    if (len - pos < sizeof(BlobHdr)) { *why = "truncated blob header"; return false; }
    BlobHdr h;
    memcpy(&h, p + pos, sizeof h);
    if (h.magic != kMagicBlob || h.fmt != 1 || h.blob_bytes < sizeof h || h.blob_bytes > len - pos) {
      *why = "bad blob header at offset " + std::to_string(pos);
      return false;
    }
    BlobView bv;
    bv.rank = h.rank;
    bv.topo_hash = h.topo_hash;
    size_t q = pos + sizeof h, end = pos + h.blob_bytes;
    for (uint32_t i = 0; i < h.n_topo; ++i) {
      if (end - q < sizeof(TopoHdr)) { *why = "truncated topology"; return false; }
      TopoHdr t;
      memcpy(&t, p + q, sizeof t);
      q += sizeof t;
      if (end - q < 4ull * t.n_members) { *why = "truncated members"; return false; }
      TopoEntry e;
      e.group = t.group;
      e.policy = t.policy;
      e.members.resize(t.n_members);
      if (t.n_members) memcpy(e.members.data(), p + q, 4ull * t.n_members);
      q += 4ull * t.n_members;
      q = pos + align_up(q - pos, 8);
      bv.topo.push_back(std::move(e));
    }
    for (uint32_t i = 0; i < h.n_recs; ++i) {
      if (end - q < sizeof(RecordHdr)) { *why = "truncated record"; return false; }
      RecordView rv;
      memcpy(&rv.h, p + q, sizeof rv.h);
      if (rv.h.magic != kMagicRecord || rv.h.fmt != 1) { *why = "bad record magic"; return false; }
      q += sizeof(RecordHdr);
      if ((end - q) / 8 < rv.h.n_c) { *why = "truncated digests"; return false; }
      rv.d = reinterpret_cast<const uint64_t*>(p + q);  // 8-aligned within an 8-aligned buffer
      q += 8 * rv.h.n_c;
      bv.recs.push_back(rv);
    }
    out->push_back(std::move(bv));
    pos = end;
  }
  return true;
}

// ---------------------------------------------------------------- O6 select
// PAPER.md:140 (any replica; discard corrupted), :148 (state i or i+1),
// :176-178 (barrier invariant), :184-188 (optimizer-step failure, hooks),
// :491 (unreplicated ZeRO shards cannot be JIT-recovered).
jitc_status select_rule(const std::vector<BlobView>& blobs_all, const std::vector<int32_t>& healthy_v,
                        Selection* sel) {
  std::set<int32_t> healthy(healthy_v.begin(), healthy_v.end());
  std::vector<const BlobView*> blobs;
  for (auto& b : blobs_all)
    if (healthy.count(b.rank)) blobs.push_back(&b);
  *sel = Selection();
  if (blobs.empty()) return sel->status = JITC_ENOREPLICA;
  for (auto* b : blobs)
    if (b->topo_hash != blobs[0]->topo_hash) return sel->status = JITC_ELAYOUT;
  std::vector<TopoEntry> topo = blobs[0]->topo;
  std::sort(topo.begin(), topo.end(), [](const TopoEntry& a, const TopoEntry& b) { return a.group < b.group; });
  sel->topo_hash = blobs[0]->topo_hash;

  struct Cls {
    uint64_t root;
    std::vector<const RecordView*> recs;
  };
  struct Per {
    std::vector<const RecordView*> R;                    // healthy members' records, by rank
    std::map<uint64_t, std::vector<const RecordView*>> cand;  // version -> winning class
    std::map<uint64_t, std::vector<uint64_t>> conflict;       // version -> differing chunks
  };
  std::map<uint32_t, Per> per;
  bool required_without_record = false;

  for (auto& e : topo) {
    Per& P = per[e.group];
    std::set<int32_t> mem(e.members.begin(), e.members.end());
    for (auto* b : blobs)
      for (auto& r : b->recs)
        if (r.h.group == e.group && mem.count(r.h.rank) && healthy.count(r.h.rank)) P.R.push_back(&r);
    std::sort(P.R.begin(), P.R.end(), [](const RecordView* a, const RecordView* b) { return a->h.rank < b->h.rank; });
    for (auto* r : P.R) {
      const RecordHdr& a = P.R[0]->h;
      if (r->h.layout_hash != a.layout_hash || r->h.chunk_bytes != a.chunk_bytes || r->h.n_c != a.n_c ||
          r->h.image_bytes != a.image_bytes) {
        sel->status = JITC_ELAYOUT;
        sel->bad_group = (int)e.group;
        return JITC_ELAYOUT;
      }
    }
    if (P.R.empty()) {
      if (e.policy == JITC_REQUIRED) required_without_record = true;
      continue;
    }
    // versions present among CLEAN records
    std::map<uint64_t, std::vector<Cls>> byv;
    for (auto* r : P.R) {
      if (r->h.phase != JITC_PHASE_CLEAN) continue;
      auto& cl = byv[r->h.version];
      auto it = std::find_if(cl.begin(), cl.end(), [&](const Cls& c) { return c.root == r->h.root; });
      if (it == cl.end()) cl.push_back(Cls{r->h.root, {r}});
      else it->recs.push_back(r);
    }
    for (auto& kv : byv) {
      auto& cl = kv.second;
      std::stable_sort(cl.begin(), cl.end(), [](const Cls& a, const Cls& b) { return a.recs.size() > b.recs.size(); });
      if (cl.size() > 1 && cl[0].recs.size() == cl[1].recs.size()) {
        std::set<uint64_t> diff;
        size_t top = cl[0].recs.size();
        for (size_t i = 0; i < cl.size() && cl[i].recs.size() == top; ++i)
          for (size_t j = i + 1; j < cl.size() && cl[j].recs.size() == top; ++j) {
            const RecordView* a = cl[i].recs[0];
            const RecordView* b = cl[j].recs[0];
            for (uint64_t c = 0; c < a->h.n_c; ++c)
              if (a->d[c] != b->d[c]) diff.insert(c);
          }
        P.conflict[kv.first] = std::vector<uint64_t>(diff.begin(), diff.end());
      } else {
        P.cand[kv.first] = cl[0].recs;
      }
    }
  }

  // V = intersection over REQUIRED groups of versions with a candidate
  bool any_required = false;
  std::set<uint64_t> V, Vc;
  bool first = true;
  for (auto& e : topo) {
    if (e.policy != JITC_REQUIRED) continue;
    any_required = true;
    std::set<uint64_t> s, sc;
    for (auto& kv : per[e.group].cand) s.insert(kv.first), sc.insert(kv.first);
    for (auto& kv : per[e.group].conflict) sc.insert(kv.first);
    if (first) {
      V = s;
      Vc = sc;
      first = false;
    } else {
      std::set<uint64_t> a, b;
      std::set_intersection(V.begin(), V.end(), s.begin(), s.end(), std::inserter(a, a.end()));
      std::set_intersection(Vc.begin(), Vc.end(), sc.begin(), sc.end(), std::inserter(b, b.end()));
      V.swap(a);
      Vc.swap(b);
    }
  }
  if (!any_required)
    for (auto& kv : per)
      for (auto& c : kv.second.cand) V.insert(c.first);

  auto fill_common = [&](const TopoEntry& e, GroupSelection& g) {
    g.group = e.group;
    g.policy = e.policy;
    g.members = e.members;
    std::sort(g.members.begin(), g.members.end());
    const Per& P = per[e.group];
    if (!P.R.empty()) {
      const RecordHdr& h = P.R[0]->h;
      g.layout_hash = h.layout_hash;
      g.chunk_bytes = h.chunk_bytes;
      g.n_c = h.n_c;
      g.image_bytes = h.image_bytes;
    }
  };

  if (V.empty()) {
    int st;
    if (required_without_record || !any_required) st = JITC_ENOREPLICA;
    else st = Vc.empty() ? JITC_ENOCONSISTENT : JITC_ECONFLICT;
    sel->status = st;
    for (auto& e : topo) {
      GroupSelection g;
      fill_common(e, g);
      const Per& P = per[e.group];
      if (P.R.empty()) g.status = JITC_G_NOREPLICA;
      else if (!P.conflict.empty()) {
        g.status = JITC_G_CONFLICT;
        g.conflict = P.conflict.rbegin()->second;
      } else if (P.cand.empty()) g.status = JITC_G_NOCANDIDATE;
      else g.status = JITC_G_OK;
      sel->groups.push_back(std::move(g));
    }
    return st;
  }

  uint64_t vs = *V.rbegin();
  sel->status = JITC_OK;
  sel->v_star = vs;
  for (auto& e : topo) {
    GroupSelection g;
    fill_common(e, g);
    const Per& P = per[e.group];
    if (P.R.empty()) {
      g.status = JITC_G_DROPPED;   // only OPTIONAL groups reach here
      sel->groups.push_back(std::move(g));
      continue;
    }
    auto it = P.cand.find(vs);
    if (it != P.cand.end()) {
      for (auto* r : it->second) g.writers.push_back(r->h.rank);
      std::sort(g.writers.begin(), g.writers.end());
      g.root = it->second[0]->h.root;
      g.status = it->second.size() == 1 ? JITC_G_UNVERIFIED_SINGLE : JITC_G_OK;
    } else {
      g.status = JITC_G_DROPPED;
      auto ct = P.conflict.find(vs);
      if (ct != P.conflict.end()) g.conflict = ct->second;
    }
    for (auto* r : P.R) {
      if (std::find(g.writers.begin(), g.writers.end(), r->h.rank) != g.writers.end()) continue;
      int why = r->h.phase == JITC_PHASE_DIRTY ? JITC_X_DIRTY
                : r->h.version != vs           ? JITC_X_STALE_VERSION
                                               : JITC_X_MINORITY;
      g.excluded.push_back({r->h.rank, why});
    }
    sel->groups.push_back(std::move(g));
  }
  return JITC_OK;
}

std::vector<uint8_t> encode_selection(const Selection& s) {
  std::vector<uint8_t> b;
  SelHdr h{};
  h.magic = kMagicSelection;
  h.fmt = 1;
  h.n_groups = (uint16_t)s.groups.size();
  h.status = s.status;
  h.bad_group = s.bad_group;
  h.v_star = s.v_star;
  h.topo_hash = s.topo_hash;
  put(b, h);
  for (auto& g : s.groups) {
    SelGroup e{};
    e.group = g.group;
    e.policy = (uint8_t)g.policy;
    e.status = (uint8_t)g.status;
    e.k = (uint16_t)g.writers.size();
    e.n_members = (uint32_t)g.members.size();
    e.n_excluded = (uint32_t)g.excluded.size();
    e.n_conflict = (uint32_t)g.conflict.size();
    e.layout_hash = g.layout_hash;
    e.chunk_bytes = g.chunk_bytes;
    e.n_c = g.n_c;
    e.image_bytes = g.image_bytes;
    e.root = g.root;
    put(b, e);
    for (int32_t w : g.writers) put(b, w);
    for (int32_t m : g.members) put(b, m);
    for (auto& x : g.excluded) {
      put(b, x.first);
      put(b, x.second);
    }
    pad8(b);
    for (uint64_t c : g.conflict) put(b, c);
  }
  reinterpret_cast<SelHdr*>(b.data())->sel_bytes = b.size();
  return b;
}

bool parse_selection(const uint8_t* p, size_t len, Selection* out, std::string* why) {
  if (!p || len < sizeof(SelHdr)) { *why = "selection too short"; return false; }
  SelHdr h;
  memcpy(&h, p, sizeof h);
  if (h.magic != kMagicSelection || h.fmt != 1 || h.sel_bytes > len) { *why = "bad selection header"; return false; }
  *out = Selection();
  out->status = h.status;
  out->bad_group = h.bad_group;
  out->v_star = h.v_star;
  out->topo_hash = h.topo_hash;
  size_t q = sizeof h;
  for (uint16_t i = 0; i < h.n_groups; ++i) {
    if (h.sel_bytes - q < sizeof(SelGroup)) { *why = "truncated selection"; return false; }
    SelGroup e;
    memcpy(&e, p + q, sizeof e);
    q += sizeof e;
    size_t need = 4ull * (e.k + e.n_members + 2ull * e.n_excluded);
    if (h.sel_bytes - q < need) { *why = "truncated selection group"; return false; }
    GroupSelection g;
    g.group = e.group;
    g.policy = e.policy;
    g.status = e.status;
    g.layout_hash = e.layout_hash;
    g.chunk_bytes = e.chunk_bytes;
    g.n_c = e.n_c;
    g.image_bytes = e.image_bytes;
    g.root = e.root;
    const int32_t* w = reinterpret_cast<const int32_t*>(p + q);
    g.writers.assign(w, w + e.k);
    g.members.assign(w + e.k, w + e.k + e.n_members);
    for (uint32_t j = 0; j < e.n_excluded; ++j)
      g.excluded.push_back({w[e.k + e.n_members + 2 * j], w[e.k + e.n_members + 2 * j + 1]});
    q = align_up(q + need, 8);
    if ((h.sel_bytes - q) / 8 < e.n_conflict) { *why = "truncated conflicts"; return false; }
    const uint64_t* c = reinterpret_cast<const uint64_t*>(p + q);
    g.conflict.assign(c, c + e.n_conflict);
    q += 8ull * e.n_conflict;
    out->groups.push_back(std::move(g));
  }
  return true;
}

}  // namespace jitc

using namespace jitc;

extern "C" {

int jitc_abi_version(void) { return JITC_ABI_VERSION; }

jitc_status jitc_select_consistent_replica(const void* blobs, size_t len, const int32_t* healthy,
                                           int32_t n_healthy, void* selection, size_t cap, size_t* sel_len) {
  if (!blobs || !sel_len || n_healthy < 0 || (n_healthy > 0 && !healthy)) {
    set_error("jitc_select_consistent_replica: null argument");
    return JITC_EINVAL;
  }
  std::vector<BlobView> bv;
  std::string why;
  if (!parse_blobs(static_cast<const uint8_t*>(blobs), len, &bv, &why)) {
    set_error("jitc_select_consistent_replica: " + why);
    return JITC_EINVAL;
  }
  Selection s;
  jitc_status st = select_rule(bv, std::vector<int32_t>(healthy, healthy + n_healthy), &s);
  std::vector<uint8_t> enc = encode_selection(s);
  *sel_len = enc.size();
  if (cap == 0) return st;
  if (cap < enc.size() || !selection) {
    set_error("jitc_select_consistent_replica: selection buffer too small");
    return JITC_EINVAL;
  }
  memcpy(selection, enc.data(), enc.size());
  if (st != JITC_OK) set_error("jitc_select_consistent_replica: no consistent replica set (status " +
                               std::to_string(st) + ")");
  return st;
}

jitc_status jitc_layout(const jitc_tensor* t, size_t n, uint64_t chunk_bytes, uint64_t* offsets,
                        uint64_t* layout_hash, uint64_t* image_bytes) {
  if ((n && !t) || !layout_hash || !image_bytes) {
    set_error("jitc_layout: null argument");
    return JITC_EINVAL;
  }
  if (chunk_bytes == 0) chunk_bytes = 1ull << 20;
  if ((chunk_bytes & (chunk_bytes - 1)) || chunk_bytes < 4096 || chunk_bytes > (64ull << 20)) {
    set_error("jitc_layout: chunk_bytes must be a power of two in [4 KiB, 64 MiB]");
    return JITC_EINVAL;
  }
  uint64_t off = 0;
  uint64_t h = fold(fold(0, n), chunk_bytes);
  for (size_t i = 0; i < n; ++i) {
    if (offsets) offsets[i] = off;
    off = align_up(off + t[i].nbytes, kAlign);
    const char* nm = t[i].name ? t[i].name : "";
    h = fold(h, fnv1a64(nm, strlen(nm)));
    h = fold(h, t[i].nbytes);
    h = fold(h, t[i].dtype);
  }
  *layout_hash = h;
  *image_bytes = off;
  return JITC_OK;
}

jitc_status jitc_shard_range(uint64_t n_c, uint32_t k, uint32_t s, uint64_t* c0, uint64_t* c1) {
  if (!c0 || !c1 || k == 0 || s >= k) {
    set_error("jitc_shard_range: need 0 <= s < k");
    return JITC_EINVAL;
  }
  unsigned __int128 a = (unsigned __int128)s * n_c / k, b = (unsigned __int128)(s + 1) * n_c / k;
  *c0 = (uint64_t)a;
  *c1 = (uint64_t)b;
  return JITC_OK;
}

}  // extern "C"
