// Internal declarations of libjitc.so (B200-native JIT checkpoint capture/restore).
// Formats are specified in DESIGN.md §Formats; the method in PAPER.md §3.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <map>
#include <string>
#include <vector>

#include "jitc.h"

namespace jitc {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;  // JF64 key step (2^64 / golden ratio)
constexpr uint64_t kAlign = 256;                       // image alignment (reading R4)
constexpr uint32_t kMaxSegBytes = 128u << 10;          // K1/K2/K3 work unit (data bytes)
constexpr int kMaxPhaseSlots = 512;
constexpr int kEventPool = 8192;

constexpr uint32_t kMagicRecord = 0x5254494Au;    // "JITR"
constexpr uint32_t kMagicBlob = 0x4254494Au;      // "JITB"
constexpr uint32_t kMagicSelection = 0x5354494Au; // "JITS"
constexpr uint32_t kMagicManifest = 0x4D54494Au;  // "JITM"
constexpr uint32_t kMagicCommit = 0x4354494Au;    // "JITC"

// MurmurHash3 64-bit finalizer (host copy used for layout/topology hashes and
// the root chain; the device copy lives in jitc_kernels.cu).
inline uint64_t mix64(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}
inline uint64_t fold(uint64_t h, uint64_t x) { return mix64(h ^ x); }
uint64_t fnv1a64(const char* s, size_t n);
inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// ------------------------------------------------------------------ segments
// One unit of K1/K2/K3 work: a piece of one tensor that never crosses a
// chunk boundary, followed by the zero padding that ends the tensor's image
// slot (only on the tensor's last piece).  32 bytes, read once per CTA.
struct Seg {
  uint64_t src;         // device address of the tensor bytes of this piece
  uint64_t img_off;     // image byte offset (256-aligned)
  uint32_t data_bytes;  // tensor bytes in this piece
  uint32_t pad_bytes;   // zero bytes after them in the image (< 256)
  uint32_t chunk;       // chunk index within the group
  uint32_t flags;       // kSegAligned16 | kSegAligned8
};
enum : uint32_t { kSegAligned16 = 1u, kSegAligned8 = 2u };
static_assert(sizeof(Seg) == 32, "Seg must be 32 bytes");

enum KernelMode : int { kDigest = 1, kPack = 2, kUnpack = 3, kPull = 4 };  // kPull: F1 fused peer pull

// A launch covers up to kMaxRanges segment ranges; range r reads/writes the
// image bytes through `base[r]`, which corresponds to image offset base_off[r].
constexpr int kMaxRanges = 16;
struct LaunchRanges {
  uint32_t n;
  uint32_t seg_begin[kMaxRanges];
  uint32_t seg_end[kMaxRanges];
  uint32_t prefix[kMaxRanges + 1];  // prefix sums of (end - begin)
  uint64_t base[kMaxRanges];        // device address (staging slot / mapped host image)
  uint64_t base_off[kMaxRanges];
};

// kernels (jitc_kernels.cu)
// d_work: 2 x u32 zero-initialised device counters, private to the stream
// (the kernel resets them when it finishes).
// d_remote (kPull only): per-segment source address in a peer's memory.
// grid: the device's SM count (segment_grid); each mode launches that many
// times its own resident CTAs per SM (jitc_kernels.cu, "CTA shape per mode").
cudaError_t launch_segments(int mode, const Seg* d_segs, const LaunchRanges& r, uint64_t* d_dig, int grid,
                            uint32_t* d_work, cudaStream_t s, const uint64_t* d_remote,
                            unsigned long long* d_span = nullptr);
cudaError_t launch_phase_write(uint64_t* dev_slot, uint64_t value, cudaStream_t s);
int segment_grid(int device);
cudaError_t device_check(int device, std::string* why);

// ------------------------------------------------------------------ formats
#pragma pack(push, 1)
struct RecordHdr {   // 64 B (O4)
  uint32_t magic;
  uint16_t fmt;
  uint8_t policy;
  uint8_t phase;
  int32_t rank;
  uint32_t group;
  uint64_t version;
  uint64_t layout_hash;
  uint64_t n_c;
  uint64_t chunk_bytes;
  uint64_t root;
  uint64_t image_bytes;
};
struct BlobHdr {     // 32 B
  uint32_t magic;
  uint16_t fmt;
  uint16_t n_topo;
  int32_t rank;
  uint32_t n_recs;
  uint64_t blob_bytes;
  uint64_t topo_hash;
};
struct TopoHdr {     // 8 B, then int32 members[n_members], padded to 8
  uint32_t group;
  uint8_t policy;
  uint8_t pad;
  uint16_t n_members;
};
struct SelHdr {      // 48 B
  uint32_t magic;
  uint16_t fmt;
  uint16_t n_groups;
  int32_t status;
  int32_t bad_group;
  uint64_t v_star;
  uint64_t topo_hash;
  uint64_t sel_bytes;
  uint64_t reserved;
};
struct SelGroup {    // 64 B, then i32 writers[k], i32 members[n_members],
                     // i32 (rank, reason)[n_excluded], pad to 8, u64 conflict[n_conflict]
  uint32_t group;
  uint8_t policy;
  uint8_t status;
  uint16_t k;
  uint32_t n_members;
  uint32_t n_excluded;
  uint32_t n_conflict;
  uint32_t reserved;
  uint64_t layout_hash;
  uint64_t chunk_bytes;
  uint64_t n_c;
  uint64_t image_bytes;
  uint64_t root;
};
struct ManifestHdr { // 64 B, then i32 writers[k] (pad 8), tensor table (pad 8), u64 d[n_c],
                     // u64 root, shard table k x ShardEnt, u64 trailer
  uint32_t magic;
  uint16_t fmt;
  uint16_t pad;
  uint32_t group;
  uint32_t n_tensors;
  uint64_t v_star;
  uint64_t layout_hash;
  uint64_t chunk_bytes;
  uint64_t n_c;
  uint64_t image_bytes;
  uint32_t k;
  uint32_t pad2;
};
struct ShardEnt {
  int32_t writer;
  uint32_t pad;
  uint64_t c0, c1;
};
struct CommitRec {   // 32 B, written last
  uint32_t magic;
  uint32_t group;
  uint64_t v_star;
  uint64_t trailer;
  uint64_t manifest_bytes;
};
#pragma pack(pop)
static_assert(sizeof(RecordHdr) == 64, "record header");
static_assert(sizeof(BlobHdr) == 32, "blob header");
static_assert(sizeof(SelHdr) == 48, "selection header");
static_assert(sizeof(SelGroup) == 64, "selection group");
static_assert(sizeof(ManifestHdr) == 64, "manifest header");
static_assert(sizeof(CommitRec) == 32, "commit record");

struct TopoEntry {
  uint32_t group;
  int policy;
  std::vector<int32_t> members;  // sorted
};

struct RecordView {
  RecordHdr h;
  const uint64_t* d;  // n_c digests (points into the caller's buffer)
};

struct BlobView {
  int32_t rank;
  uint64_t topo_hash;
  std::vector<TopoEntry> topo;
  std::vector<RecordView> recs;
};

// Parsed selection (host).
struct GroupSelection {
  uint32_t group = 0;
  int policy = 0;
  int status = 0;
  uint64_t layout_hash = 0, chunk_bytes = 0, n_c = 0, image_bytes = 0, root = 0;
  std::vector<int32_t> writers, members;
  std::vector<std::pair<int32_t, int32_t>> excluded;
  std::vector<uint64_t> conflict;
};
struct Selection {
  int status = 0;
  int bad_group = -1;
  uint64_t v_star = 0, topo_hash = 0;
  std::vector<GroupSelection> groups;
  const GroupSelection* find(uint32_t g) const {
    for (auto& x : groups)
      if (x.group == g) return &x;
    return nullptr;
  }
};

uint64_t topo_hash(const std::vector<TopoEntry>& topo);
std::vector<uint8_t> encode_blob(int32_t rank, const std::vector<TopoEntry>& topo,
                                 const std::vector<std::pair<RecordHdr, const uint64_t*>>& recs);
bool parse_blobs(const uint8_t* p, size_t len, std::vector<BlobView>* out, std::string* why);
jitc_status select_rule(const std::vector<BlobView>& blobs, const std::vector<int32_t>& healthy,
                        Selection* sel);
std::vector<uint8_t> encode_selection(const Selection& s);
bool parse_selection(const uint8_t* p, size_t len, Selection* out, std::string* why);
inline void shard_range(uint64_t n_c, uint64_t k, uint64_t s, uint64_t* c0, uint64_t* c1) {
  *c0 = (s * n_c) / k;
  *c1 = ((s + 1) * n_c) / k;
}
uint64_t root_of(uint64_t layout_hash, const uint64_t* d, uint64_t n_c);

// ------------------------------------------------------------------ restore plan (jitc_plan.cc)
enum : uint8_t { kOpH2D = 1, kOpAllGather = 2, kOpPack = 3, kOpSend = 4, kOpRecv = 5, kOpUnpack = 6,
                 kOpDigestSend = 7, kOpDigestRecv = 8, kOpD2H = 9 };
constexpr uint32_t kMagicPlan = 0x5054494Au;      // "JITP"
#pragma pack(push, 1)
struct PlanOp {      // 48 B
  uint32_t round;
  uint8_t kind;
  uint8_t slot;      // staging slot (double/multi-buffer index)
  uint16_t pad;
  int32_t peer;      // comm rank: H2D/PACK = self, SEND/RECV/DIGEST_* = the other side,
                     // UNPACK = block owner
  uint32_t pad2;
  uint64_t a, b;     // image byte range
  uint64_t off;      // staging byte offset (ALLGATHER: base of the n blocks)
  uint64_t bytes;    // bytes moved (ALLGATHER: block size R per rank)
};
struct PlanHdr {     // 24 B
  uint32_t magic;
  uint32_t n_ops;
  uint64_t round_bytes;
  uint32_t slots;
  uint32_t n_rounds;   // rounds every participant executes (some may carry no operation for this rank)
};
#pragma pack(pop)
static_assert(sizeof(PlanOp) == 48, "plan op");
static_assert(sizeof(PlanHdr) == 24, "plan header");
struct PlanInput {
  int mode = 0;
  uint64_t n_c = 0, chunk_bytes = 0, image_bytes = 0;
  int n = 1, me = 0;                   // communicator size and this rank
  std::vector<int32_t> writers, dests;  // comm ranks (PEER)
  std::vector<int32_t> participants;    // comm ranks of the group's members, sorted (HOST)
  std::vector<int32_t> movers;          // comm ranks that D2H a lane of the image (capture fan-out)
  uint64_t staging_bytes = 0, slot_bytes = 0;
};
bool build_restore_plan(const PlanInput& in, std::vector<PlanOp>* ops, uint64_t* round_bytes, uint32_t* slots,
                        std::string* why, uint32_t* n_rounds = nullptr);
// Capture with NVLink fan-out: writer s packs its O5(n_c, k, s)
// shard; mover q D2Hs lane O5(n_c, m, q) of the image; the part of a shard
// that lies in another rank's lane travels writer -> mover over NVLink.
bool build_capture_plan(const PlanInput& in, std::vector<PlanOp>* ops, uint64_t* round_bytes, uint32_t* slots,
                        std::string* why, uint32_t* n_rounds);
bool capture_plan_input(const GroupSelection& gs, const int32_t* movers, int32_t n_movers,
                        const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank, uint64_t staging_bytes,
                        uint64_t slot_bytes, PlanInput* in, std::string* why);
uint64_t manifest_trailer(const uint8_t* p, size_t n);

// thread-local error text
void set_error(const std::string& s);
const std::string& get_error();

}  // namespace jitc
