// libjitc.so durable tier (NEXT-4): persist a committed host image to disk and
// stage it back (§6.3).
#include "jitc_ctx.h"

using namespace jitc;

// ------------------------------------------------------------ durable tier (NEXT-4)
// PAPER.md:341, :356 §6.3: JIT and low-frequency periodic checkpoints share
// code and file format; a catastrophic multi-node failure needs a persistent
// copy.  jitc_persist streams a committed host image to a directory on disk
// with parallel O_DIRECT writes (64 MiB pieces), then writes the manifest and,
// LAST, the commit record; jitc_stage_in reads such a copy back
// into the host image (checking the commit record and the layout) so that
// jitc_restore's K3 verification covers it end to end.
constexpr int kDurableThreads = 8;

// Reads go through two reused, page-aligned 64 MiB bounce buffers per thread:
// the memcpy of one piece into the image runs on a helper thread while the
// next piece is read.  O_DIRECT reads straight into a large fresh destination
// (the pinned /dev/shm image) ran at 3.2-3.4 GB/s on the pool's virtio disks
// against 4.7 GB/s into a reused buffer (tools/disk_dest_probe.py,
// profiles/r02e_disk_dest_probe.txt).  Writes go straight from the image
// (they run at the disk's rate).
// bounce: bounce buffers per reading thread (0 = read straight into the image)
static bool rw_parallel(int fd, uint8_t* buf, uint64_t n, bool write, int threads, int bounce) {
  const uint64_t piece = 64ull << 20;
  std::vector<std::thread> th;
  std::vector<int> ok(threads, 1);
  for (int t = 0; t < threads; ++t)
    th.emplace_back([&, t] {
      uint8_t* tmp[2] = {nullptr, nullptr};
      if (bounce && !write)
        for (int i = 0; i < bounce; ++i)
          if (posix_memalign(reinterpret_cast<void**>(&tmp[i]), 4096, piece) != 0) tmp[i] = nullptr;
      const bool bb = tmp[0] != nullptr;
      const bool two = bb && tmp[1] != nullptr;
      std::thread copier;
      int cur = 0;
      for (uint64_t off = (uint64_t)t * piece; off < n && ok[t]; off += (uint64_t)threads * piece) {
        uint64_t len = std::min(piece, n - off), done = 0;
        uint8_t* dst = bb ? tmp[cur] : buf + off;
        while (done < len) {
          ssize_t r = write ? pwrite(fd, buf + off + done, len - done, (off_t)(off + done))
                            : pread(fd, dst + done, len - done, (off_t)(off + done));
          if (r <= 0) {
            if (r < 0 && errno == EINTR) continue;
            ok[t] = 0;
            break;
          }
          done += (uint64_t)r;
        }
        if (!bb || !ok[t]) continue;
        if (!two) {
          memcpy(buf + off, tmp[0], len);
          continue;
        }
        if (copier.joinable()) copier.join();  // the other buffer is free again
        copier = std::thread([=] { memcpy(buf + off, tmp[cur], len); });
        cur ^= 1;
      }
      if (copier.joinable()) copier.join();
      free(tmp[0]);
      free(tmp[1]);
    });
  for (auto& x : th) x.join();
  for (int v : ok)
    if (!v) return false;
  return true;
}

// I/O threads of persist / stage-in (JITC_DURABLE_THREADS overrides; tools/durable_bench.py)
static int durable_threads() {
  const char* e = getenv("JITC_DURABLE_THREADS");
  int n = e ? atoi(e) : kDurableThreads;
  return n < 1 ? 1 : (n > 64 ? 64 : n);
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
  bool ok = rw_parallel(fd, g.img_h, g.img_bytes, true, durable_threads(), 0) && fdatasync(fd) == 0;
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
  const bool direct = (fcntl(fd, F_GETFL) & O_DIRECT) != 0;
  int bounce = 2;  // JITC_DURABLE_BOUNCE = 0 / 1 / 2 (tools/durable_bench.py A/B)
  if (const char* e = getenv("JITC_DURABLE_BOUNCE")) bounce = std::max(0, std::min(2, atoi(e)));
  bool ok = rw_parallel(fd, g.img_h, g.img_bytes, false, durable_threads(), direct ? bounce : 0);
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

