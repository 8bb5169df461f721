// ThreadSanitizer stress driver for libjitc_tsan.so (tests/test_tsan.py; SURVEY.md §5 sanitizers).
//
// Runs every thread the library starts -- the IPC heartbeat thread, the
// liveness heartbeat thread (jitc_liveness_init), the watchdog thread and its
// on-hang capture action (local and collective), the parallel pinning pool of
// jitc_register, the durable tier's I/O and copier threads -- while other threads make the calls the header allows
// during a watchdog (jitc_watch_event, jitc_watchdog_wait, jitc_watchdog_failed,
// jitc_watchdog_stop).  Built with -fsanitize=thread (the runtime lives in
// this executable); the library's host code is instrumented too.  Prints
// "tsan-ok" when every iteration fired, captured and committed.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <atomic>
#include <chrono>
#include <string>
#include <thread>
#include <vector>

#include "jitc.h"

#define CHECK(x)                                                                          \
  do {                                                                                    \
    jitc_status s_ = (x);                                                                 \
    if (s_ != JITC_OK) {                                                                  \
      fprintf(stderr, "%s:%d %s -> %d: %s\n", __FILE__, __LINE__, #x, s_, jitc_last_error(nullptr)); \
      exit(1);                                                                            \
    }                                                                                     \
  } while (0)

static std::atomic<int> g_callbacks{0};
static void on_hang(void* user, uint64_t tag, double waited_ms) {
  (void)tag;
  (void)waited_ms;
  static_cast<std::atomic<int>*>(user)->fetch_add(1);
}

int main(int argc, char** argv) {
  if (argc < 2) return 2;
  const std::string dir = argv[1];
  const int iters = argc > 2 ? atoi(argv[2]) : 6;
  const std::string img = dir + "/img", comm = dir + "/comm", live = dir + "/live";
  jitc_config cfg;
  memset(&cfg, 0, sizeof cfg);
  cfg.device = 0;
  cfg.rank = 0;
  cfg.world = 1;
  cfg.chunk_bytes = 4096;
  cfg.staging_bytes = 8u << 20;
  cfg.slot_bytes = 1u << 20;
  cfg.image_dir = img.c_str();
  jitc_ctx* c = nullptr;
  CHECK(jitc_create(&cfg, &c));
  // a ragged table of 24 tensors in one allocation, filled by the K4 generator
  const uint64_t sizes[] = {1, 7, 4096, 4097, 65536, 3 << 20, 12345, 256, 255, 1 << 20, 77, 8,
                            9000, 5 << 20, 33, 4100, 1 << 16, 2, 31, 128 << 10, 640, 3, 100000, 2 << 20};
  const int n = sizeof sizes / sizeof sizes[0];
  uint64_t total = 0;
  for (int i = 0; i < n; ++i) total += (sizes[i] + 511) / 512 * 512;
  uint8_t* base = nullptr;
  if (cudaMalloc(&base, total) != cudaSuccess) return 3;
  std::vector<jitc_tensor> t(n);
  std::vector<std::string> names(n);
  uint64_t off = 0;
  for (int i = 0; i < n; ++i) {
    names[i] = "t" + std::to_string(i);
    t[i].name = names[i].c_str();
    t[i].ptr = base + off;
    t[i].nbytes = sizes[i];
    t[i].dtype = 0;
    CHECK(jitc_gen_fill(t[i].ptr, 0, sizes[i], 99, 0, (uint32_t)i, 1, 254, 0, nullptr));
    off += (sizes[i] + 511) / 512 * 512;
  }
  cudaDeviceSynchronize();
  const int32_t me = 0;
  uint64_t lh = 0, L = 0;
  setenv("JITC_PIN_PIECE_MB", "1", 1);  // the pinning pool registers many pieces on several threads
  CHECK(jitc_register(c, 0, JITC_REQUIRED, &me, 1, t.data(), n, &lh, &L));
  CHECK(jitc_liveness_init(c, live.c_str()));           // liveness heartbeat thread
  CHECK(jitc_comm_init_ipc(c, comm.c_str(), 1, 0, nullptr));  // IPC heartbeat thread
  cudaStream_t hs;
  cudaStreamCreateWithFlags(&hs, cudaStreamNonBlocking);
  int fired_total = 0;
  for (int it = 0; it < iters; ++it) {
    CHECK(jitc_mark(c, 0, 10 + it, JITC_PHASE_CLEAN, nullptr));
    const uint32_t slot = (uint32_t)(it % 8);
    CHECK(jitc_inject_hang(hs, 8, slot));               // an emulated hung collective
    cudaEvent_t ev;
    cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    cudaEventRecord(ev, hs);
    CHECK(jitc_watch_event(c, ev, (uint64_t)it));
    const int32_t action = (it % 2) ? JITC_ON_HANG_COLLECTIVE_CAPTURE : JITC_ON_HANG_LOCAL_CAPTURE;
    CHECK(jitc_watchdog_start(c, 30, action, on_hang, &g_callbacks));
    std::atomic<bool> stop{false};
    std::vector<std::thread> pokers;
    for (int k = 0; k < 3; ++k)
      pokers.emplace_back([&, k] {
        std::vector<cudaEvent_t> mine;
        while (!stop.load()) {
          int32_t ranks[8], nr = 0;
          jitc_watchdog_failed(c, ranks, 8, &nr);
          if (k == 0 && mine.size() < 16) {              // more (completed) events join the watch-list
            cudaEvent_t e2;
            cudaEventCreateWithFlags(&e2, cudaEventDisableTiming);
            cudaEventRecord(e2, nullptr);
            mine.push_back(e2);
            jitc_watch_event(c, e2, 1000 + mine.size());
          }
          int32_t fired = 0;
          if (k == 1) jitc_watchdog_wait(c, 1, &fired, nullptr, nullptr, nullptr, nullptr);
          std::this_thread::sleep_for(std::chrono::microseconds(300));
        }
        for (cudaEvent_t e2 : mine) {  // recorded on the legacy stream: never behind the hang
          cudaEventSynchronize(e2);
          cudaEventDestroy(e2);
        }
      });
    int32_t fired = 0;
    uint64_t tag = 0;
    double waited = 0, action_ms = 0;
    jitc_stats st;
    jitc_status r = jitc_watchdog_wait(c, 60000, &fired, &tag, &waited, &action_ms, &st);
    stop = true;
    for (auto& th : pokers) th.join();
    CHECK(jitc_inject_release(slot));
    cudaStreamSynchronize(hs);
    CHECK(jitc_watchdog_stop(c));
    cudaEventDestroy(ev);
    if (r != JITC_OK || !fired || st.image_bytes != L) {
      fprintf(stderr, "iteration %d: status %d fired %d image_bytes %llu (L %llu): %s\n", it, r, fired,
              (unsigned long long)st.image_bytes, (unsigned long long)L, jitc_last_error(nullptr));
      return 4;
    }
    fired_total += fired;
  }
  // the durable tier's I/O threads and stage-in's bounce-buffer copier threads
  // (argv[3]: a directory on a disk file system, so that O_DIRECT is used)
  if (argc > 3) {
    jitc_stats ds;
    CHECK(jitc_persist(c, 0, argv[3], &ds));
    CHECK(jitc_stage_in(c, 0, argv[3], &ds));
    CHECK(jitc_restore(c, 0, JITC_RESTORE_HOST, nullptr, 0, &ds));
    uint64_t bad = 0;
    CHECK(jitc_verify(c, 0, nullptr, 0, &bad));
  }
  int32_t dead[4], nd = 0;
  CHECK(jitc_comm_dead(c, dead, 4, &nd));
  jitc_destroy(c);
  cudaFree(base);
  printf("tsan-ok iterations=%d fired=%d callbacks=%d dead=%d\n", iters, fired_total, g_callbacks.load(), nd);
  return (fired_total == iters && g_callbacks.load() == iters && nd == 0) ? 0 : 5;
}
