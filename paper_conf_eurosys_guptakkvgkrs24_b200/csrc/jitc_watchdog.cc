// libjitc.so hang detection (NEXT-1): event watch-list + native watchdog
// thread (§3.1-3.2).
#include "jitc_ctx.h"

using namespace jitc;

// ------------------------------------------------------------ watchdog (NEXT-1)
// PAPER.md:124-126 §3.1: events recorded after collectives are put on a
// watch-list; a watchdog thread polls them with cudaEventQuery and treats
// one that stays incomplete past a timeout as a hang of the collective.
// PAPER.md:132-134 §3.2: the checkpoint is then taken on a side stream by the
// watchdog thread itself -- here entirely in C++ (no Python callback, so the
// GIL cannot block it) on the library's non-blocking streams.

// The paper's user-level protocol run by the survivors themselves
// (PAPER.md:105-116): peers whose heartbeat went stale are dead (IPC control
// block, or the liveness table of jitc_liveness_init for NCCL); drop them
// from the communicator (ncclCommShrink(ABORT), which also aborts the hung
// collective, or an IPC shrink), then fingerprint -> exchange -> select ->
// sharded capture -> commit among the survivors, all on this thread.
static jitc_status collective_capture(jitc_ctx* c, jitc_stats* st) {
  if (!has_comm(c)) return local_capture(c, st);
  if (!c->ipc && !c->live)
    return fail(JITC_ESTATE, "collective capture needs failure localisation: use the IPC transport, "
                             "jitc_liveness_init (NCCL transport), or JITC_ON_HANG_NOTIFY and shrink from the harness");
  std::vector<int32_t> failed = stale_ranks(c, c->timeout_ms);
  jitc_status r = JITC_OK;
  if (!failed.empty()) {
    r = jitc_comm_shrink(c, failed.data(), (int32_t)failed.size());
    if (r) return r;
  }
  {
    std::lock_guard<std::mutex> lk(c->wmu);  // read by jitc_watchdog_failed on other threads
    c->fired_failed = failed;
  }
  size_t len = 0;
  r = jitc_fingerprint(c, JITC_ALL_GROUPS, nullptr, 0, &len);
  if (r) return r;
  std::vector<uint8_t> blob(len);
  r = jitc_fingerprint(c, JITC_ALL_GROUPS, blob.data(), blob.size(), &len);
  if (r) return r;
  size_t all_len = 0;
  r = jitc_exchange_records(c, blob.data(), len, nullptr, 0, &all_len);
  if (r) return r;
  std::vector<uint8_t> all(all_len);
  r = jitc_exchange_records(c, blob.data(), len, all.data(), all.size(), &all_len);
  if (r) return r;
  size_t sl = 0;
  jitc_select_consistent_replica(all.data(), all_len, c->comm_job.data(), (int32_t)c->comm_job.size(), nullptr, 0,
                                 &sl);
  std::vector<uint8_t> sel(sl);
  r = jitc_select_consistent_replica(all.data(), all_len, c->comm_job.data(), (int32_t)c->comm_job.size(),
                                     sel.data(), sel.size(), &sl);
  if (r) return r;
  r = jitc_capture(c, sel.data(), sl, JITC_ALL_GROUPS, st);
  if (r) return r;
  return commit_impl(c, sel.data(), sl, true);
}

static void watchdog_loop(jitc_ctx* c) {
  cudaSetDevice(c->device);
  const double t0 = now_ms();
  for (;;) {
    std::unique_lock<std::mutex> lk(c->wmu);
    if (!c->wrun) return;
    double now = now_ms();
    bool hang = false;
    for (size_t i = 0; i < c->watches.size();) {
      cudaError_t q = cudaEventQuery(c->watches[i].ev);
      if (q == cudaSuccess) {
        c->watches.erase(c->watches.begin() + i);
        continue;
      }
      if (q != cudaErrorNotReady) cudaGetLastError();
      if (now - c->watches[i].t_added >= c->timeout_ms) {
        hang = true;
        c->fired_tag = c->watches[i].tag;
        c->waited_ms = now - c->watches[i].t_added;
        break;
      }
      ++i;
    }
    if (hang) {
      c->fired = true;
      c->detect_ms = now - t0;
      lk.unlock();
      double ta = now_ms();
      if (c->action == JITC_ON_HANG_LOCAL_CAPTURE || c->action == JITC_ON_HANG_COLLECTIVE_CAPTURE) {
        jitc_stats st{};
        jitc_status r = c->action == JITC_ON_HANG_LOCAL_CAPTURE ? local_capture(c, &st) : collective_capture(c, &st);
        // the error text is thread-local: hand this thread's to jitc_watchdog_wait
        const std::string err = r ? get_error() : std::string();
        lk.lock();
        c->action_status = r;
        c->action_stats = st;
        c->action_error = err;
        lk.unlock();
      }
      if (c->hang_fn) c->hang_fn(c->hang_user, c->fired_tag, c->waited_ms);
      lk.lock();
      c->action_ms = now_ms() - ta;
      c->action_done = true;
      c->wrun = false;
      c->wcv.notify_all();
      return;
    }
    c->wcv.wait_for(lk, std::chrono::microseconds(200));
  }
}

static void stop_thread(jitc_ctx* c) {
  {
    std::lock_guard<std::mutex> lk(c->wmu);
    c->wrun = false;
    c->wcv.notify_all();
  }
  if (c->wthread.joinable()) c->wthread.join();
}


jitc_status jitc_watch_event(jitc_ctx* c, void* event, uint64_t tag) {
  if (!c || !event) return fail(JITC_EINVAL, "jitc_watch_event: null argument");
  std::lock_guard<std::mutex> lk(c->wmu);
  c->watches.push_back({(cudaEvent_t)event, tag, now_ms()});
  return JITC_OK;
}

jitc_status jitc_watchdog_start(jitc_ctx* c, uint32_t timeout_ms, int32_t action, jitc_hang_fn fn, void* user) {
  if (!c) return fail(JITC_EINVAL, "jitc_watchdog_start: null ctx");
  if (action != JITC_ON_HANG_NOTIFY && action != JITC_ON_HANG_LOCAL_CAPTURE &&
      action != JITC_ON_HANG_COLLECTIVE_CAPTURE)
    return fail(JITC_EINVAL, "jitc_watchdog_start: bad action");
  stop_thread(c);  // a previous watchdog; the watch-list is kept
  std::lock_guard<std::mutex> lk(c->wmu);
  c->timeout_ms = timeout_ms;
  c->action = action;
  c->hang_fn = fn;
  c->hang_user = user;
  c->fired = c->action_done = false;
  c->action_status = JITC_OK;
  c->action_error.clear();
  c->fired_failed.clear();
  c->action_stats = jitc_stats{};
  c->action_stats.first_bad_chunk = -1;
  c->wrun = true;
  c->wthread = std::thread(watchdog_loop, c);
  return JITC_OK;
}

jitc_status jitc_watchdog_wait(jitc_ctx* c, uint32_t max_ms, int32_t* fired, uint64_t* tag, double* waited_ms,
                               double* action_ms, jitc_stats* action_stats) {
  if (!c || !fired) return fail(JITC_EINVAL, "jitc_watchdog_wait: null argument");
  std::unique_lock<std::mutex> lk(c->wmu);
  c->wcv.wait_for(lk, std::chrono::milliseconds(max_ms), [c] { return c->action_done; });
  *fired = c->action_done ? 1 : 0;
  if (tag) *tag = c->fired_tag;
  if (waited_ms) *waited_ms = c->waited_ms;
  if (action_ms) *action_ms = c->action_ms;
  if (action_stats) *action_stats = c->action_stats;
  jitc_status st = c->action_done ? c->action_status : JITC_OK;
  if (st) set_error("jitc_watchdog_wait: the on-hang capture failed with status " + std::to_string(st) + ": " +
                    c->action_error);
  return st;
}

jitc_status jitc_watchdog_failed(jitc_ctx* c, int32_t* ranks, int32_t cap, int32_t* n) {
  if (!c || !n) return fail(JITC_EINVAL, "jitc_watchdog_failed: null argument");
  std::lock_guard<std::mutex> lk(c->wmu);
  *n = (int32_t)c->fired_failed.size();
  for (int32_t i = 0; i < *n && i < cap && ranks; ++i) ranks[i] = c->fired_failed[i];
  return JITC_OK;
}

jitc_status jitc_watchdog_stop(jitc_ctx* c) {
  if (!c) return fail(JITC_EINVAL, "jitc_watchdog_stop: null ctx");
  stop_thread(c);
  std::lock_guard<std::mutex> lk(c->wmu);
  c->watches.clear();
  return JITC_OK;
}

