/*
 * jitc.h -- C ABI of the B200-native just-in-time checkpoint capture/restore
 * library (libjitc.so).  Hot path of "Just-In-Time Checkpointing: Low Cost
 * Error Recovery from Deep Learning Training Failures" (Gupta et al.,
 * EuroSys '24); paper text at PAPER.md, cited as PAPER.md:<line> (§section).
 *
 * The paper's user-level library takes a user `save_checkpoint` callback and
 * returns a replica checkpoint path (PAPER.md:99 §3, :132 §3.2, :140 §3.3).
 * This ABI replaces both with explicit calls on the GPU state of healthy
 * data-parallel replicas:
 *
 *   register (steady state) -> mark (every optimizer step)
 *   on failure: fingerprint -> exchange_records -> select_consistent_replica
 *               -> capture (shard s of k) -> commit
 *   on restart / replacement: restore -> verify
 *
 * Conventions (all functions):
 *  - Every call returns a jitc_status; 0 == JITC_OK.  On error, the text of
 *    jitc_last_error(ctx) (or jitc_last_error(NULL) for ctx-less calls,
 *    thread-local) says why.  No call aborts the process.
 *  - Pointers: "device" = CUDA device memory of cfg.device (e.g. torch
 *    tensors' data_ptr); "host" = ordinary host memory.  Tensor pointers,
 *    staging and streams are CALLER-OWNED and must stay valid and unmoved
 *    until jitc_destroy or a re-register; the library never frees them.  Host
 *    images, manifests, digests and events are LIBRARY-OWNED.
 *  - Blocking: each call returns after its GPU work has completed.  It waits
 *    only on the library's own non-blocking streams and events -- never on
 *    the legacy default stream, never cudaDeviceSynchronize -- and
 *    fingerprint / capture / restore / verify never allocate, free or pin
 *    (all of that happens in create / register).  This generalises
 *    PAPER.md:134 (copies re-issued on a new stream because the default
 *    stream is blocked behind the hung collective).
 *  - Threading: one thread per ctx at a time; callable from a non-Python
 *    watchdog thread (no callbacks, so no GIL).
 *  - Collective calls (every member of the library communicator must call):
 *    jitc_comm_init, jitc_comm_shrink, jitc_exchange_records, jitc_commit,
 *    jitc_restore, jitc_capture_fanout.  Local: register, declare_group,
 *    attach_image, mark, fingerprint, capture, verify.  Pure (no ctx, no
 *    GPU): jitc_layout, jitc_shard_range, jitc_select_consistent_replica,
 *    jitc_restore_plan, jitc_capture_plan.
 *  - No CPU fallback: if the device or the sm_100a kernels are unavailable
 *    the call fails with JITC_ECUDA.
 *  - Binary formats (record blob, selection, manifest, commit record) are
 *    little-endian and specified in DESIGN.md §Formats.
 */
#ifndef JITC_H_
#define JITC_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define JITC_ABI_VERSION 2  /* 2: jitc_stats.groups_done / groups_skipped, timeline spans */
#define JITC_ALL_GROUPS 0xFFFFFFFFu

typedef struct jitc_ctx jitc_ctx;
typedef int32_t jitc_status;

enum {
    JITC_OK = 0,
    JITC_EINVAL = -1,          /* bad argument                                          */
    JITC_ESTATE = -2,          /* call out of order (e.g. capture before fingerprint)   */
    JITC_ENOMEM = -3,          /* device / pinned host allocation failed                 */
    JITC_ECUDA = -4,           /* CUDA runtime error (incl. no device / no sm_100a)      */
    JITC_ENCCL = -5,           /* NCCL error                                             */
    JITC_ELAYOUT = -6,         /* replicas registered different tensors / topology       */
    JITC_ENOREPLICA = -7,      /* a REQUIRED group has no healthy replica */
    JITC_ECONFLICT = -8,       /* tie between differing replica classes                  */
    JITC_ENOCONSISTENT = -9,   /* no version common to all REQUIRED groups*/
    JITC_EUNSTABLE = -10,      /* bytes changed between fingerprint and capture          */
    JITC_ECORRUPT = -11,       /* restored bytes do not match the manifest digests       */
    JITC_EINCOMPLETE = -12,    /* checkpoint not committed (PAPER.md:136 metadata last)  */
    JITC_EIO = -13,            /* file / shm error                                       */
    JITC_EPEER = -14           /* a communicator peer died while this call waited on it
                                  (IPC transport: its heartbeat went stale); see
                                  jitc_comm_dead, then jitc_comm_shrink and retry          */
};

/* Optimizer-step phase of a group, written by jitc_mark (PAPER.md:188 hooks). */
enum { JITC_PHASE_CLEAN = 0, JITC_PHASE_DIRTY = 1 };
/* Group policy: REQUIRED state must be recovered; OPTIONAL (grads-like) state
 * is kept only if consistent at the selected version (reading R1). */
enum { JITC_REQUIRED = 0, JITC_OPTIONAL = 1 };
/* Restore source: HOST = the committed host image (every rank restarts,
 * PAPER.md:116); PEER = the writers' live HBM over NVLink (only the
 * replacement lost its state). */
enum { JITC_RESTORE_HOST = 0, JITC_RESTORE_PEER = 1 };
/* Per-group selection status (jitc_sel_group.status). */
enum { JITC_G_OK = 0, JITC_G_UNVERIFIED_SINGLE = 1, JITC_G_NOREPLICA = 2, JITC_G_DROPPED = 3,
       JITC_G_CONFLICT = 4, JITC_G_NOCANDIDATE = 5 };
/* Reason a healthy member is not a writer (O6 step 10). */
enum { JITC_X_DIRTY = 1, JITC_X_STALE_VERSION = 2, JITC_X_MINORITY = 3 };
/* jitc_config.flags */
enum {
    JITC_F_ZERO_COPY_D2H = 1u << 0,  /* capture: K2 stores straight into mapped pinned host memory */
    JITC_F_ZERO_COPY_H2D = 1u << 1,  /* restore: K3 loads straight from mapped pinned host memory  */
    JITC_F_TIME_KERNELS = 1u << 2,   /* bracket every kernel launch with CUDA events (stats)        */
    JITC_F_RESERVED_3 = 1u << 3      /* reserved, no effect: the library never deletes host images
                                        (image_dir belongs to the launcher)            */
};

typedef struct {
    int32_t device;          /* CUDA device ordinal                                          */
    int32_t rank;            /* this process's job rank (member lists use job ranks)         */
    int32_t world;           /* job world size                                               */
    uint32_t flags;          /* JITC_F_*                                                     */
    uint64_t chunk_bytes;    /* digest chunk C: power of two in [4 KiB, 64 MiB]; 0 => 1 MiB  */
    void* staging;           /* device staging buffer (caller-owned) or NULL => library      */
    uint64_t staging_bytes;  /* staging size; 0 => 1 GiB.  Split into rounds of slot_bytes.  */
    uint64_t slot_bytes;     /* bytes per pipeline round (multiple of C); 0 => 256 MiB       */
    const char* image_dir;   /* host image location: a directory on /dev/shm shared by the
                                ranks of one box (survives process death; the library never
                                deletes it -- the launcher removes it when the job ends), or
                                NULL => private pinned memory (writers must stay alive)       */
    void* streams[2];        /* caller-created non-blocking cudaStream_t (compute, copy) or
                                NULL => library-created                                       */
} jitc_config;

/* dtype is an opaque tag folded into layout_hash (the workloads use
 * 0=u8, 1=bf16, 2=f32); the path itself moves bytes. */
typedef struct {
    const char* name;        /* stable name, identical on every replica   */
    void* ptr;               /* device pointer; any alignment (16-B aligned is fastest)      */
    uint64_t nbytes;         /* may be 0 and need not be a multiple of anything              */
    uint32_t dtype;
} jitc_tensor;

/* Per-call statistics (optional out-parameter; may be NULL). */
typedef struct {
    double ms_host;            /* wall time of the call                                        */
    double ms_device;          /* CUDA-event span of the call on the library streams           */
    double ms_kernel;          /* sum of the call's kernel durations (needs JITC_F_TIME_KERNELS)*/
    uint64_t image_bytes;      /* image bytes this rank packed / unpacked / digested           */
    uint64_t d2h_bytes, h2d_bytes, p2p_bytes;  /* p2p: bytes this rank received from peers (NCCL: plus sent) */
    uint64_t kernel_launches;  /* launches of this library's kernels during the call           */
    uint32_t rounds;           /* pipeline rounds                                              */
    int32_t first_bad_chunk;   /* ECORRUPT: first chunk whose digest mismatched, else -1       */
    uint32_t groups_done;      /* restore: groups restored by this call                         */
    uint32_t groups_skipped;   /* restore: OPTIONAL groups left out -- dropped by the selection,
                                  or (HOST without a selection) committed at a version other
                                  than the REQUIRED groups' v* (reading R1)                    */
} jitc_stats;

/* Cumulative per-kernel counters (bench roofline): kind 1 = K1 digest,
 * 2 = K2 pack+digest, 3 = K3 unpack+verify, 4 = K5 peer pull+verify. */
typedef struct {
    uint64_t launches;
    uint64_t bytes;            /* algorithmic image bytes processed                            */
    double ms;                 /* sum of CUDA-event launch durations (JITC_F_TIME_KERNELS)     */
    double span_ms;            /* sum of in-kernel spans, first CTA start -> last CTA end
                                  (%globaltimer; diagnostic, JITC_F_TIME_KERNELS)              */
} jitc_kernel_counter;

/* ---- lifecycle --------------------------------------------------------- */
/* Creates a context on cfg->device: streams (unless given), events, staging
 * (unless given).  Fails with JITC_ECUDA if the device is not sm_100. */
jitc_status jitc_create(const jitc_config* cfg, jitc_ctx** out);
void jitc_destroy(jitc_ctx* ctx);
/* Thread-local text of the last error (ctx may be NULL). Never NULL. */
const char* jitc_last_error(const jitc_ctx* ctx);
int jitc_abi_version(void);

/* ---- steady state ------------------------------------------------------ */
/* A1: registers `n` tensors of `group` held by this rank and
 * declares the group's policy and job-rank members (this rank must be one).
 * Builds the image layout (registration order, 256-B aligned offsets, zero
 * padding; reading R4), the segment table, per-group digest buffers, and
 * maps/pins the host image (image_dir/g<group>.img, or private pinned).
 * Out: layout_hash (fold of names, sizes, dtypes, C) and image_bytes (L). */
jitc_status jitc_register(jitc_ctx* ctx, uint32_t group, int32_t policy, const int32_t* members,
                          int32_t n_members, const jitc_tensor* t, size_t n, uint64_t* layout_hash,
                          uint64_t* image_bytes);
/* Declares a group this rank does NOT hold (e.g. another rank's ZeRO shard),
 * so the selection can tell "no replica" from "not part of the job". */
jitc_status jitc_declare_group(jitc_ctx* ctx, uint32_t group, int32_t policy, const int32_t* members,
                               int32_t n_members);
/* A2: stream-ordered phase word of `group`: version<<1 | phase, one atomic
 * 8-B write into mapped pinned host memory, issued with cuStreamWriteValue64
 * on `stream` (after the optimizer kernels already queued there; no kernel,
 * no sync).  stream == NULL writes immediately from the host.  Mirrors the
 * pre/post-optimizer-step hooks of PAPER.md:188. */
jitc_status jitc_mark(jitc_ctx* ctx, uint32_t group, uint64_t version, int32_t phase, void* stream);
/* Reads the phase word as the capture will see it. */
jitc_status jitc_phase(jitc_ctx* ctx, uint32_t group, uint64_t* version, int32_t* phase);

/* ---- communicator (NCCL over NVLink/NVSwitch) ---------------------------- */
/* 128-byte ncclUniqueId (rank 0 creates, the harness distributes it). */
jitc_status jitc_get_unique_id(void* id128);
/* Library-owned NCCL communicator of `nranks`; comm rank i <-> job rank
 * job_ranks[i] (NULL => identity). */
jitc_status jitc_comm_init(jitc_ctx* ctx, const void* id128, int32_t nranks, int32_t comm_rank,
                           const int32_t* job_ranks);
/* Drops `failed` job ranks with ncclCommShrink(NCCL_SHRINK_ABORT), which also
 * aborts collectives hung on the old communicator (PAPER.md:180 re-establish
 * comms; Table 7 shows this dominates recovery). */
jitc_status jitc_comm_shrink(jitc_ctx* ctx, const int32_t* failed, int32_t n_failed);
jitc_status jitc_comm_destroy(jitc_ctx* ctx);
/* Intra-node IPC transport instead of NCCL, for ranks of ONE box.  The ranks
 * share a control block in `comm_dir/ctl` (a fresh directory per
 * communicator, like a unique id) and map each other's staging buffers with
 * CUDA IPC.  Exchange, barrier and restore then need no NCCL: progress
 * counters are written by the GPU in stream order (cuStreamWriteValue64 into
 * the mapped control block) and polled by the peers, and K3 reads each
 * peer's block directly from the peer's staging (NVLink peer loads), fusing
 * the slice exchange into the unpack+verify kernel.  jitc_comm_shrink drops
 * ranks; every other call behaves as with NCCL. */
jitc_status jitc_comm_init_ipc(jitc_ctx* ctx, const char* comm_dir, int32_t nranks, int32_t comm_rank,
                               const int32_t* job_ranks);

/* ---- on failure: capture --------------------------------------------------- */
/* A3 = K1: JF64 chunk digests of every registered byte of `group` (or all
 * held groups with JITC_ALL_GROUPS), read from live HBM, plus the phase word.
 * Output: this rank's record blob (header, topology, one record per group;
 * DESIGN.md §Formats).  cap == 0 => only *len (the needed size) is set.
 * The checksum primitive the paper uses for replay validation,
 * here the replica-consistency evidence. */
jitc_status jitc_fingerprint(jitc_ctx* ctx, uint32_t group, void* blob, size_t cap, size_t* len);
/* A4 = C1: all-gathers every member's blob over the library communicator
 * (blob sizes first, then the padded blobs) and writes them, compacted and
 * in comm-rank order, to `all`.  Without a communicator (single process)
 * copies `mine`.  cap == 0 => only *all_len. */
jitc_status jitc_exchange_records(jitc_ctx* ctx, const void* mine, size_t len, void* all, size_t cap,
                                  size_t* all_len);
/* A5 (pure): the consistency rule O6.  Keeps blobs of
 * `healthy` job ranks; per group the unique largest class of identical CLEAN
 * records per version; v* = max version at which every REQUIRED group has a
 * candidate; writers = that class; the rest excluded
 * with a reason.  Returns the overall status (also stored in the selection);
 * the selection is written even on ELAYOUT/ENOREPLICA/ECONFLICT/
 * ENOCONSISTENT for diagnostics.  Every rank computes the same bytes. */
jitc_status jitc_select_consistent_replica(const void* blobs, size_t len, const int32_t* healthy,
                                           int32_t n_healthy, void* selection, size_t cap,
                                           size_t* sel_len);
/* A6+A7 = K2 + D2H: if this rank is writer s of k for `group` (or for each
 * held group with JITC_ALL_GROUPS) it packs its chunk range
 * [floor(s*n_c/k), floor((s+1)*n_c/k)) (O5) into the host image, in rounds:
 * K2 gathers the tensors into a staging slot (or straight into mapped host
 * memory with JITC_F_ZERO_COPY_D2H) re-digesting every chunk, and the copy
 * stream drains the slot D2H while K2 fills the next.  The rounds of all
 * groups of the call form one pipeline whose first round is 512 MiB (so the
 * copy engine starts at once).  A re-digest that differs from the last
 * jitc_fingerprint => JITC_EUNSTABLE (checked after the pipeline drained;
 * the group then counts as not captured, so jitc_commit refuses it).  On any
 * error the call returns only after its copies finished.  A non-writer
 * returns JITC_OK having done nothing, so every rank can call it. */
jitc_status jitc_capture(jitc_ctx* ctx, const void* selection, size_t sel_len, uint32_t group,
                         jitc_stats* stats);
/* A8: after every writer's capture, writes per group the manifest (header,
 * tensor table, digests, root, shard map, v*) and LAST the commit record
 * ("metadata file is stored at the end").  Collective: a
 * barrier on the communicator orders "all shards done" before the manifest;
 * the lowest-rank writer of each group writes it. */
jitc_status jitc_commit(jitc_ctx* ctx, const void* selection, size_t sel_len);

/* Capture with NVLink fan-out.  Capture is
 * bound by each writer's host link (PCIe), so a group with few writers --
 * k = 1 for the TP partition whose other replica died (C5), a ZeRO shard
 * (C4) -- would leave the other GPUs' links idle.  Collective over the
 * communicator (every comm rank calls it, with the same arguments).  For
 * `group` (or every group of the selection, in increasing id, with
 * JITC_ALL_GROUPS): writer s still packs and re-digests exactly its O5(n_c,
 * k, s) shard (JITC_EUNSTABLE as for jitc_capture), but the image is D2H'd
 * in m lanes, lane q = O5(n_c, m, q) by the q-th of `movers` (job ranks,
 * taken in sorted order, all in the communicator); the part of shard s that
 * falls in another mover's lane is sent to it over NVLink (NCCL send/recv,
 * or with the IPC transport a peer-to-peer copy out of the writer's
 * staging) and that mover D2Hs it with its own copy engine and PCIe link.
 * Every mover must hold the group's host image: its own (a member) or one
 * attached with jitc_attach_image.  The image bytes, the manifest and the
 * shard table are exactly those of jitc_capture; jitc_commit follows as
 * usual.  Needs a shared image_dir. */
jitc_status jitc_capture_fanout(jitc_ctx* ctx, const void* selection, size_t sel_len, uint32_t group,
                                const int32_t* movers, int32_t n_movers, jitc_stats* stats);
/* Steady-state preparation of a fan-out mover for a group it does not hold
 * (declared with jitc_declare_group): maps image_dir/g<group>.img, sized for
 * an image of `image_bytes` (the L that jitc_register of the group's members
 * returns), and pins it, so that jitc_capture_fanout neither maps nor pins in
 * the failure path.  JITC_EINVAL if the group is held or undeclared, or the
 * context has no image_dir. */
jitc_status jitc_attach_image(jitc_ctx* ctx, uint32_t group, uint64_t image_bytes);

/* Local (non-collective) capture of every held group by this rank alone:
 * fingerprint -> select over its own record -> capture (k = 1) -> commit.
 * The paper's user-level protocol in which each healthy rank saves its own
 * state, and the host round trip of transient
 * recovery (copy to host, reset, copy back).  A DIRTY group
 * makes it fail with JITC_ENOCONSISTENT.  This is what the
 * watchdog runs with JITC_ON_HANG_LOCAL_CAPTURE. */
jitc_status jitc_capture_local(jitc_ctx* ctx, jitc_stats* stats);

/* The user's CPU state -- iteration number, RNG state, data-loader position
 * (save_checkpoint saves "any CPU state") -- as an opaque blob
 * carried in every group's manifest of the next jitc_commit (covered by the
 * manifest trailer and the commit record), and read back after a HOST
 * restore (or on the committing writer) with jitc_get_aux.  cap == 0 =>
 * only *len. */
jitc_status jitc_set_aux(jitc_ctx* ctx, const void* data, size_t len);
jitc_status jitc_get_aux(jitc_ctx* ctx, uint32_t group, void* out, size_t cap, size_t* len);

/* ---- restore ------------------------------------------------------------- */
/* A9-A11.  HOST: refuses an uncommitted image (JITC_EINCOMPLETE); each comm
 * rank loads chunk range O5(n_c, n, r) H2D, the ranks all-gather the slices
 * over NVLink in rounds, and K3 scatters every round into the registered
 * tensors while re-digesting it; any chunk whose digest differs from the
 * manifest => JITC_ECORRUPT (stats->first_bad_chunk).  PEER: the selection's
 * writers pack their ranges from live HBM (K2) and send them to every member
 * that is not a writer (the replacement, and members excluded as DIRTY /
 * MINORITY / STALE), which unpack+verify with K3 against the writers'
 * digests.  selection may be NULL in HOST mode (taken from the manifest). */
jitc_status jitc_restore(jitc_ctx* ctx, uint32_t group, int32_t mode, const void* selection,
                         size_t sel_len, jitc_stats* stats);
/* F1 fusion -- intra-node PEER restore by direct peer-memory reads (no NCCL,
 * no staging).  A writer (after jitc_fingerprint, while its state stays
 * quiesced) publishes CUDA IPC handles of the allocations holding its
 * registered tensors and its digests into image_dir (g<group>.peer.<rank>).
 * The replacement maps every selected writer's export and ONE kernel (K5)
 * reads writer s's chunk range O5(n_c, k, s) over NVLink, scatters it into
 * its own tensors and re-digests it in the same pass; digests that differ
 * from the writers' => JITC_ECORRUPT (stats->first_bad_chunk).  The mappings
 * are closed before returning, after which the writers may resume.  Not for
 * VMM / expandable-segment allocations (not IPC-exportable: JITC_ECUDA). */
jitc_status jitc_peer_export(jitc_ctx* ctx, uint32_t group);
jitc_status jitc_restore_pull(jitc_ctx* ctx, uint32_t group, const void* selection, size_t sel_len,
                              jitc_stats* stats);
/* A12: K1 over the live tensors of `group`, compared with `expected` (a
 * record blob holding that group) or, if NULL, with the manifest digests of
 * the last restore / commit.  Mismatch => JITC_ECORRUPT, *first_bad_chunk
 * set (else UINT64_MAX). */
jitc_status jitc_verify(jitc_ctx* ctx, uint32_t group, const void* expected, size_t len,
                        uint64_t* first_bad_chunk);

/* ---- pure helpers --------------------------------------------------------- */
/* O1 layout: offsets (may be NULL; n entries), layout_hash, image_bytes. */
jitc_status jitc_layout(const jitc_tensor* t, size_t n, uint64_t chunk_bytes, uint64_t* offsets,
                        uint64_t* layout_hash, uint64_t* image_bytes);
/* O5 shard rule: writer s of k gets chunks [*c0, *c1). */
jitc_status jitc_shard_range(uint64_t n_c, uint32_t k, uint32_t s, uint64_t* c0, uint64_t* c1);
/* The round schedule jitc_restore executes for `group` on comm rank
 * `comm_rank` of an n-rank communicator whose comm rank i is job rank
 * comm_job_ranks[i], given the staging geometry.  Output: a 24-B header
 * ('JITP', n_ops, round_bytes, slots, n_rounds) followed by n_ops 48-B operations
 * {round, kind (1 H2D, 2 ALLGATHER, 3 PACK, 4 SEND, 5 RECV, 6 UNPACK,
 * 7 DIGEST_SEND, 8 DIGEST_RECV), slot, peer, image range [a, b), staging
 * offset, bytes}.  Only the group's members get operations
 * (DESIGN.md §8).  Pure: lets the multi-rank schedule be checked without
 * GPUs.  cap == 0 => only *len. */
jitc_status jitc_restore_plan(const void* selection, size_t sel_len, uint32_t group, int32_t mode,
                              const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank,
                              uint64_t staging_bytes, uint64_t slot_bytes, void* plan, size_t cap,
                              size_t* len);

/* The round schedule jitc_capture_fanout executes for `group` on comm rank
 * `comm_rank` (same header and 48-B operations as jitc_restore_plan; kinds
 * 3 PACK, 4 SEND, 5 RECV, 9 D2H).  Pure.  cap == 0 => only *len. */
jitc_status jitc_capture_plan(const void* selection, size_t sel_len, uint32_t group, const int32_t* movers,
                              int32_t n_movers, const int32_t* comm_job_ranks, int32_t n, int32_t comm_rank,
                              uint64_t staging_bytes, uint64_t slot_bytes, void* plan, size_t cap, size_t* len);

/* ---- durable tier (NEXT-4; §6.3) ---------------------- */
/* Streams the committed host image of `group` to `dir` (parallel O_DIRECT
 * writes when the file system supports them, then fdatasync), then the
 * manifest, then LAST the commit record -- the low-frequency periodic copy
 * that survives losing every replica, in the same format.
 * JITC_EINCOMPLETE if the group has no committed checkpoint. */
jitc_status jitc_persist(jitc_ctx* ctx, uint32_t group, const char* dir, jitc_stats* stats);
/* Reads a durable copy back into the host image (validating the commit
 * record, the manifest trailer and the layout: JITC_EINCOMPLETE /
 * JITC_ELAYOUT) and installs its manifest, so that jitc_restore(HOST)
 * restores it with full K3 verification.  O_DIRECT reads go through two
 * 64 MiB bounce buffers per I/O thread (8 threads; JITC_DURABLE_THREADS),
 * the copy into the image overlapping the next read. */
jitc_status jitc_stage_in(jitc_ctx* ctx, uint32_t group, const char* dir, jitc_stats* stats);

/* ---- hang detection (NEXT-1; §3.1-3.2) ------------------ */
/* The caller records a CUDA event after each collective on its NCCL stream
 * (the event the compute stream waits on, PAPER.md:122 / Fig. 3) and puts it
 * on the watch-list; completed events drop off.  A native watchdog thread
 * polls the list with cudaEventQuery every 200 us; an event still incomplete
 * `timeout_ms` after it was added is a hang.  On a hang the watchdog thread
 * runs the action itself -- JITC_ON_HANG_LOCAL_CAPTURE: fingerprint, select
 * over this rank's own record, capture, commit (no collective; the paper's
 * user-level protocol), entirely in C++ on the library's
 * non-blocking streams, so neither the GIL nor the blocked default stream can
 * stop it -- then calls fn(user, tag, waited_ms) if given,
 * and stops.  While the watchdog runs, other threads may call only
 * jitc_watch_event / jitc_watchdog_wait / jitc_watchdog_stop on the ctx. */
typedef void (*jitc_hang_fn)(void* user, uint64_t tag, double waited_ms);
/* JITC_ON_HANG_COLLECTIVE_CAPTURE (IPC transport): peers whose heartbeat (a
 * thread started by jitc_comm_init_ipc refreshes it every 10 ms) is older
 * than timeout_ms are dead; the survivors drop them (jitc_comm_shrink) and
 * run fingerprint -> exchange -> select -> sharded capture -> commit among
 * themselves on their watchdog threads -- the paper's whole user-level
 * protocol with no Python and no scheduler. */
/* The same action over an NCCL communicator (jitc_comm_init) needs the
 * liveness table below: failed ranks are dropped with
 * ncclCommShrink(NCCL_SHRINK_ABORT), and the exchange and the commit barrier
 * run over the shrunk NCCL communicator.  Without either table the action
 * returns JITC_ESTATE. */
enum { JITC_ON_HANG_NOTIFY = 0, JITC_ON_HANG_LOCAL_CAPTURE = 1, JITC_ON_HANG_COLLECTIVE_CAPTURE = 2 };
/* Liveness table for failure localisation with the NCCL transport
 * (§3.1: the survivors must tell a dead peer from a hung
 * one).  Maps <dir>/liveness -- a directory on /dev/shm shared by the ranks of
 * ONE box, created on first use, 8 KiB -- and starts a thread that writes this
 * rank's CLOCK_MONOTONIC heartbeat (slot = job rank cfg.rank, < 1024) every
 * 10 ms until jitc_destroy.  A communicator member whose heartbeat is older
 * than the watchdog timeout, or was never written, counts as dead, so every
 * rank calls this before arming its watchdog.  Local; may be called again
 * (re-maps).  Errors: JITC_EINVAL (null ctx/dir, rank out of range),
 * JITC_EIO (file or mapping). */
jitc_status jitc_liveness_init(jitc_ctx* ctx, const char* dir);
/* Job ranks of the current communicator whose heartbeat (IPC control block,
 * or the liveness table) is older than the dead-peer threshold: 2000 ms, or
 * JITC_PEER_DEAD_MS read at communicator init.  Writes up to cap ranks and
 * *n = count.  Local.  The recovery for reading R9 (a writer dies during the
 * capture): a collective call returns JITC_EPEER, every survivor calls this,
 * rebuilds the communicator without the dead ranks, and re-runs fingerprint
 * -> exchange -> select -> capture -> commit with k - 1 writers (HBM still
 * holds the state).  IPC transport: jitc_comm_shrink(dead).  NCCL: the
 * failed collective is still in flight on the library's stream and
 * ncclCommShrink cannot be trusted with it (measured: one survivor's shrink
 * failed, the other's hung), so jitc_comm_shrink refuses (JITC_ESTATE);
 * jitc_comm_destroy aborts the communicator and jitc_comm_init with a fresh
 * unique id among the survivors (job_ranks) rebuilds it. */
jitc_status jitc_comm_dead(jitc_ctx* ctx, int32_t* ranks, int32_t cap, int32_t* n);
jitc_status jitc_watch_event(jitc_ctx* ctx, void* event, uint64_t tag);
jitc_status jitc_watchdog_start(jitc_ctx* ctx, uint32_t timeout_ms, int32_t action, jitc_hang_fn fn, void* user);
/* Blocks up to max_ms for the hang action to finish.  *fired = 1 if it did;
 * returns the action's status (JITC_OK when nothing fired). */
jitc_status jitc_watchdog_wait(jitc_ctx* ctx, uint32_t max_ms, int32_t* fired, uint64_t* tag, double* waited_ms,
                               double* action_ms, jitc_stats* action_stats);
jitc_status jitc_watchdog_stop(jitc_ctx* ctx);
/* Job ranks the collective action found dead (up to cap; *n = count). */
jitc_status jitc_watchdog_failed(jitc_ctx* ctx, int32_t* ranks, int32_t cap, int32_t* n);

/* ---- analytic model (NEXT-3; §5, eqs. 1-8) ------------------------ */
enum { JITC_MODEL_PERIODIC_OPTIMAL = 0, JITC_MODEL_PERIODIC = 1, JITC_MODEL_USER_JIT = 2,
       JITC_MODEL_TRANSPARENT_JIT = 3 };
/* Wasted GPU time per GPU per unit of useful time (w) and the wasted-time
 * fraction w_f = w / (1 + w) (eq. 6) for N GPUs with per-GPU failure rate f
 * (1/s), checkpoint time o (s), fixed recovery time r (s), minibatch time m
 * (s), JIT steady-state overhead o_jit (fraction) and, for
 * JITC_MODEL_PERIODIC, checkpoint frequency c (1/s).  *c_opt (may be NULL)
 * receives the optimal periodic frequency c* = sqrt(N f / (2 o)) (eq. 3; the
 * printed "2α" is read as 2o).  Pure. */
jitc_status jitc_waste_model(int32_t kind, double n_gpus, double f, double o, double r, double m, double o_jit,
                             double c, double* c_opt, double* w, double* w_f);

/* ---- counters ---------------------------------------------------------------- */
jitc_status jitc_kernel_counters(jitc_ctx* ctx, int32_t kind, jitc_kernel_counter* out);
jitc_status jitc_reset_counters(jitc_ctx* ctx);

/* ---- timeline (overlap evidence; nsys is not available on the boxes) --------- */
/* One span of work on a library stream: a kernel launch (kind 1 K1, 2 K2,
 * 3 K3, 4 K5), a copy-engine transfer batch (10 D2H, 11 H2D, 12 peer copy)
 * of one pipeline round.  t0/t1 are CUDA-event times in ms relative to the
 * jitc_timeline_start event; stream 0 = compute, 1 = copy. */
typedef struct {
    int32_t kind;
    int32_t stream;
    uint32_t group;
    uint32_t round;
    double t0_ms, t1_ms;
    uint64_t bytes;
} jitc_span;
/* Starts recording spans of the following calls (up to max_spans; events are
 * created here, in steady state).  Each span costs two timing-event records
 * (~40 us each next to a copy-engine transfer), so this is a
 * diagnostic, not the bench's timed configuration. */
jitc_status jitc_timeline_start(jitc_ctx* ctx, uint32_t max_spans);
/* Stops recording and writes up to cap spans (after the recorded calls
 * returned); *n = spans recorded.  cap == 0 => only *n. */
jitc_status jitc_timeline_read(jitc_ctx* ctx, jitc_span* out, size_t cap, size_t* n);

/* ---- test/bench harness kernels (K4; not part of the method) ------------- */
/* Fills numel elements of a device tensor with the O9 counter-based generator
 * (dtype 0=u8,1=bf16,2=f32,3=zeros,4=ones).  Integer-only, so bit-identical
 * with the oracle's generator. */
jitc_status jitc_gen_fill(void* dptr, uint32_t dtype, uint64_t numel, uint64_t seed, uint32_t group,
                          uint32_t gen_id, uint32_t exp_lo, uint32_t exp_hi, int32_t force_pos,
                          void* stream);
/* O10 synthetic optimizer update U_v on elements [e0, e0+count) of the fp32
 * device tensor whose element 0 is at dptr; and bf16 params re-derived as
 * RNE(master). */
jitc_status jitc_inject_update(void* dptr, uint64_t e0, uint64_t count, uint32_t gen_id, uint64_t v,
                               void* stream);
jitc_status jitc_inject_rne(const void* master_f32, void* param_bf16, uint64_t count, void* stream);
/* Flips bit `bit` of byte `byte` of device memory at dptr. */
jitc_status jitc_inject_bitflip(void* dptr, uint64_t byte, uint32_t bit, void* stream);
/* Emulates a collective hung on a failed peer: launches
 * n_ctas spinning CTAs on `stream` that wait on device flag `slot` (0..63),
 * as NCCL kernels wait on flags their peers write; jitc_inject_release(slot)
 * sets the flag from a kernel on a separate stream and lets them exit. */
jitc_status jitc_inject_hang(void* stream, int32_t n_ctas, uint32_t slot);
jitc_status jitc_inject_release(uint32_t slot);

#ifdef __cplusplus
}
#endif
#endif /* JITC_H_ */
