#!/usr/bin/env python
"""JIT capture+restore benchmark (BASELINE.json metric).

One step = one pass of the whole hot path over the
synthetic training state of the configuration:
    fingerprint (K1) -> exchange records -> select -> capture (K2 + D2H, shard
    s of k) -> commit (manifest, commit record) -> restore HOST (H2D [+ NVLink
    all-gather] + K3 unpack+verify) -> verify (K1 vs manifest)
value = replica-state bytes L / step time (GB/s); seconds_to_recover = step time.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl jitc|reference]

N > 1 runs under torchrun (one process per GPU, NCCL over NVLink; every rank
holds a full DP replica, capture is sharded k = N ways, the image lives in a
/dev/shm file shared by the ranks of the box).  The state is larger than L2
(24.9 GB for C2 vs 126 MB), so no L2 flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import numpy as np
import os
import shutil
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

HOST_LINK_NOMINAL = 63.0   # PCIe Gen5 x16 GB/s per direction (context)
# measured on this pool's B200 boxes (profiles/r01_pcie_probe.txt, tools/pcie_probe.cu): the copy-engine
# limit for 4 GiB transfers, identical for cudaHostAlloc / shm+register / malloc+register and 1-4 streams
HOST_LINK_MEASURED = {"d2h": 57.2, "h2d": 55.6}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d.get("hbm_gbs", 6650.0)), "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""

    def __init__(self, gpu: int):
        self.gpu, self.rows, self.proc = gpu, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu),
                 "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
                 "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
                 "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({n for r in self.rows for n, v in zip(names, r[4:8]) if v.lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def calibrate_links(device: int, world: int, nccl_group=None, host_gib: int = 2):
    """In-run link calibration, untimed, before the
    timed region: B_d2h / B_h2d with every rank copying at once (64 MiB
    cudaMemcpyAsync pieces of pinned memory, best of 5), B_hbm from a 4 GiB
    device-to-device copy (read + write bytes), B_nvl from a 256 MiB-per-rank
    NCCL all-gather (bus bandwidth (n-1)/n * total / t) when an NCCL group is
    given.  Returns GB/s (per rank for the host link)."""
    import torch
    import torch.distributed as dist
    n = host_gib << 30
    piece = 64 << 20
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(n, dtype=torch.uint8, device=f"cuda:{device}")
    s = torch.cuda.Stream(device)
    out = {}

    def timed(fn, reps=5):
        best = None
        for _ in range(reps):
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(s):
                e0.record(s)
                fn()
                e1.record(s)
            e1.synchronize()
            t = e0.elapsed_time(e1) * 1e-3
            best = t if best is None else min(best, t)
        return best

    def d2h():
        for o in range(0, n, piece):
            h[o:o + piece].copy_(d[o:o + piece], non_blocking=True)

    def h2d():
        for o in range(0, n, piece):
            d[o:o + piece].copy_(h[o:o + piece], non_blocking=True)

    out["d2h_GBps"] = round(n / timed(d2h) / 1e9, 2)
    out["h2d_GBps"] = round(n / timed(h2d) / 1e9, 2)
    del h
    a = torch.empty(4 << 30, dtype=torch.uint8, device=f"cuda:{device}")
    b = torch.empty_like(a)
    out["hbm_copy_GBps"] = round(2 * a.numel() / timed(lambda: b.copy_(a)) / 1e9, 1)
    # read-only reference for K1 (which only reads): torch's int64 sum over the
    # same 4 GiB (a reduction with a negligible write)
    a.zero_()
    out["hbm_read_GBps"] = round(a.numel() / timed(lambda: a.view(torch.int64).sum()) / 1e9, 1)
    del a, b, d
    if nccl_group is not None and world > 1:
        blk = torch.empty(256 << 20, dtype=torch.uint8, device=f"cuda:{device}")
        allb = torch.empty(world * blk.numel(), dtype=torch.uint8, device=f"cuda:{device}")
        t = timed(lambda: dist.all_gather_into_tensor(allb, blk, group=nccl_group))
        out["nvl_allgather_busbw_GBps"] = round((world - 1) * blk.numel() / t / 1e9, 1)
    torch.cuda.empty_cache()
    out["how"] = (f"{host_gib} GiB pinned, 64 MiB pieces, all {world} rank(s) at once, best of 5, after the warm-up steps; "
                  "HBM: 4 GiB D2D copy (read+write); HBM read: torch int64 sum over the 4 GiB")
    return out


def per_tensor_d2h(states, device: int, world: int, buf_gib: int = 4, reps: int = 2):
    """the CE-only "pure copy" baseline -- every registered
    tensor copied D2H on its own (one cudaMemcpyAsync per tensor, like a
    per-tensor torch.save), with no fingerprint and no staging.  Destinations
    wrap around a pinned buffer of buf_gib GiB at 256-B-aligned offsets (the
    link, not the host footprint, is what is measured).  Every rank copies its
    FULL state at once (the paper's every-rank-saves protocol at raw copy
    speed).  Untimed region; CUDA events on the copy stream, best of reps."""
    import torch
    import torch.distributed as dist
    tensors = [st.tensor_bytes(i) for st in states.values() for i in range(len(st.spec.tensors))]
    total = sum(t.numel() for t in tensors)
    h = torch.empty(buf_gib << 30, dtype=torch.uint8, pin_memory=True)
    s = torch.cuda.Stream(device)
    best = None
    for _ in range(reps):
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(s)
            pos = 0
            for t in tensors:
                n = t.numel()
                if pos + n > h.numel():
                    pos = 0
                h[pos:pos + n].copy_(t, non_blocking=True)
                pos += (n + 255) // 256 * 256
            e1.record(s)
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        best = ms if best is None else min(best, ms)
    del h
    return {"tensors": len(tensors), "bytes": total, "ms": round(best, 2),
            "GBps": round(total / (best * 1e-3) / 1e9, 2),
            "how": "one cudaMemcpyAsync D2H per registered tensor into pinned memory (no digest, no staging); "
                   "all ranks at once; CUDA events, best of %d" % reps}


def host_link_roofline(d2h_bytes_rank, h2d_bytes_rank, capture_ms, restore_ms, links):
    """Capture / restore GB/s of the busiest rank's host link (its D2H bytes
    over the capture phase, its H2D bytes over the restore phase; max over
    ranks) against nominal PCIe Gen5 x16, the pool's probe
    (profiles/r01_pcie_probe.txt) and, when run, this run's own calibration
    (calibrate_links, all ranks at once)."""
    cap = d2h_bytes_rank / (capture_ms * 1e-3) / 1e9
    res = h2d_bytes_rank / (restore_ms * 1e-3) / 1e9
    out = {"capture_GBps_per_rank": round(cap, 2), "restore_GBps_per_rank": round(res, 2),
           "d2h_bytes_busiest_rank": int(d2h_bytes_rank), "h2d_bytes_busiest_rank": int(h2d_bytes_rank),
           "nominal_GBps": HOST_LINK_NOMINAL, "probe_GBps": HOST_LINK_MEASURED,
           "capture_frac_nominal": round(cap / HOST_LINK_NOMINAL, 3),
           "restore_frac_nominal": round(res / HOST_LINK_NOMINAL, 3),
           "capture_frac_probe": round(cap / HOST_LINK_MEASURED["d2h"], 3),
           "restore_frac_probe": round(res / HOST_LINK_MEASURED["h2d"], 3)}
    if links:
        out["calibrated"] = links
        out["capture_frac_calibrated"] = round(cap / links["d2h_GBps"], 3)
        out["restore_frac_calibrated"] = round(res / links["h2d_GBps"], 3)
    return out


# ---------------------------------------------------------------------- reference arm / cpu baseline
def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def host_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


class OracleRecover:
    """The oracle's capture + restore of one replica,
    phase by phase: layout (O1), pack (O2), JF64 (O3: the fingerprint), select
    (O6), shard (O5), unpack + verify (O3 over the image, compare with the
    digests, O8).  State generation (O9) is not timed.  Pack and unpack+verify
    run on every `every`-th chunk of each group (evenly spaced, chunk_sample)
    and are extrapolated to the whole image by bytes; JF64 runs over the whole
    committed /dev/shm image when one is given (the bytes the GPU digested, so
    it doubles as a bit-exact check of the K1 digests), else on the sample.
    Every step calls the oracle as it stands; `threads` runs the same calls on
    disjoint chunk / tensor ranges."""

    def __init__(self, w, rank: int, every: int, C: int = 1 << 20):
        from oracle import oracle as O
        from oracle import stream as S
        self.O, self.S, self.w, self.every, self.C = O, S, w, every, C
        self.groups = w.groups_of(rank)
        self.lays = {g.group: O.layout_of_group(g, C) for g in self.groups}
        self.samples = {g.group: S.chunk_sample(g, w.seed, self.lays[g.group], every) for g in self.groups}
        self.L = sum(l.L for l in self.lays.values())
        self.sample_bytes = sum(cs.nbytes for cs in self.samples.values())

    def run(self, threads: int, blob: bytes = None, committed: dict = None, digests: dict = None) -> dict:
        """One recovery of the replica; returns per-phase seconds (sampled
        phases extrapolated), the measured (unextrapolated) seconds, and the
        digest checks.  blob: this rank's record blob for O6 (built from the
        sample's own digests when None); committed: group -> image array;
        digests: group -> the GPU's K1 digests to check against."""
        O, S = self.O, self.S
        ph, meas, checks = {}, {}, {}
        t = time.perf_counter()
        lays = {g.group: O.layout_of_group(g, self.C) for g in self.groups}
        ph["layout"] = meas["layout"] = time.perf_counter() - t
        imgs, scale = {}, {}
        t = time.perf_counter()
        for gid, cs in self.samples.items():
            imgs[gid] = O.pack(cs.pieces, cs.lay, threads=threads)
        meas["pack"] = time.perf_counter() - t
        ph["pack"] = meas["pack"] * self.L / max(self.sample_bytes, 1)
        d_fp = {}
        t = time.perf_counter()
        if committed:
            for gid, lay in lays.items():
                d_fp[gid] = S.jf64_image(committed[gid], self.C, lay.L, threads)
            meas["jf64"] = ph["jf64"] = time.perf_counter() - t
            cover = "full"
        else:
            for gid, cs in self.samples.items():
                d_fp[gid] = S.jf64_sample(imgs[gid], cs, lays[gid].n_c, threads)
            meas["jf64"] = time.perf_counter() - t
            ph["jf64"] = meas["jf64"] * self.L / max(self.sample_bytes, 1)
            cover = "sampled"
        if digests:
            for gid, d in d_fp.items():
                idx = slice(None) if committed else self.samples[gid].chunks
                bad = int(np.count_nonzero(np.asarray(d)[idx] != np.asarray(digests[gid])[idx]))
                checks[gid] = {"chunks": int(np.asarray(d)[idx].size), "mismatch": bad, "coverage": cover}
        if blob is None:
            recs = [O.Record(0, g.group, g.policy, O.CLEAN, 1, lays[g.group].layout_hash, self.C, lays[g.group].L,
                             d_fp[g.group], O.root(lays[g.group].layout_hash, d_fp[g.group])) for g in self.groups]
            blob = O.encode_blob(0, [O.TopoEntry(g.group, g.policy, [0]) for g in self.groups], recs)
        t = time.perf_counter()
        sel = O.select(blob, [0])
        ph["select"] = meas["select"] = time.perf_counter() - t
        assert sel.status == O.OK, sel.status
        t = time.perf_counter()
        for gs in sel.groups:
            for s_ in range(len(gs.writers)):
                O.shard_bytes(gs.n_c, len(gs.writers), s_, gs.C, gs.L)
        ph["shard"] = meas["shard"] = time.perf_counter() - t
        t = time.perf_counter()
        for gid, cs in self.samples.items():
            d = S.jf64_sample(imgs[gid], cs, lays[gid].n_c, threads)
            if not np.array_equal(d[cs.chunks], np.asarray(d_fp[gid])[cs.chunks]):
                raise RuntimeError(f"oracle restore: group {gid} digests differ (ECORRUPT)")
            O.unpack(imgs[gid], cs.lay, threads=threads)
        meas["unpack_verify"] = time.perf_counter() - t
        ph["unpack_verify"] = meas["unpack_verify"] * self.L / max(self.sample_bytes, 1)
        total = sum(ph.values())
        return {"phases_s": {k: round(v, 4) for k, v in ph.items()},
                "measured_s": {k: round(v, 4) for k, v in meas.items()},
                "s_to_recover": round(total, 3), "GBps": round(self.L / total / 1e9, 4),
                "measured_total_s": round(sum(meas.values()), 3), "checks": checks}


def cpu_baseline(w, rank: int, blob: bytes, committed: dict, digests: dict, every: int, every_1t: int) -> dict:
    """SURVEY.md §8(d) d.7 on rank 0 at N = 1: the oracle's recovery of the
    same replica on all host cores and on 1 core.  JF64 covers the whole
    committed image at nproc threads (and checks every K1 digest); pack and
    unpack+verify are sampled (1/every of the chunks, evenly spaced) and
    extrapolated; the 1-core leg samples everything at 1/every_1t."""
    nth = host_threads()
    rec = OracleRecover(w, rank, every)
    t0 = time.perf_counter()
    full = rec.run(nth, blob=blob, committed=committed, digests=digests)
    del rec
    rec1 = OracleRecover(w, rank, every_1t)
    one = rec1.run(1, blob=blob, digests=digests)
    wall = time.perf_counter() - t0
    return {"value": full["GBps"], "unit": "GB/s", "cores": nth, "kind": "oracle",
            "sample": f"{w.name}: whole replica ({rec1.L / 1e9:.2f} GB); "
                      + ("JF64 over the committed /dev/shm image (every chunk, checked against the K1 digests); "
                         if committed else f"JF64 on 1/{every} of the chunks (no /dev/shm image to read); ")
                      + f"pack and unpack+verify on 1/{every} of the chunks, evenly spaced, extrapolated by bytes; "
                      f"{nth} threads",
            "s_to_recover": full["s_to_recover"], "phases_s": full["phases_s"], "measured_s": full["measured_s"],
            "coverage": {"layout": "full", "pack": f"sampled 1/{every}",
                         "jf64": "full (committed image)" if committed else f"sampled 1/{every}",
                         "select": "full", "shard": "full", "unpack_verify": f"sampled 1/{every}"},
            "digest_check": full["checks"],
            "single_thread": {"value": one["GBps"], "cores": 1, "s_to_recover": one["s_to_recover"],
                              "phases_s": one["phases_s"],
                              "sample": f"every phase sampled at 1/{every_1t} of the chunks, extrapolated"},
            "cpu_model": cpu_model(), "nproc": os.cpu_count(), "wall_s": round(wall, 1)}


def run_reference(args):
    """The reference arm: the oracle as it stands, on the box's host cores, on
    the same config, metric and unit (capture + restore GB/s of one replica).
    Each step is the oracle's whole recovery path (OracleRecover.run) over an
    evenly spaced 1/ref_every chunk sample of the replica -- bounded so that
    --steps K --warmup W end within minutes; value = sampled bytes / step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from workloads import configs as W
    w = W.CONFIGS[args.config](world=max(args.gpus, 2) if args.config == "C1" else args.gpus)
    rec = OracleRecover(w, 0, args.ref_every)
    nth = host_threads()
    for _ in range(args.warmup):
        rec.run(nth)
    t0 = time.perf_counter()
    last = None
    for _ in range(args.steps):
        last = rec.run(nth)
    dt = (time.perf_counter() - t0) / args.steps
    v = rec.sample_bytes / dt / 1e9
    line = {"impl": "reference", "metric": "JIT capture+restore GB/s", "value": round(v, 4), "unit": "GB/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(dt * 1e3, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic (O9 counter-based generator)",
            "config": {"workload": w.name, "image_bytes": rec.L, "sample_bytes": rec.sample_bytes,
                       "note": f"oracle layout/pack/JF64/select/shard/unpack+verify over 1/{args.ref_every} of the "
                               "chunks of every group, evenly spaced"},
            "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": nth, "kind": "oracle",
                             "cpu_model": cpu_model(),
                             "sample": f"1/{args.ref_every} of the chunks of {w.name} ({rec.sample_bytes / 1e9:.2f} GB "
                                       f"of {rec.L / 1e9:.1f} GB), evenly spaced, {nth} threads",
                             "phases_s_last_step": last["measured_s"],
                             "s_to_recover_extrapolated": last["s_to_recover"]},
            "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------- jitc arm
# the failed rank of each multi-group scenario
VICTIM = {"C4": 2, "C5": 5}


def make_workload(args, world):
    """The config's synthetic state.  C1-C3 are pure DP (one replica per
    rank); C4 (ZeRO-1 hybrid S=4 x R=2) and C5 (TP4 x DP2) are 8-rank
    topologies whose victim is excluded from the healthy set.  --clip N
    clips every tensor to N elements (dry runs of the 8-rank path on one GPU,
    JITC_BENCH_SHARE_GPU=1); a clipped run is labelled in config.workload."""
    from workloads import configs as W
    if args.config in ("C1", "C2", "C3"):
        w = W.CONFIGS[args.config](world=max(world, 2) if args.config == "C1" else world)
    else:
        if world != 8:
            raise SystemExit(f"{args.config} is an 8-rank topology: run it with --gpus 8 (on a 1-GPU box: "
                             "JITC_BENCH_SHARE_GPU=1 torchrun --nproc-per-node 8 ... --clip N)")
        w = W.c4(world=8, shards=4) if args.config == "C4" else W.c5(world=8)
    if args.clip:
        w = W.scaled(w, args.clip)
        for g in w.groups:
            for t in g.tensors:
                if t.dtype == "bf16" and t.numel % 2:
                    t.numel += 1      # whole u32 words, so the synthetic update U_v covers bf16 tensors too
    return w, VICTIM.get(args.config)


def scenario_setup(args, w, J, ctx, states, rank, victim):
    """C4 (S8): one synthetic ZeRO-1 step
    from version V to V+1 on every rank -- mark(opt, DIRTY), U_{V+1} on the
    optimizer shard, mark(opt, V+1); mark(params, DIRTY), param gather,
    mark(params, V+1) -- where the victim (rank 2) dies after updating half of
    its shard, and the params gather completes only inside {4..7}, the gather
    group without the victim.  The expected selection: v* = V+1, params from
    {4..7}, shard 2 from rank 6 alone, grads (still at V) dropped.  C5: the
    state stays CLEAN at V; the victim (rank 5) simply leaves the healthy set,
    so TP partition 1 keeps a single writer (k = 1).  Untimed."""
    import torch
    if args.config != "C4":
        return
    V = 1000
    for g in w.groups:
        if rank not in g.members or g.group < 2:
            continue
        st = states[g.group]
        ctx.mark(g.group, V, J.DIRTY)
        n = len(g.tensors) if rank != victim else max(1, len(g.tensors) // 2)
        for i in range(n):
            t = g.tensors[i]
            J.inject_update(st.ptrs[i], 0, t.nbytes // 4, t.gen_id, V + 1)
        if rank != victim:
            ctx.mark(g.group, V + 1, J.CLEAN)
    pst = states[0]
    ctx.mark(0, V, J.DIRTY)
    if rank >= 4:                     # the gather group {4..7} completes the params update
        for i, t in enumerate(w.groups[0].tensors):
            J.inject_update(pst.ptrs[i], 0, t.nbytes // 4, t.gen_id, V + 1)
        ctx.mark(0, V + 1, J.CLEAN)
    torch.cuda.synchronize()


def run_jitc(args):
    import torch
    import torch.distributed as dist

    from paper_conf_eurosys_guptakkvgkrs24_b200 import build as B
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    from workloads import configs as W

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("JITC_BENCH_SHARE_GPU"):   # functional test of the N>1 path on a 1-GPU box; not a measurement
        local = 0
        if args.transport == "nccl":   # NCCL refuses two ranks per GPU on one host: one fake host per rank
            os.environ.update(NCCL_HOSTID=f"jitc-bench-host-{rank}", NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1",
                              NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0")
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    B.build()
    if world > 1:
        dist.init_process_group("gloo")

    w, victim = make_workload(args, world)
    # a fresh directory per run: the IPC transport's control block must never
    # be a stale one (a crashed earlier run with the same torchrun run id
    # would leave published IPC handles of dead processes behind)
    job = [f"{os.getpid()}-{int(time.time() * 1e3) % 10**9}"]
    if world > 1:
        dist.broadcast_object_list(job, src=0)
    job = job[0]
    shm = args.image_dir or f"/dev/shm/jitc-bench-{job}"
    # N = 1 on a box whose /dev/shm cannot hold the image: private pinned host
    # memory instead (jitc_config.image_dir = NULL, reading R16).
    # N > 1 needs the shared image (every rank loads a slice of it).
    image_kind = "shared /dev/shm"
    if world == 1 and not args.image_dir:
        need = sum(J.layout([(t.name, t.nbytes, 0) for t in g.tensors], 1 << 20)[2] for g in w.groups_of(rank))
        try:
            vfs = os.statvfs("/dev/shm")
            free = vfs.f_bavail * vfs.f_frsize
        except OSError:
            free = 0
        if args.private_image:
            shm, image_kind = None, "private pinned (--private-image)"
        elif free < need + (1 << 30):
            shm, image_kind = None, f"private pinned (/dev/shm has {free / 1e9:.1f} GB free < {need / 1e9:.1f} GB)"
            print(f"bench: {image_kind}", file=sys.stderr)
    if rank == 0 and shm and not args.image_dir:   # also on an exception: never leave a 128 GB image behind
        import atexit
        atexit.register(lambda: [shutil.rmtree(d, ignore_errors=True) for d in (shm, f"{shm}-comm", f"{shm}-comm2")])
    flags = J.F_TIME_KERNELS
    if args.zero_copy:
        flags |= J.F_ZERO_COPY_D2H | J.F_ZERO_COPY_H2D
    t_setup = time.perf_counter()
    setup = {"state_s": 0.0, "register_s": 0.0}
    ctx = J.Context(device=local, rank=rank, world=world, chunk_bytes=1 << 20,
                    staging_bytes=args.staging << 20, slot_bytes=args.slot << 20, image_dir=shm, flags=flags)
    states = {}
    L_total = 0
    for g in w.groups_of(rank):
        t0 = time.perf_counter()
        st = GroupState(g, w.seed, device=local)
        states[g.group] = st
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        lh, L = ctx.register(g.group, g.policy, g.members, st.table(), keepalive=st)
        setup["state_s"] += t1 - t0
        setup["register_s"] += time.perf_counter() - t1
        L_total += L
        ctx.mark(g.group, 1000, J.CLEAN)
    L_group = {g.group: J.layout([(t.name, t.nbytes, 0) for t in g.tensors], 1 << 20)[2] for g in w.groups}
    L_unique = sum(L_group.values())     # every distinct byte of the job's state (one replica per group)
    fanout = args.capture == "fanout" or (args.capture == "auto" and args.config in ("C4", "C5") and world > 1)
    for g in w.groups:
        if rank not in g.members:
            ctx.declare_group(g.group, g.policy, g.members)
            if fanout:   # a fan-out mover D2Hs lanes of groups it does not hold (steady-state attach)
                t1 = time.perf_counter()
                ctx.attach_image(g.group, L_group[g.group])
                setup["register_s"] += time.perf_counter() - t1
    scenario_setup(args, w, J, ctx, states, rank, victim)
    t_comm = time.perf_counter()
    if world > 1:
        if args.transport == "nccl":
            uid = [J.get_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            ctx.comm_init(uid[0], world, rank)
        else:   # intra-node CUDA IPC transport (fresh directory per communicator)
            ctx.comm_init_ipc(f"{shm}-comm", world, rank)
    comm_init_ms = (time.perf_counter() - t_comm) * 1e3
    torch.cuda.synchronize()
    setup_s = time.perf_counter() - t_setup
    nccl_group = None
    if world > 1 and not os.environ.get("JITC_BENCH_SHARE_GPU"):
        nccl_group = dist.new_group(backend="nccl")

    healthy = [r for r in range(world) if r != victim]
    per = {"fingerprint": [], "select": [], "capture": [], "commit": [], "restore": [], "verify": []}
    launches = [0]

    last_blob, last_sel = [None], [None]
    last_cap = [(0, 0.0)]              # this rank's D2H bytes and capture seconds of the last step
    moved = {"d2h": [], "h2d": []}   # this rank's host-link bytes per timed step
    p2p_k3 = []                       # restore bytes K3 read from peers' staging (IPC) per timed step

    def step(record: bool, use_fanout=None):
        t = {}
        t0 = time.perf_counter()
        blob = ctx.fingerprint()
        last_blob[0] = blob
        t1 = time.perf_counter()
        allb = ctx.exchange_records(blob)
        st_, sel = J.select_consistent_replica(allb, healthy)
        if st_ != J.OK:
            raise RuntimeError(f"select: {J.parse_selection(sel)}")
        t2 = time.perf_counter()
        cap = ctx.capture_fanout(sel, healthy) if (fanout if use_fanout is None else use_fanout) else ctx.capture(sel)
        t3 = time.perf_counter()
        last_cap[0] = (cap["d2h_bytes"], t3 - t2)
        ctx.commit(sel)
        t4 = time.perf_counter()
        res = ctx.restore(J.ALL_GROUPS, J.HOST)
        t5 = time.perf_counter()
        kept = {gs["group"] for gs in J.parse_selection(sel)["groups"] if gs["writers"]}
        for gid in states:
            if gid in kept:          # a dropped OPTIONAL group has no checkpoint to verify against
                ctx.verify(gid)
        t6 = time.perf_counter()
        last_sel[0] = sel
        if record:
            for k, (a, b) in zip(per, [(t0, t1), (t1, t2), (t2, t3), (t3, t4), (t4, t5), (t5, t6)]):
                per[k].append((b - a) * 1e3)
            launches[0] += cap["kernel_launches"] + res["kernel_launches"] + 2 * len(states)
            moved["d2h"].append(cap["d2h_bytes"])
            moved["h2d"].append(res["h2d_bytes"])
            p2p_k3.append(res["p2p_bytes"])
        return cap, res, len(allb)

    for _ in range(args.warmup):
        step(False)
    # link calibration after the warm-up steps, when the host image's pages and
    # the pinned buffers are settled (one box read 41 GB/s D2H right after
    # registering 25 GB, 56 GB/s later); still outside the timed region
    links = calibrate_links(local, world, nccl_group) if not args.no_calibrate else None
    f3 = per_tensor_d2h(states, local, world) if not args.no_calibrate else None
    # Settling (untimed): a job registers its host image at start-up, long
    # before a failure.  On some boxes the D2H into a freshly registered image
    # ran far below the link for tens of seconds (35.7 GB/s in one run's timed
    # steps, recovering to 54.5 GB/s a minute later, while D2H into fresh
    # cudaHostAlloc memory ran at 55.7; profiles/r02f_pin_fused_ab.txt).  So
    # extra untimed steps run, at most --settle-max, while any rank's last
    # capture of >= 4 GiB moved its bytes below 0.9 of its calibrated D2H;
    # the count is reported as config.settle_steps.
    settle = 0
    if links and args.settle_max > 0:
        while True:
            b, t = last_cap[0]
            # only captures long enough to be link-bound (>= 4 GiB per rank) are judged
            slow = 1.0 if (b >= (4 << 30) and t > 0 and b / t / 1e9 < 0.9 * links["d2h_GBps"]) else 0.0
            if world > 1:
                f = torch.tensor([slow], dtype=torch.float64)
                dist.all_reduce(f, op=dist.ReduceOp.MAX)
                slow = f.item()
            if not slow or settle >= args.settle_max:
                break
            step(False)
            settle += 1
    ctx.reset_counters()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        wall0 = time.perf_counter()
        e0.record()
        for _ in range(args.steps):
            cap, res, rec_bytes = step(True)
        e1.record()
        torch.cuda.synchronize()
        wall1 = time.perf_counter()
    if world > 1:
        dist.barrier()
    ms_step = e0.elapsed_time(e1) / args.steps
    ms_step_wall = (wall1 - wall0) * 1e3 / args.steps
    med = {k: statistics.median(v) for k, v in per.items()}
    link_bytes = [max(moved["d2h"]), max(moved["h2d"])]
    if world > 1:   # max over ranks: step times, phase medians, per-rank host-link bytes
        tt = torch.tensor([ms_step, ms_step_wall] + [med[k] for k in per] + link_bytes, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        vals = tt.tolist()
        ms_step, ms_step_wall = vals[:2]
        med = dict(zip(per, vals[2:2 + len(per)]))
        link_bytes = vals[2 + len(per):]
    sel_info = J.parse_selection(last_sel[0])

    # kernel counters of the timed region only (the extra variants below launch more)
    kc_timed = {k: ctx.kernel_counters(k) for k in (J.K_DIGEST, J.K_PACK, J.K_UNPACK)}

    # the paper's own protocol as an in-run comparison (
    # PAPER.md:108, :136): every healthy rank saves its FULL state (k = 1 per
    # rank, n * L over the host links) instead of a 1/k shard.  N > 1 only.
    paper_protocol = None
    if world > 1 and not args.no_paper_protocol and args.config in ("C1", "C2", "C3"):
        dist.barrier()
        t0 = time.perf_counter()
        ctx.capture_local()
        dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64)
        dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        paper_protocol = {"what": "every rank saves its full replica (own fingerprint, k=1 capture, commit); "
                                  "host wall clock, max over ranks",
                          "capture_s": round(dt.item(), 4), "host_link_bytes_total": world * L_total,
                          "sharded_capture_s": round(statistics.median(per["capture"]) * 1e-3, 4),
                          "sharded_host_link_bytes_total": L_total}

    # PEER restore (SURVEY.md §8(d) d.5 "PEER restore"; PAPER.md:174, :184 copy
    # from a replica): the victim (the last rank for C1-C3) plays the
    # replacement.  The survivors take the selection over their own records;
    # the replacement's state is overwritten and it calls jitc_restore(PEER)
    # WITHOUT a selection -- it receives the selection and the writers'
    # digests over the communicator -- while the writers
    # pack their O5 ranges from live HBM and send them (NVLink on a multi-GPU
    # box) and every non-writer member unpacks + verifies.  Max over ranks,
    # host wall clock.
    peer_restore = None
    if world > 1 and not args.no_peer_restore:
        repl = victim if victim is not None else world - 1
        blob = ctx.fingerprint()
        allb = ctx.exchange_records(blob)
        st_p, sel_p = J.select_consistent_replica(allb, [r for r in range(world) if r != repl])
        if st_p != J.OK:
            raise RuntimeError(f"peer select: {J.parse_selection(sel_p)}")
        kept_p = {gs["group"] for gs in J.parse_selection(sel_p)["groups"] if gs["writers"]}
        if rank == repl:
            for st in states.values():
                st.scramble()
        torch.cuda.synchronize()
        dist.barrier()
        t0 = time.perf_counter()
        res_p = ctx.restore(J.ALL_GROUPS, J.PEER, None if rank == repl else sel_p)
        if rank == repl:
            for gid in states:
                if gid in kept_p:
                    ctx.verify(gid)
        dt = torch.tensor([time.perf_counter() - t0], dtype=torch.float64)
        dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        pb = torch.tensor([res_p["p2p_bytes"] if rank == repl else 0], dtype=torch.float64)
        dist.all_reduce(pb, op=dist.ReduceOp.MAX)
        lr = torch.tensor([L_total if rank == repl else 0], dtype=torch.float64)
        dist.all_reduce(lr, op=dist.ReduceOp.MAX)
        peer_restore = {"replacement": repl, "writers_k": {gs["group"]: len(gs["writers"])
                                                           for gs in J.parse_selection(sel_p)["groups"]},
                        "s": round(dt.item(), 4), "replacement_state_bytes": int(lr.item()),
                        "GBps": round(lr.item() / dt.item() / 1e9, 3), "replacement_ingress_bytes": int(pb.item()),
                        "transport": args.transport, "replacement_passed_selection": False,
                        "how": "selection over the survivors; the replacement's tensors overwritten first; "
                               "jitc_restore(PEER) on every rank (the replacement without a selection) + "
                               "jitc_verify on the replacement; host wall clock, max over ranks"}

    # NVLink fan-out vs plain sharded capture:
    # one more step with the other capture mode, untimed by the main clock;
    # capture phase on the host clock, max over ranks.
    capture_compare = None
    if world > 1 and args.config in ("C4", "C5"):
        dist.barrier()
        t0 = time.perf_counter()
        blob = ctx.fingerprint()
        st_c, sel_c = J.select_consistent_replica(ctx.exchange_records(blob), healthy)
        t1 = time.perf_counter()
        ctx.capture(sel_c) if fanout else ctx.capture_fanout(sel_c, healthy)
        t2 = time.perf_counter()
        ctx.commit(sel_c)
        t3 = time.perf_counter()
        tt = torch.tensor([t3 - t0], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        other = tt.item() * 1e3
        mine = med["fingerprint"] + med["select"] + med["capture"] + med["commit"]
        capture_compare = {"fanout_T_capture_ms": round(mine if fanout else other, 2),
                           "plain_T_capture_ms": round(other if fanout else mine, 2),
                           "movers": healthy,
                           "how": "T_capture (fingerprint -> commit) of the timed mode (median) and of one step "
                                  "of the other mode; max over ranks"}

    # robustness variant: one more step while an emulated
    # hung collective (32 spinning CTAs on another stream) occupies the GPU,
    # as when a NCCL kernel waits forever on a dead peer
    under_hang = None
    if args.hang_ctas > 0:
        hs = torch.cuda.Stream()
        J.inject_hang(hs.cuda_stream, args.hang_ctas, slot=5)
        try:
            t0 = time.perf_counter()
            cap_h, res_h, _ = step(False)
            dt = time.perf_counter() - t0
        finally:
            J.inject_release(5)
        hs.synchronize()
        under_hang = {"hung_ctas": args.hang_ctas, "step_s": round(dt, 4),
                      "value_GBps": round(L_unique / dt / 1e9, 3),
                      "capture_GBps": round(cap_h["image_bytes"] / (cap_h["ms_host"] * 1e-3) / 1e9, 3),
                      "restore_GBps": round(res_h["image_bytes"] / (res_h["ms_host"] * 1e-3) / 1e9, 3)}

    # NEXT-1: the native watchdog detects
    # an emulated hung collective and captures on its own thread.  N = 1 only:
    # waited = event age when the watchdog fired (>= the timeout), action =
    # fingerprint -> select -> capture -> commit run by the watchdog thread.
    on_hang = None
    if world == 1 and args.hang_ctas > 0 and not args.no_watchdog:
        hs = torch.cuda.Stream()
        J.inject_hang(hs.cuda_stream, args.hang_ctas, slot=6)
        ev = torch.cuda.Event()
        ev.record(hs)
        try:
            ctx.watch_event(ev.cuda_event, tag=7)
            ctx.watchdog_start(timeout_ms=args.watchdog_ms, action=J.ON_HANG_LOCAL_CAPTURE)
            r = ctx.watchdog_wait(120000)
        finally:
            J.inject_release(6)
        hs.synchronize()
        ctx.watchdog_stop()
        st_w = r["stats"]
        on_hang = {"timeout_ms": args.watchdog_ms, "fired": r["fired"], "waited_ms": round(r["waited_ms"], 2),
                   "detect_overshoot_ms": round(r["waited_ms"] - args.watchdog_ms, 2),
                   "action_ms": round(r["action_ms"], 1),
                   "capture_GBps": round(st_w["image_bytes"] / (r["action_ms"] * 1e-3) / 1e9, 2)
                   if r["action_ms"] else None,
                   "hung_ctas": args.hang_ctas,
                   "how": "jitc_watchdog_start(ON_HANG_LOCAL_CAPTURE) on an event after spinning CTAs; the "
                          "action (fingerprint, own select, capture, commit) runs on the watchdog thread"}

    # communicator rebuild (SURVEY.md §8(d) d.6 T_comm; the paper's dominant
    # recovery cost, Table 7): the survivors drop the last rank
    # (jitc_comm_shrink), then all ranks build a fresh communicator including a
    # "replacement" (jitc_comm_init / _ipc).  Host wall clock, max over ranks.
    comm_rebuild = None
    if world > 1 and not args.no_comm_rebuild:
        gone = victim if victim is not None else world - 1
        dist.barrier()
        t0 = time.perf_counter()
        if rank != gone:
            ctx.comm_shrink([gone])
        t_shrink = time.perf_counter() - t0
        dist.barrier()
        if args.transport == "nccl":
            uid = [J.get_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
        dist.barrier()
        t0 = time.perf_counter()
        if args.transport == "nccl":
            ctx.comm_init(uid[0], world, rank)
        else:
            ctx.comm_init_ipc(f"{shm}-comm2", world, rank)
        t_init = time.perf_counter() - t0
        tt = torch.tensor([t_shrink, t_init], dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        comm_rebuild = {"transport": args.transport, "shrink_ms": round(tt[0].item() * 1e3, 2),
                        "reinit_ms": round(tt[1].item() * 1e3, 2),
                        "how": f"survivors shrink away rank {gone}, then all {world} ranks init a new "
                               "communicator (warm-up included); host wall clock, max over ranks"}

    # per-kernel rooflines, the dominant kernel (the
    # largest summed CUDA-event time in the timed region) reported as
    # `roofline`.  Algorithmic bytes per launch: K1 reads its range once; K2
    # reads the tensors and writes staging; K3 reads a staging block and writes
    # the tensors.  With the IPC transport at N > 1 a K3 launch reads the
    # blocks of the other n-1 ranks straight from THEIR staging over NVLink
    # (the stats' p2p bytes): those bytes are NVLink ingress, not local HBM
    # reads, and the kernel's bound is whichever of HBM (local bytes) and
    # NVLink (remote bytes, measured peer-copy reference 770 GB/s per direction,
    # or this run's calibration) it runs closer to.
    kinds = {J.K_DIGEST: "K1_digest", J.K_PACK: "K2_pack_digest", J.K_UNPACK: "K3_unpack_verify"}
    kc = kc_timed
    peak, peak_src = _peaks()
    nvl_peak, nvl_src = (links["nvl_allgather_busbw_GBps"], "this run's NCCL all-gather bus bandwidth") \
        if links and "nvl_allgather_busbw_GBps" in links else (770.0, "B200_PROFILING.md measured peer copy, 770 GB/s")
    remote_k3 = sum(p2p_k3) if args.transport == "ipc" else 0

    def kernel_roof(k):
        c = kc[k]
        n = max(c["launches"], 1)
        ms = c["ms"] / n
        if ms <= 0:
            return None
        io = c["bytes"] / n                      # image bytes per launch
        remote = remote_k3 / n if k == J.K_UNPACK else 0
        local = (1 if k == J.K_DIGEST else 2) * io - remote
        out = {"kernel": kinds[k], "launches": c["launches"], "ms_per_launch": round(ms, 4),
               "image_bytes_per_launch": io, "hbm": {"bytes_per_launch": local,
                                                     "achieved": round(local / (ms * 1e-3) / 1e9, 1),
                                                     "frac": round(local / (ms * 1e-3) / 1e9 / peak, 4)}}
        out["bound"] = "hbm"
        if k == J.K_DIGEST and links and links.get("hbm_read_GBps"):   # K1 only reads: also vs a read-only rate
            out["hbm"]["frac_of_read_calibration"] = round(local / (ms * 1e-3) / 1e9 / links["hbm_read_GBps"], 4)
        if remote:
            out["nvlink"] = {"bytes_per_launch": remote, "achieved": round(remote / (ms * 1e-3) / 1e9, 1),
                             "frac": round(remote / (ms * 1e-3) / 1e9 / nvl_peak, 4)}
            if out["nvlink"]["frac"] > out["hbm"]["frac"]:
                out["bound"] = "nvlink"
        span = c.get("span_ms", 0.0) / n
        if span > 0:
            out["kernel_span_ms_per_launch"] = round(span, 4)
        return out

    roofs = {kinds[k]: kernel_roof(k) for k in kinds}
    dom = max(kc, key=lambda k: kc[k]["ms"])
    rd = roofs[kinds[dom]]
    bnd = rd["bound"] if rd else "hbm"
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp) and rd:
        tr = json.load(open(tp)).get(kinds[dom])
        if tr:
            traffic = tr["dram_bytes"] / tr["image_bytes"] * rd["image_bytes_per_launch"]
    roofline = None
    if rd:
        b = rd[bnd]
        span = rd.get("kernel_span_ms_per_launch")
        roofline = {"kernel": kinds[dom], "bound": bnd, "achieved": b["achieved"],
                    "peak": peak if bnd == "hbm" else nvl_peak, "unit": "GB/s", "frac": b["frac"],
                    "traffic": traffic if bnd == "hbm" else None,
                    "peak_source": peak_src if bnd == "hbm" else nvl_src,
                    "bytes_per_launch": b["bytes_per_launch"], "ms_per_launch": rd["ms_per_launch"],
                    "launches": rd["launches"],
                    "kernel_span": {"ms_per_launch": span,
                                    "achieved": round(b["bytes_per_launch"] / (span * 1e-3) / 1e9, 1) if span else None,
                                    "frac": round(b["bytes_per_launch"] / (span * 1e-3) / 1e9 /
                                                  (peak if bnd == "hbm" else nvl_peak), 4) if span else None,
                                    "how": "diagnostic: %globaltimer first-CTA-start to last-CTA-end per launch; "
                                           "`achieved` above is the CUDA-event figure"}}

    if rank == 0:
        value = L_unique / (ms_step * 1e-3) / 1e9
        e2e = L_unique / (ms_step_wall * 1e-3) / 1e9
        med = {k: round(v, 3) for k, v in med.items()}
        # T_capture runs from jitc_fingerprint start to
        # jitc_commit return; T_restore from jitc_restore start to jitc_verify OK
        cap_ms = med["fingerprint"] + med["select"] + med["capture"] + med["commit"]
        res_ms = med["restore"] + med["verify"]
        line = {
            "metric": "JIT capture+restore GB/s", "value": round(value, 3), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 3),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic training state (O9 integer generator; bf16 params, fp32 master/m/v, bf16 grads)",
            "config": {"workload": w.name, "image_bytes": L_unique, "rank0_image_bytes": L_total,
                       "tensors": sum(len(g.tensors) for g in w.groups), "clip": args.clip or None,
                       "writers_k": {gs["group"]: len(gs["writers"]) for gs in sel_info["groups"]},
                       "restore_mode": "HOST", "image": image_kind,
                       "capture": "fanout" if fanout else "sharded", "victim": victim,
                       "transport": args.transport if world > 1 else None,
                       "comm_init_ms": round(comm_init_ms, 1) if world > 1 else None,
                       "zero_copy": bool(args.zero_copy), "chunk_bytes": 1 << 20,
                       "staging_mib": args.staging, "slot_mib": args.slot,
                       "l2": f"state {L_total / 1e9:.1f} GB >> 126 MB L2; no flush needed", "setup_s": round(setup_s, 1),
                       "setup_breakdown_s": {k: round(v, 1) for k, v in setup.items()},
                       "settle_steps": settle},
            "seconds_to_recover": round(ms_step * 1e-3, 4),
            "phases_ms_median": med,
            "capture_GBps": round(L_unique / (cap_ms * 1e-3) / 1e9, 3),
            "restore_GBps": round(L_unique / (res_ms * 1e-3) / 1e9, 3),
            "selection": {"v_star": sel_info["v_star"], "healthy": healthy,
                          "groups": [{"group": gs["group"], "policy": gs["policy"], "status": gs["status"],
                                      "k": len(gs["writers"]), "writers": gs["writers"],
                                      "excluded": gs["excluded"]} for gs in sel_info["groups"]]},
            "capture_compare": capture_compare,
            "capture_restore_spans": {"T_capture_ms": round(cap_ms, 3), "T_restore_ms": round(res_ms, 3),
                                      "how": "SURVEY.md d.6: T_capture = fingerprint + exchange/select + capture + "
                                             "commit; T_restore = restore + verify (medians over the timed steps)"},
            "host_link_roofline": host_link_roofline(link_bytes[0], link_bytes[1], med["capture"], med["restore"],
                                                     links),
            "per_tensor_d2h_baseline": f3,
            "roofline": roofline,
            "kernels": roofs,
            "e2e": {"value": round(e2e, 3), "unit": "GB/s", "h2d_bytes_per_step": L_unique,
                    "d2h_bytes_per_step": L_unique + rec_bytes,
                    "note": "host wall clock around the public Python API step (ctypes, manifest file I/O included)"},
            "gpu_launches": launches[0],
            "under_hang": under_hang,
            "paper_protocol": paper_protocol,
            "peer_restore": peer_restore,
            "comm_rebuild": comm_rebuild,
            "watchdog_on_hang": on_hang,
            "clocks": clk.summary(),
        }
        if not args.no_cpu_baseline and world == 1:
            from oracle import oracle as O
            [(_, _, _, recs)] = O.decode_blobs(last_blob[0])
            committed = ({gid: np.memmap(f"{shm}/g{gid}.img", dtype=np.uint8, mode="r") for gid in states}
                         if shm else None)
            line["cpu_baseline"] = cpu_baseline(w, rank, last_blob[0], committed, {r.group: r.d for r in recs},
                                                args.cpu_every, args.cpu_every_1t)
            del committed
        print(json.dumps(line), flush=True)
    ctx.close()
    if world > 1:
        dist.barrier()
    if rank == 0 and shm and not args.image_dir:
        shutil.rmtree(shm, ignore_errors=True)
        shutil.rmtree(f"{shm}-comm", ignore_errors=True)
        shutil.rmtree(f"{shm}-comm2", ignore_errors=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3", choices=["C1", "C2", "C3", "C4", "C5"],
                    help="workload (SURVEY.md §8(d) d.1); C3 = Llama-3-8B, the north-star shape and the largest "
                         "single-GPU config")
    ap.add_argument("--impl", default="jitc", choices=["jitc", "reference"])
    ap.add_argument("--clip", type=int, default=0,
                    help="clip every tensor to N elements (8-rank dry runs of C4/C5 on one GPU; labelled)")
    ap.add_argument("--capture", default="auto", choices=["auto", "sharded", "fanout"],
                    help="auto: NVLink fan-out for C4/C5 at N > 1 (k = 1 groups), plain sharded capture otherwise")
    ap.add_argument("--staging", type=int, default=16384, help="MiB of device staging (2 round slots)")
    ap.add_argument("--slot", type=int, default=8192,
                    help="MiB per pipeline round (8 GiB: the ~42 us cost of a timing-event record next to a "
                         "copy-engine transfer is amortised over 17 GB of K2/K3 traffic; DESIGN.md §7)")
    ap.add_argument("--zero-copy", action="store_true")
    ap.add_argument("--image-dir", default=None)
    ap.add_argument("--private-image", action="store_true",
                    help="N = 1: private pinned host image (image_dir = NULL) instead of /dev/shm; also chosen "
                         "automatically when /dev/shm cannot hold the image")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-paper-protocol", action="store_true",
                    help="N > 1: skip the in-run comparison with the paper's every-rank-saves-everything protocol")
    ap.add_argument("--no-watchdog", action="store_true", help="N = 1: skip the watchdog on-hang capture variant")
    ap.add_argument("--watchdog-ms", type=int, default=200, help="watchdog hang timeout for that variant")
    ap.add_argument("--no-comm-rebuild", action="store_true", help="N > 1: skip timing shrink + re-init")
    ap.add_argument("--no-peer-restore", action="store_true", help="N > 1: skip the PEER-restore variant")
    ap.add_argument("--settle-max", type=int, default=8,
                    help="at most this many extra untimed steps while the capture D2H runs below 0.9 of the "
                         "calibrated link (a freshly registered image; reported as config.settle_steps)")
    ap.add_argument("--no-calibrate", action="store_true", help="skip the in-run host-link / HBM / NVLink calibration")
    ap.add_argument("--hang-ctas", type=int, default=32, help="CTAs of the emulated hung collective (0 = skip)")
    ap.add_argument("--transport", default="ipc", choices=["ipc", "nccl"],
                    help="N > 1 communicator: intra-node CUDA IPC (default; tested on B200 with real processes) or NCCL")
    ap.add_argument("--ref-every", type=int, default=128,
                    help="reference arm: every step runs the oracle on 1/ref-every of the chunks")
    ap.add_argument("--cpu-every", type=int, default=16,
                    help="cpu_baseline: pack / unpack+verify sampled on 1/cpu-every of the chunks (1 = full state)")
    ap.add_argument("--cpu-every-1t", type=int, default=128, help="cpu_baseline 1-thread leg: sample 1/N of the chunks")
    args = ap.parse_args()
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.impl == "reference":
        run_reference(args)
    else:
        run_jitc(args)


if __name__ == "__main__":
    main()
