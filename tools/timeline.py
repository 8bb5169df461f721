"""Overlap evidence for the capture and restore pipelines (VERDICT r01
missing #7; nsys is not installed on the boxes): one fingerprint -> select ->
capture -> commit -> restore(HOST) -> verify pass of a config in bench.py's
launch configuration, with every kernel launch and copy-engine batch
recorded as a span (jitc_timeline_start / _read: CUDA events on the launching
stream).  Writes a Chrome trace (chrome://tracing, Perfetto) and a summary:
how much of K2 runs under the D2H copies during capture, and of K3 under the
H2D copies during restore.

    python tools/timeline.py [--config C3] [--slot 8192] [--staging 16384] --out profiles/r02_timeline_c3
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def union(iv):
    out = []
    for a, b in sorted(iv):
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def length(iv):
    return sum(b - a for a, b in iv)


def intersect(x, y):
    i = j = 0
    out = []
    while i < len(x) and j < len(y):
        a, b = max(x[i][0], y[j][0]), min(x[i][1], y[j][1])
        if a < b:
            out.append([a, b])
        if x[i][1] < y[j][1]:
            i += 1
        else:
            j += 1
    return out


def overlap_report(spans, kern, copy, t0, t1):
    k = union([(s["t0_ms"], s["t1_ms"]) for s in spans if s["kind"] == kern and t0 <= s["t0_ms"] <= t1])
    c = union([(s["t0_ms"], s["t1_ms"]) for s in spans if s["kind"] == copy and t0 <= s["t0_ms"] <= t1])
    both = intersect(k, c)
    span = (max(b for _, b in k + c) - min(a for a, _ in k + c)) if (k or c) else 0.0
    return {f"{kern}_busy_ms": round(length(k), 3), f"{copy}_busy_ms": round(length(c), 3),
            "overlap_ms": round(length(both), 3), "phase_span_ms": round(span, 3),
            f"{kern}_hidden_under_{copy}": round(length(both) / length(k), 4) if k else None,
            f"{copy}_busy_frac_of_span": round(length(c) / span, 4) if span else None,
            f"{kern}_exposed_ms": round(length(k) - length(both), 3)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--slot", type=int, default=8192)
    ap.add_argument("--staging", type=int, default=16384)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r02_timeline"))
    args = ap.parse_args()
    import torch
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build as B
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    from workloads import configs as W
    B.build()
    w = W.CONFIGS[args.config](world=1)
    shm = f"/dev/shm/jitc-timeline-{os.getpid()}"
    ctx = J.Context(device=0, chunk_bytes=1 << 20, staging_bytes=args.staging << 20, slot_bytes=args.slot << 20,
                    image_dir=shm)
    states = {}
    for g in w.groups:
        states[g.group] = GroupState(g, w.seed)
        ctx.register(g.group, g.policy, [0], states[g.group].table(), keepalive=states[g.group])
        ctx.mark(g.group, 7, J.CLEAN)
    try:
        def step(tl):
            marks = {}
            if tl:
                ctx.timeline_start(8192)
            t = time.perf_counter()
            blob = ctx.fingerprint()
            st, sel = J.select_consistent_replica(ctx.exchange_records(blob), [0])
            assert st == J.OK
            ctx.capture(sel)
            ctx.commit(sel)
            marks["capture_host_ms"] = (time.perf_counter() - t) * 1e3
            t = time.perf_counter()
            ctx.restore(J.ALL_GROUPS, J.HOST)
            for gid in states:
                ctx.verify(gid)
            marks["restore_host_ms"] = (time.perf_counter() - t) * 1e3
            return (ctx.timeline_read() if tl else None), marks

        step(False)                       # warm-up: pages settled, kernels loaded
        spans, marks = step(True)
    finally:
        ctx.close()
        import shutil
        shutil.rmtree(shm, ignore_errors=True)
    # phases: capture = up to the last D2H; restore = from the first H2D
    d2h_end = max(s["t1_ms"] for s in spans if s["kind"] == "D2H")
    h2d_start = min(s["t0_ms"] for s in spans if s["kind"] == "H2D")
    rep = {"config": w.name, "slot_mib": args.slot, "staging_mib": args.staging, "spans": len(spans),
           "host_ms": {k: round(v, 2) for k, v in marks.items()},
           "capture": overlap_report(spans, "K2", "D2H", 0.0, d2h_end),
           "restore": overlap_report(spans, "K3", "H2D", h2d_start, float("inf")),
           "how": "CUDA events around every kernel launch and copy batch of one step (jitc_timeline_*); each "
                  "event record costs ~40 us next to a copy-engine transfer, so the spans are slightly longer "
                  "than in the bench's timed steps"}
    trace = [{"name": s["kind"] + (f" g{s['group']} r{s['round']}"), "ph": "X", "pid": 0,
              "tid": "copy engine" if s["stream"] else "compute",
              "ts": s["t0_ms"] * 1e3, "dur": (s["t1_ms"] - s["t0_ms"]) * 1e3,
              "args": {"bytes": s["bytes"], "GBps": round(s["bytes"] / max(s["t1_ms"] - s["t0_ms"], 1e-9) / 1e6, 1)}}
             for s in spans]
    json.dump({"traceEvents": trace, "displayTimeUnit": "ms"}, open(args.out + ".trace.json", "w"))
    json.dump(rep, open(args.out + ".summary.json", "w"), indent=1)
    print(json.dumps(rep, indent=1))


if __name__ == "__main__":
    main()
