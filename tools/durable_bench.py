"""NEXT-4 durable tier throughput (VERDICT r01 item 8; PAPER.md:341, :356
§6.3): capture + commit a config's state into the /dev/shm image, then
jitc_persist it to a directory on the box's disk (parallel O_DIRECT writes,
fdatasync, manifest, commit record last) and jitc_stage_in it back (commit
record, trailer and layout checked), then a HOST restore verifies every chunk
against the manifest.  Prints one JSON line with GB/s of both directions and
the file system the directory is on.

    python tools/durable_bench.py [--config C2] [--dir /tmp/jitc-durable]
"""
import argparse
import json
import os
import shutil
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--dir", default="/tmp/jitc-durable")
    args = ap.parse_args()
    import torch
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build as B
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    from workloads import configs as W
    B.build()
    w = W.CONFIGS[args.config](world=1)
    os.makedirs(args.dir, exist_ok=True)
    st = os.statvfs(args.dir)
    free = st.f_bavail * st.f_frsize
    g = w.groups[0]
    if g.nbytes * 1.05 > free:
        raise SystemExit(f"{args.dir}: {free / 1e9:.1f} GB free < {g.nbytes / 1e9:.1f} GB")
    fs = subprocess.run(["df", "-T", args.dir], capture_output=True, text=True).stdout.splitlines()[-1]
    shm = f"/dev/shm/jitc-durable-{os.getpid()}"
    ctx = J.Context(device=0, chunk_bytes=1 << 20, staging_bytes=8 << 30, slot_bytes=4 << 30, image_dir=shm)
    try:
        s = GroupState(g, w.seed)
        ctx.register(g.group, g.policy, [0], s.table(), keepalive=s)
        ctx.mark(g.group, 3, J.CLEAN)
        blob = ctx.fingerprint()
        rc, sel = J.select_consistent_replica(ctx.exchange_records(blob), [0])
        ctx.capture(sel)
        ctx.commit(sel)
        t = time.perf_counter()
        p = ctx.persist(g.group, args.dir)
        t_p = time.perf_counter() - t
        with open(f"{shm}/g{g.group}.img", "r+b") as f:    # lose the host image
            f.write(b"\0" * (1 << 20))
        subprocess.run(["sync"])
        cold = True
        try:
            with open("/proc/sys/vm/drop_caches", "w") as f:  # read the copy from the device, not the page cache
                f.write("1\n")
        except OSError:
            cold = False
        t = time.perf_counter()
        q = ctx.stage_in(g.group, args.dir)
        t_s = time.perf_counter() - t
        s.scramble()
        r = ctx.restore(g.group, J.HOST)
        ctx.verify(g.group, blob)
        out = {"config": w.name, "group_bytes": r["image_bytes"], "dir": args.dir, "fs": fs,
               "persist_s": round(t_p, 3), "persist_GBps": round(p["image_bytes"] / t_p / 1e9, 3),
               "stage_in_s": round(t_s, 3), "stage_in_GBps": round(q["image_bytes"] / t_s / 1e9, 3),
               "page_cache_dropped_before_stage_in": cold,
               "restore_after_stage_in": "bit-exact (every chunk digest == manifest; verify == fingerprint)"}
        print(json.dumps(out), flush=True)
    finally:
        ctx.close()
        shutil.rmtree(shm, ignore_errors=True)
        shutil.rmtree(args.dir, ignore_errors=True)


if __name__ == "__main__":
    main()
