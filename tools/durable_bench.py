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


def raw_disk(dirpath: str, nbytes: int, threads: int = 8, piece: int = 64 << 20) -> dict:
    """The disk's own rate for the library's access pattern (the NEXT-4
    roofline): `threads` threads pwrite / pread 64 MiB pieces of one file with
    O_DIRECT, fdatasync after the writes, page cache dropped before the reads."""
    import mmap
    import threading
    path = os.path.join(dirpath, "raw-baseline.bin")
    buf = mmap.mmap(-1, piece)                      # page-aligned, as O_DIRECT needs
    buf.write(os.urandom(1 << 20) * (piece >> 20))

    def run(write: bool) -> float:
        flags = (os.O_WRONLY | os.O_CREAT | os.O_TRUNC) if write else os.O_RDONLY
        fd = os.open(path, flags | getattr(os, "O_DIRECT", 0), 0o600)
        if write:
            os.ftruncate(fd, nbytes)
        mv = memoryview(buf)

        def work(t):
            for off in range(t * piece, nbytes, threads * piece):
                n = min(piece, nbytes - off)
                if write:
                    os.pwrite(fd, mv[:n], off)
                else:
                    os.preadv(fd, [mv[:n]], off)
        t0 = time.perf_counter()
        ths = [threading.Thread(target=work, args=(t,)) for t in range(threads)]
        for th in ths:
            th.start()
        for th in ths:
            th.join()
        if write:
            os.fdatasync(fd)
        dt = time.perf_counter() - t0
        os.close(fd)
        return nbytes / dt / 1e9
    w = run(True)
    subprocess.run(["sync"])
    try:
        with open("/proc/sys/vm/drop_caches", "w") as f:
            f.write("1\n")
    except OSError:
        pass
    r = run(False)
    os.unlink(path)
    return {"bytes": nbytes, "threads": threads, "piece_MiB": piece >> 20, "write_GBps": round(w, 3),
            "read_GBps": round(r, 3), "how": "O_DIRECT pwrite/pread of 64 MiB pieces, fdatasync, cache dropped"}


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
        raw = raw_disk(args.dir, min(g.nbytes, 16 << 30), threads=int(os.environ.get("JITC_DURABLE_THREADS", 8)))
        out["raw_disk"] = raw
        out["persist_frac_of_raw_write"] = round(out["persist_GBps"] / raw["write_GBps"], 3)
        out["stage_in_frac_of_raw_read"] = round(out["stage_in_GBps"] / raw["read_GBps"], 3)
        print(json.dumps(out), flush=True)
    finally:
        ctx.close()
        shutil.rmtree(shm, ignore_errors=True)
        shutil.rmtree(args.dir, ignore_errors=True)


if __name__ == "__main__":
    main()
