"""Profiling driver for ncu: a ~2 GiB prefix of the C2 state, one fingerprint
(K1), capture (K2, staging+CE), restore (K3), verify -- the same kernels and
launch configuration bench.py times, on a smaller state so that ncu's
save/restore replays stay cheap.

    ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 2 -c 6 \
        -o gpurun_out/prof python tools/prof_kernels.py
"""
import copy
import os
import shutil
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J  # noqa: E402
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState  # noqa: E402
from workloads import configs as W  # noqa: E402


def main(budget=int(os.environ.get("PROF_BYTES", 2 << 30)), reps=int(os.environ.get("PROF_REPS", 2))):
    w = W.c2()
    g = copy.deepcopy(w.groups[0])
    keep, tot = [], 0
    for t in g.tensors:
        if tot >= budget:
            break
        keep.append(t)
        tot += t.nbytes
    g.tensors = keep
    shm = f"/dev/shm/jitc-prof-{os.getpid()}"
    st = GroupState(g, w.seed)
    ctx = J.Context(device=0, chunk_bytes=1 << 20, staging_bytes=int(os.environ.get("PROF_STAGING_MB", 1024)) << 20,
                    slot_bytes=int(os.environ.get("PROF_SLOT_MB", 256)) << 20, image_dir=shm,
                    flags=J.F_TIME_KERNELS | int(os.environ.get("PROF_FLAGS", "0")))
    ctx.register(0, J.REQUIRED, [0], st.table(), keepalive=st)
    ctx.mark(0, 1, J.CLEAN)
    for _ in range(reps):
        blob = ctx.fingerprint()
        s, sel = J.select_consistent_replica(blob, [0])
        ctx.capture(sel)
        ctx.commit(sel)
        ctx.restore(0, J.HOST)
        ctx.verify(0)
    torch.cuda.synchronize()
    for k, n in ((1, "K1"), (2, "K2"), (3, "K3")):
        c = ctx.kernel_counters(k)
        rw = 1 if k == 1 else 2
        print(n, "launches", c["launches"], "us/launch %.1f" % (1e3 * c["ms"] / max(c["launches"], 1)),
              "MB/launch %.1f" % (c["bytes"] / max(c["launches"], 1) / 1e6),
              "GB/s=%.1f" % (rw * c["bytes"] / (c["ms"] * 1e-3) / 1e9 if c["ms"] else 0))
    ctx.close()
    shutil.rmtree(shm, ignore_errors=True)


if __name__ == "__main__":
    main()
