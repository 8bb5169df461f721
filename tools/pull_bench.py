"""Measures the F1 fused peer pull (K5) at full size: a writer process holds
the C2 (or C3) state and exports it, a replacement process pulls + verifies
it through CUDA IPC.  On one B200 the peer mapping is the same HBM (the
kernel is HBM read+write bound); on an NVLink box it is NVLink-bound.

    python tools/pull_bench.py [C2|C3] [reps]
"""
import json
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WRITER = """
import os, sys, time
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
w = W.CONFIGS[{cfg!r}](world=2)
shm = {shm!r}
ctx = J.Context(device=0, rank=0, world=2, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=64 << 20, slot_bytes=16 << 20)
keep = []
for g in w.groups:
    st = GroupState(g, w.seed); keep.append(st)
    ctx.register(g.group, g.policy, [0, 1], st.table(), keepalive=st)
    ctx.mark(g.group, 7, J.CLEAN)
open(shm + "/blob.0", "wb").write(ctx.fingerprint())
for g in w.groups:
    ctx.peer_export(g.group)
open(shm + "/ready", "w").write("1")
t0 = time.time()
while not os.path.exists(shm + "/done") and time.time() - t0 < 900:
    time.sleep(0.05)
"""

DEST = """
import json, os, sys, time
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
w = W.CONFIGS[{cfg!r}](world=2)
shm = {shm!r}
ctx = J.Context(device=0, rank=1, world=2, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=64 << 20, slot_bytes=16 << 20,
                flags=J.F_TIME_KERNELS)
keep = []
L = 0
for g in w.groups:
    st = GroupState(g, w.seed, fill=False); st.scramble(); keep.append(st)
    L += ctx.register(g.group, g.policy, [0, 1], st.table(), keepalive=st)[1]
t0 = time.time()
while not os.path.exists(shm + "/ready") and time.time() - t0 < 900:
    time.sleep(0.05)
try:
    s_, sel = J.select_consistent_replica(open(shm + "/blob.0", "rb").read(), [0])
    for rep in range({reps} + 1):
        if rep == 1:
            ctx.reset_counters()
        ms = 0.0
        for g in w.groups:
            ms += ctx.restore_pull(g.group, sel)["ms_device"]
        if rep == 0:
            continue
    for g in w.groups:
        ctx.verify(g.group)
    k = ctx.kernel_counters(J.K_PULL)
    print(json.dumps(dict(workload=w.name, image_bytes=L, reps={reps}, launches=k["launches"],
                          kernel_ms_per_pull=round(k["ms"] / {reps}, 3),
                          K5_GBps_rw=round(2 * k["bytes"] / (k["ms"] * 1e-3) / 1e9, 1),
                          pull_GBps_state=round(k["bytes"] / (k["ms"] * 1e-3) / 1e9, 1),
                          note="writer and replacement are separate processes on ONE B200: the IPC peer mapping is "
                               "local HBM, so K5 is HBM read+write bound; over NVLink the same kernel is link-bound")),
          flush=True)
finally:
    open(shm + "/done", "w").write("1")
"""


def main(cfg="C2", reps=3):
    shm = f"/dev/shm/jitc-pullbench-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        wp = subprocess.Popen([sys.executable, "-c", textwrap.dedent(WRITER.format(root=ROOT, cfg=cfg, shm=shm))],
                              cwd=ROOT)
        d = subprocess.run([sys.executable, "-c", textwrap.dedent(DEST.format(root=ROOT, cfg=cfg, shm=shm, reps=reps))],
                           cwd=ROOT, capture_output=True, text=True, timeout=1500)
        wp.wait(timeout=300)
        print(d.stdout.strip().splitlines()[-1] if d.returncode == 0 else d.stdout + d.stderr)
    finally:
        shutil.rmtree(shm, ignore_errors=True)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "C2", int(sys.argv[2]) if len(sys.argv) > 2 else 3)
