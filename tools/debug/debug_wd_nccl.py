"""Debug probe for reading R9 over NCCL (socket transport, three processes on
one GPU, one NCCL_HOSTID each): rank 1 dies; ranks 0 and 2 enter a library
collective (argv[1]: "exchange" = record all-gather, "barrier" = commit
barrier) that can no longer complete, get JITC_EPEER from the liveness-aware
wait, and shrink (argv[2]: "shrink" = jitc_comm_shrink, "abort" =
jitc_comm_destroy then a fresh jitc_comm_init among the survivors).  Every
step prints; a stuck rank dumps its Python stack after 40 s and is killed
after 80 s."""
import os
import subprocess
import sys
import textwrap
import time
import uuid

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

RANK = r"""
import faulthandler, os, sys, time
faulthandler.dump_traceback_later(40, exit=False)
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
rank, shm, op, how = {rank}, {shm!r}, {op!r}, {how!r}
T0 = time.time()
def say(*a): print(f"[{{rank}} {{time.time() - T0:7.3f}}]", *a, flush=True)
w = W.scaled(W.c2(), 40000)
ctx = J.Context(device=0, rank=rank, world=3, chunk_bytes=1 << 20, image_dir=shm + "/img", staging_bytes=48 << 20,
                slot_bytes=8 << 20)
keep = []
for g in w.groups:
    st = GroupState(g, w.seed, shuffle_seed=rank); keep.append(st)
    ctx.register(g.group, g.policy, [0, 1, 2], st.table(), keepalive=st)
    ctx.mark(g.group, 50, J.CLEAN)
torch.cuda.synchronize()
ctx.liveness_init(shm + "/live")
def uid(name, me):
    p = shm + "/" + name
    if me == 0:
        open(p + ".tmp", "wb").write(J.get_unique_id()); os.rename(p + ".tmp", p)
    while not os.path.exists(p):
        time.sleep(0.01)
    return open(p, "rb").read()
ctx.comm_init(uid("uid", rank), 3, rank)
say("comm_init")
if rank == 1:
    time.sleep(0.3); os._exit(1)
time.sleep(0.8)
blob = ctx.fingerprint()
try:
    if op == "exchange":
        ctx.exchange_records(blob)
    else:
        allb = ctx.exchange_records(blob)
        raise SystemExit("exchange should have failed")
except J.JitcError as e:
    say("collective failed:", e)
dead = ctx.comm_dead()
say("dead", dead)
if how == "shrink":
    ctx.comm_shrink(dead)
    say("shrunk")
else:
    ctx.comm_destroy()
    say("destroyed")
    ctx.comm_init(uid("uid2", 0 if rank == 0 else 1), 2, 0 if rank == 0 else 1, job_ranks=[0, 2])
    say("re-init")
allb = ctx.exchange_records(ctx.fingerprint())
say("exchange ok", len(allb))
ctx.close()
say("closed")
"""


def main():
    op = sys.argv[1] if len(sys.argv) > 1 else "exchange"
    how = sys.argv[2] if len(sys.argv) > 2 else "shrink"
    shm = f"/dev/shm/jitc-dbgwd-{os.getpid()}-{uuid.uuid4().hex[:6]}"
    os.makedirs(shm)
    procs = []
    for r in range(3):
        env = dict(os.environ, JITC_PEER_DEAD_MS="500", NCCL_HOSTID=f"dbg-host-{r}", NCCL_SOCKET_IFNAME="lo",
                   NCCL_IB_DISABLE="1", NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0",
                   NCCL_DEBUG=os.environ.get("NCCL_DEBUG", "WARN"), JITC_DEBUG_SHRINK="1")
        procs.append(subprocess.Popen([sys.executable, "-c", textwrap.dedent(RANK.format(
            root=ROOT, rank=r, shm=shm, op=op, how=how))], cwd=ROOT, stdout=subprocess.PIPE,
            stderr=subprocess.STDOUT, text=True, env=env))
    t0 = time.time()
    while time.time() - t0 < 80 and any(p.poll() is None for p in procs):
        time.sleep(0.5)
    for p in procs:
        if p.poll() is None:
            p.kill()
    for r, p in enumerate(procs):
        print(f"===== rank {r} rc={p.returncode}")
        print(p.communicate()[0][-6000:])
    subprocess.run(["rm", "-rf", shm])


if __name__ == "__main__":
    main()
