"""Can several ranks share one GPU in an NCCL communicator?  (Probe.)

NCCL refuses two ranks with the same (host hash, PCI bus id) ("Duplicate GPU
detected").  The host hash honours NCCL_HOSTID, so giving every rank its own
NCCL_HOSTID makes them look like separate hosts: NCCL then connects them with
its socket network transport over loopback.  Slow, but it runs the library's
NCCL code (unique id, init, all-gather, grouped send/recv, shrink) with real
processes on a 1-GPU box.

    python tools/nccl_same_gpu.py            # spawns 2 ranks
"""
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def nccl_env(rank: int) -> dict:
    return dict(os.environ, NCCL_HOSTID=f"jitc-fake-host-{rank}", NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1",
                NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0", NCCL_DEBUG="WARN")


def rank_main(rank: int, world: int, path: str):
    import numpy as np
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    ctx = J.Context(device=0, rank=rank, world=world, staging_bytes=64 << 20, slot_bytes=16 << 20)
    if rank == 0:
        open(path + ".tmp", "wb").write(J.get_unique_id())
        os.rename(path + ".tmp", path)
    while not os.path.exists(path):
        time.sleep(0.01)
    uid = open(path, "rb").read()
    t0 = time.time()
    ctx.comm_init(uid, world, rank)
    print(rank, "comm_init OK %.2fs" % (time.time() - t0), flush=True)
    ctx.close()


if __name__ == "__main__":
    if len(sys.argv) > 1:
        rank_main(int(sys.argv[1]), int(sys.argv[2]), sys.argv[3])
        sys.exit(0)
    world = 2
    path = f"/dev/shm/nccl_uid.{os.getpid()}"
    ps = [subprocess.Popen([sys.executable, __file__, str(r), str(world), path], env=nccl_env(r))
          for r in range(world)]
    rc = [p.wait(timeout=300) for p in ps]
    os.unlink(path)
    print("exit codes", rc)
    sys.exit(max(rc))
