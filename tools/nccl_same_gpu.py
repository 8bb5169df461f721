"""Can two ranks share one GPU in an NCCL communicator?  (Probe; argv[1]=rank.)"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
rank = int(sys.argv[1]); path = "/dev/shm/nccl_uid"
ctx = J.Context(device=0, rank=rank, world=2, staging_bytes=64 << 20, slot_bytes=16 << 20)
if rank == 0:
    open(path + ".tmp", "wb").write(J.get_unique_id()); os.rename(path + ".tmp", path)
while not os.path.exists(path):
    time.sleep(0.01)
uid = open(path, "rb").read()
try:
    ctx.comm_init(uid, 2, rank)
    print(rank, "comm_init OK", flush=True)
except Exception as e:
    print(rank, "comm_init failed:", e, flush=True)
