"""Helpers for the multi-process GPU tests (one process per rank).

On a box with several GPUs every rank gets its own device (rank % count), so
NCCL uses its P2P / NVLS transports over NVLink and the IPC transport's peer
loads cross NVLink; on a 1-GPU box all ranks share GPU 0 and NCCL, which
refuses two ranks per device on one host, is given one fake host per rank
(NCCL_HOSTID) and connects them with its socket transport over loopback."""
import os

# pasted into each rank's script after `rank` is defined
DEVICE_LINES = "import torch as _t\ndevice = rank % _t.cuda.device_count()\n_t.cuda.set_device(device)\n"


def gpu_count() -> int:
    import torch
    return torch.cuda.device_count()


def nccl_env(tag: str, rank: int, base=None) -> dict:
    env = dict(base if base is not None else os.environ)
    if gpu_count() <= 1:
        env.update(NCCL_HOSTID=f"jitc-{tag}-host-{rank}", NCCL_SOCKET_IFNAME="lo", NCCL_IB_DISABLE="1",
                   NCCL_P2P_DISABLE="1", NCCL_SHM_DISABLE="1", NCCL_NVLS_ENABLE="0", NCCL_DEBUG="WARN")
    return env
