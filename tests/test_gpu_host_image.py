"""The shared host image's placement: the rank that creates
an image gives each rank's slice a NUMA memory policy on the node of that
rank's GPU before the pages are allocated (JITC_NUMA=force applies it on the
single-node GPU boxes of this pool too), and the capture/restore through the
placed image stays bit-exact against the oracle."""
import os
import shutil
import uuid

import numpy as np
import pytest
import torch

from oracle import oracle as O
from workloads import configs as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return jitc


def _gpu_node(dev=0):
    """NUMA node of GPU `dev` from sysfs (nvidia-smi's bus id, lower case)."""
    import subprocess
    out = subprocess.run(["nvidia-smi", "-i", str(dev), "--query-gpu=pci.bus_id", "--format=csv,noheader"],
                         capture_output=True, text=True).stdout.strip()
    try:
        return int(open(f"/sys/bus/pci/devices/{out.lower()[-12:]}/numa_node").read())
    except Exception:
        return None


def test_image_slices_get_numa_policy(J, monkeypatch):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    monkeypatch.setenv("JITC_NUMA", "force")
    d = f"/dev/shm/jitc-numa-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    try:
        g = W.scaled(W.c2(), 40000).groups[0]
        st = GroupState(g, 3)
        ctx = J.Context(device=0, rank=0, world=4, chunk_bytes=1 << 20, image_dir=d, staging_bytes=16 << 20,
                        slot_bytes=4 << 20)
        ctx.register(0, J.REQUIRED, [0, 1, 2, 3], st.table(), keepalive=st)
        node = _gpu_node(0)
        maps = [l for l in open("/proc/self/numa_maps") if f"{d}/g0.img" in l]
        assert maps, "image not mapped"
        if node is not None and node >= 0:
            # 4 slices, each preferred on GPU 0's node (one GPU: every rank's GPU is 0)
            assert sum(f"prefer:{node}" in l for l in maps) >= 1, maps
        ctx.mark(0, 1, J.CLEAN)
        blob = ctx.fingerprint()
        s_, sel = J.select_consistent_replica(ctx.exchange_records(blob), [0])
        assert s_ == J.OK
        ctx.capture(sel)
        ctx.commit(sel)
        lay = O.layout_of_group(g, 1 << 20)
        img = np.fromfile(f"{d}/g0.img", dtype=np.uint8)[:lay.L]
        assert np.array_equal(img, O.pack(O.gen_group(g, 3), lay))
        ctx.close()
    finally:
        shutil.rmtree(d, ignore_errors=True)
