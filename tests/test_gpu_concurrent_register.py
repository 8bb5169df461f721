"""The ranks of a box register the SAME /dev/shm image concurrently.
Unserialised concurrent cudaHostRegister of fresh tmpfs pages fails for
images >= 8 GiB (tools/pin_probe2.py); jitc_register pre-allocates the pages
and serialises the registration with flock.  Three processes register a
12 GiB group at the same time and must all succeed."""
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = """
import sys, time
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
device = {rank} % torch.cuda.device_count()
torch.cuda.set_device(device)
x = torch.empty(12 << 30, dtype=torch.uint8, device="cuda")
ctx = J.Context(device=device, rank={rank}, world=3, image_dir={shm!r}, staging_bytes=64 << 20, slot_bytes=16 << 20)
while time.time() < {start}:
    time.sleep(0.001)
t = time.time()
ctx.register(0, J.REQUIRED, [0, 1, 2], [("big", x.data_ptr(), x.numel(), 0)], keepalive=x)
print("registered in %.1f s" % (time.time() - t), flush=True)
"""


def test_concurrent_register_same_image():
    import time
    shm = f"/dev/shm/jitc-creg-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    start = time.time() + 25           # all three call jitc_register at the same instant
    try:
        ps = [subprocess.Popen([sys.executable, "-c", textwrap.dedent(CHILD.format(root=ROOT, rank=r, shm=shm,
                                                                                  start=start))],
                               cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True)
              for r in range(3)]
        outs = [p.communicate(timeout=400)[0] for p in ps]
        for p, o in zip(ps, outs):
            assert p.returncode == 0 and "registered" in o, o
    finally:
        shutil.rmtree(shm, ignore_errors=True)
