"""F1 fusion: PEER restore by direct peer-memory reads (CUDA IPC), with real
separate processes on one B200 (IPC works between processes on the same
device; on an 8-GPU box the same mappings are NVLink peer memory).

k writer processes fingerprint and export their live state; a replacement
process selects the writers from their record blobs, maps their tensors and
pulls + scatters + verifies everything with one kernel (K5).  The restored
bytes must equal the oracle's; a writer whose state changes after its export
must be caught at the exact chunk."""
import os
import shutil
import subprocess
import sys
import textwrap
import time
import uuid

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

WRITER = """
import os, sys, time
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
rank, world, shm, flip = {rank}, {world}, {shm!r}, {flip}
import torch as _t
device = rank % _t.cuda.device_count()
_t.cuda.set_device(device)
w = W.scaled(W.c2(), 60000)
ctx = J.Context(device=device, rank=rank, world=world, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=64 << 20,
                slot_bytes=16 << 20)
keep = []
for g in w.groups:
    st = GroupState(g, w.seed, device=device, shuffle_seed=11 + rank); keep.append(st)
    ctx.register(g.group, g.policy, list(range(world)), st.table(), keepalive=st)
    ctx.mark(g.group, 21, J.CLEAN)
blob = ctx.fingerprint()
for g in w.groups:
    ctx.peer_export(g.group)
if flip:                                     # the state changes after the export
    J.inject_bitflip(keep[0].ptrs[5], 100, 2)
    torch.cuda.synchronize()
open(f"{{shm}}/blob.{{rank}}", "wb").write(blob)
open(f"{{shm}}/ready.{{rank}}", "w").write("1")
t0 = time.time()
while not os.path.exists(f"{{shm}}/done") and time.time() - t0 < 180:
    time.sleep(0.05)
print("writer done", flush=True)
"""

DEST = """
import os, sys, time
sys.path.insert(0, {root!r})
import numpy as np, torch
from oracle import oracle as O
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
rank, world, shm, writers, expect_bad = {rank}, {world}, {shm!r}, {writers}, {expect_bad}
import torch as _t
device = rank % _t.cuda.device_count()
_t.cuda.set_device(device)
w = W.scaled(W.c2(), 60000)
ctx = J.Context(device=device, rank=rank, world=world, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=64 << 20,
                slot_bytes=16 << 20, flags=J.F_TIME_KERNELS)
sts = {{}}
for g in w.groups:
    st = GroupState(g, w.seed, device=device, fill=False, shuffle_seed=99); st.scramble(); sts[g.group] = st
    ctx.register(g.group, g.policy, list(range(world)), st.table(), keepalive=st)
t0 = time.time()
while not all(os.path.exists(f"{{shm}}/ready.{{r}}") for r in writers) and time.time() - t0 < 180:
    time.sleep(0.05)
blobs = b"".join(open(f"{{shm}}/blob.{{r}}", "rb").read() for r in writers)
st_, sel = J.select_consistent_replica(blobs, writers)
assert st_ == J.OK, J.parse_selection(sel)
try:
    if expect_bad >= 0:
        try:
            ctx.restore_pull(0, sel)
            raise SystemExit("corruption not detected")
        except J.JitcError as e:
            assert e.status == J.ECORRUPT and e.first_bad == expect_bad, (e.status, e.first_bad, expect_bad)
            print("corruption caught at chunk", e.first_bad, flush=True)
    else:
        tot = 0.0
        for g in w.groups:
            s = ctx.restore_pull(g.group, sel)
            assert s["image_bytes"] == O.layout_of_group(g, 1 << 20).L and s["kernel_launches"] == 1
            tot += s["ms_device"]
            ctx.verify(g.group)
        torch.cuda.synchronize()
        for g in w.groups:
            for i, t in enumerate(g.tensors):
                assert np.array_equal(sts[g.group].tensor_bytes(i).cpu().numpy(),
                                      O.gen_tensor_bytes(t, w.seed, g.group)), t.name
        k = ctx.kernel_counters(J.K_PULL)
        print("pulled bit-exact", k["launches"], round(2 * k["bytes"] / (k["ms"] * 1e-3) / 1e9, 1), "GB/s", flush=True)
finally:
    open(f"{{shm}}/done", "w").write("1")
"""


def _run(k, flip=False):
    from oracle import oracle as O
    from workloads import configs as W
    shm = f"/dev/shm/jitc-pull-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    world = k + 1
    expect_bad = -1
    if flip:
        g = W.scaled(W.c2(), 60000).groups[0]
        lay = O.layout_of_group(g, 1 << 20)
        expect_bad = (lay.offsets[5] + 100) >> 20
    try:
        ws = [subprocess.Popen([sys.executable, "-c", textwrap.dedent(WRITER.format(
            root=ROOT, rank=r, world=world, shm=shm, flip=flip and r == 0))], cwd=ROOT,
            stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True) for r in range(k)]
        d = subprocess.run([sys.executable, "-c", textwrap.dedent(DEST.format(
            root=ROOT, rank=k, world=world, shm=shm, writers=list(range(k)), expect_bad=expect_bad))],
            cwd=ROOT, capture_output=True, text=True, timeout=400)
        outs = [p.communicate(timeout=200)[0] for p in ws]
        assert d.returncode == 0, d.stdout + d.stderr + "\n".join(outs)
        assert all(p.returncode == 0 for p in ws), "\n".join(outs)
        return d.stdout
    finally:
        shutil.rmtree(shm, ignore_errors=True)


@pytest.mark.parametrize("k", [1, 2])
def test_peer_pull_bit_exact(k):
    out = _run(k)
    assert "pulled bit-exact" in out, out


def test_peer_pull_detects_writer_change():
    out = _run(1, flip=True)
    assert "corruption caught" in out, out
