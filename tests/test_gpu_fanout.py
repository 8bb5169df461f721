"""Capture with NVLink fan-out with real
processes on one B200, over both transports.

TP2 x DP2 (partitions p = 0, 1 with replicas {p, p + 2}); rank 3 died, so
partition 1 has a single writer (rank 1).  The three survivors form the
communicator; each declares the partition it does not hold and attaches its
host image (steady state), then fingerprint -> exchange -> select ->
jitc_capture_fanout over movers {0, 1, 2} -> commit.  Each survivor D2Hs a
third of each partition's image; the parts of a writer's shard that lie in
another survivor's lane cross over (NCCL send/recv, or a peer-to-peer copy
out of the writer's staging with the IPC transport).  The committed images
must equal the oracle's pack byte for byte, and a replacement process must
restore partition 1 from its image bit-exact against the oracle."""
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

import numpy as np
import pytest

from oracle import oracle as O
from workloads import configs as W

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
C = 1 << 20

SETUP = r"""
import copy, os, sys, time
sys.path.insert(0, {root!r})
import numpy as np, torch
from oracle import oracle as O
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W

rank, shm, transport = {rank}, {shm!r}, {transport!r}
device = rank % torch.cuda.device_count()
torch.cuda.set_device(device)
base = W.scaled(W.c2(), 40000).groups[0]
groups = []
for p in (0, 1):
    g = copy.deepcopy(base)
    g.group, g.members = p, [p, p + 2]
    groups.append(g)
seed = 0x4A4954435F563105
"""

RANK = SETUP + r"""
comm = [0, 1, 2]
ctx = J.Context(device=device, rank=rank, world=4, chunk_bytes={C}, image_dir=shm + "/img",
                staging_bytes=24 << 20, slot_bytes=4 << 20, flags=J.F_TIME_KERNELS)
st = None
for g in groups:
    if rank in g.members:
        st = GroupState(g, seed, device=device, shuffle_seed=3 + rank)
        ctx.register(g.group, g.policy, g.members, st.table(), keepalive=st)
        ctx.mark(g.group, 12, J.CLEAN)
    else:
        ctx.declare_group(g.group, g.policy, g.members)
        L = J.layout([(t.name, t.nbytes, 0) for t in g.tensors], {C})[2]
        ctx.attach_image(g.group, L)
if transport == "ipc":
    ctx.comm_init_ipc(shm + "/comm", 3, rank)
else:
    uid_path = shm + "/uid"
    if rank == 0:
        open(uid_path + ".tmp", "wb").write(J.get_unique_id())
        os.rename(uid_path + ".tmp", uid_path)
    t0 = time.time()
    while not os.path.exists(uid_path) and time.time() - t0 < 120:
        time.sleep(0.01)
    ctx.comm_init(open(uid_path, "rb").read(), 3, rank)
blob = ctx.fingerprint()
allb = ctx.exchange_records(blob)
s_, sel = J.select_consistent_replica(allb, comm)
assert s_ == J.OK, J.parse_selection(sel)
gsel = {{g["group"]: g for g in J.parse_selection(sel)["groups"]}}
assert gsel[0]["writers"] == [0, 2] and gsel[1]["writers"] == [1], gsel
for rep in range(2):      # twice: slot reuse and the IPC round generations across calls
    cap = ctx.capture_fanout(sel, comm)
    ctx.commit(sel)
print("fanout ok", cap["d2h_bytes"], cap["p2p_bytes"], cap["image_bytes"], flush=True)
ctx.close()
"""

REPLACEMENT = SETUP + r"""
ctx = J.Context(device=device, rank=3, world=4, chunk_bytes={C}, image_dir=shm + "/img",
                staging_bytes=24 << 20, slot_bytes=4 << 20)
g = groups[1]
st = GroupState(g, seed, device=device, fill=False, shuffle_seed=11)
st.scramble()
ctx.register(g.group, g.policy, g.members, st.table(), keepalive=st)
ctx.declare_group(0, groups[0].policy, groups[0].members)
ctx.restore(1, J.HOST)
ctx.verify(1)
torch.cuda.synchronize()
for i, t in enumerate(g.tensors):
    assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, seed, g.group)), t.name
print("replacement ok", flush=True)
ctx.close()
"""


def _env(transport, rank):
    from tests.mp_util import nccl_env
    return dict(os.environ) if transport == "ipc" else nccl_env("fanout", rank)


def _run(code, env):
    return subprocess.Popen([sys.executable, "-c", code], cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT,
                            text=True, env=env)


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_fanout_capture_tp2_dp2_lone_writer(transport):
    shm = f"/dev/shm/jitc-fan-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        procs = [_run(textwrap.dedent(RANK.format(root=ROOT, rank=r, shm=shm, transport=transport, C=C)),
                      _env(transport, r)) for r in range(3)]
        outs = [p.communicate(timeout=600)[0] for p in procs]
        assert all(p.returncode == 0 for p in procs), "\n=====\n".join(outs)
        stats = [list(map(int, o.split("fanout ok")[1].split()[:3])) for o in outs]
        base = W.scaled(W.c2(), 40000).groups[0]
        seed = 0x4A4954435F563105
        import copy
        Ls = {}
        for p in (0, 1):
            g = copy.deepcopy(base)
            g.group, g.members = p, [p, p + 2]
            lay = O.layout_of_group(g, C)
            want = O.pack(O.gen_group(g, seed), lay)
            got = np.fromfile(f"{shm}/img/g{p}.img", dtype=np.uint8)[:lay.L]
            assert np.array_equal(got, want), f"partition {p}: fan-out image differs from the oracle pack"
            Ls[p] = lay.L
        # each survivor moved one third of each partition (lanes O5 over 3 movers)
        total = Ls[0] + Ls[1]
        assert sum(s[0] for s in stats) == total
        assert all(abs(s[0] - total / 3) <= 2 * C for s in stats), stats
        assert stats[1][1] > 0, "the lone writer of partition 1 ships over NVLink"
        r = _run(textwrap.dedent(REPLACEMENT.format(root=ROOT, shm=shm, transport=transport, C=C, rank=3)),
                 dict(os.environ))
        out = r.communicate(timeout=600)[0]
        assert r.returncode == 0 and "replacement ok" in out, out
    finally:
        shutil.rmtree(shm, ignore_errors=True)


def test_attach_image_and_fanout_argument_errors():
    """jitc_attach_image is for declared (non-held) groups of a context with a
    shared image_dir; jitc_capture_fanout needs a communicator."""
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc as J
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    build.build()
    shm = f"/dev/shm/jitc-fan-err-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    try:
        g = W.scaled(W.c1(), 2000).groups[0]
        st = GroupState(g, 5)
        ctx = J.Context(device=0, rank=0, world=2, chunk_bytes=4096, image_dir=shm, staging_bytes=1 << 20,
                        slot_bytes=1 << 18)
        _, L = ctx.register(0, J.REQUIRED, [0, 1], st.table(), keepalive=st)
        ctx.declare_group(1, J.OPTIONAL, [1])      # rank 1 is not healthy below: the group is dropped
        with pytest.raises(J.JitcError):
            ctx.attach_image(0, L)            # held: already has its image
        with pytest.raises(J.JitcError):
            ctx.attach_image(7, L)            # undeclared
        with pytest.raises(J.JitcError):
            ctx.attach_image(1, L + 1)        # not a multiple of 256
        ctx.attach_image(1, L)
        ctx.attach_image(1, L)                # idempotent
        assert os.path.getsize(f"{shm}/g1.img") >= L
        ctx.mark(0, 3, J.CLEAN)
        blob = ctx.fingerprint()
        s_, sel = J.select_consistent_replica(blob, [0])
        assert s_ == J.OK, J.parse_selection(sel)
        with pytest.raises(J.JitcError, match="communicator"):
            ctx.capture_fanout(sel, [0])      # no communicator
        ctx.close()
        nodir = J.Context(device=0, rank=0, world=2, chunk_bytes=4096, staging_bytes=1 << 20, slot_bytes=1 << 18)
        nodir.declare_group(1, J.REQUIRED, [1])
        with pytest.raises(J.JitcError):
            nodir.attach_image(1, L)          # private pinned images cannot be shared
        nodir.close()
    finally:
        shutil.rmtree(shm, ignore_errors=True)
