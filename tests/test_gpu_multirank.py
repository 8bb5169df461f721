"""The whole multi-rank runtime on one B200 with real processes, through each
of the library's two transports: the intra-node IPC transport
(jitc_comm_init_ipc) and NCCL (jitc_comm_init).  NCCL refuses two ranks with
the same (host hash, bus id); every rank gets its own NCCL_HOSTID, so NCCL
sees separate hosts and connects them with its socket transport over
loopback (functional, not a measurement).  Covered: record exchange, selection, k-way sharded capture into
the shared image, commit barrier, HOST restore with the slice exchange fused
into K3 (each rank loads 1/n of the image and reads the others' slices from
their staging through CUDA IPC), and PEER restore of a replacement process
from the writers' live HBM.  A subset group (members {0, 1} of 3 ranks)
exercises the point-to-point exchange among members only.  Every restored
byte is compared with the oracle."""
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

RANK = r"""
import os, sys, time
sys.path.insert(0, {root!r})
import numpy as np, torch
from oracle import oracle as O
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W

rank, world, shm, phase, transport = {rank}, {world}, {shm!r}, {phase!r}, {transport!r}
base = W.scaled(W.c2(), 30000)
groups = [base.groups[0], base.groups[1]]           # REQUIRED + OPTIONAL, on every rank
sub = W.scaled(W.c1(), 4000).groups[0]; sub.group = 2; sub.members = [0, 1]   # a subset group
groups.append(sub)
seed = base.seed


# one process per GPU when the box has several (NVLink / NVSwitch: NCCL P2P and
# NVLS, CUDA IPC peer loads); all on GPU 0 of a 1-GPU box
device = rank % torch.cuda.device_count()
torch.cuda.set_device(device)


def init_comm(ctx, comm_dir, n, me, job_ranks=None):
    if transport == "ipc":
        ctx.comm_init_ipc(comm_dir, n, me, job_ranks)
    else:                                           # NCCL: comm rank 0 publishes the unique id
        uid_path = comm_dir + ".uid"
        if me == 0:
            open(uid_path + ".tmp", "wb").write(J.get_unique_id())
            os.rename(uid_path + ".tmp", uid_path)
        t0 = time.time()
        while not os.path.exists(uid_path) and time.time() - t0 < 120:
            time.sleep(0.01)
        ctx.comm_init(open(uid_path, "rb").read(), n, me, job_ranks)


def make_ctx(comm_dir, scramble, comm=True):
    ctx = J.Context(device=device, rank=rank, world=world, chunk_bytes=1 << 20, image_dir=shm + "/img",
                    staging_bytes=48 << 20, slot_bytes=4 << 20, flags=J.F_TIME_KERNELS)
    sts = {{}}
    for g in groups:
        members = g.members if g.group == 2 else list(range(world))
        if rank in members:
            st = GroupState(g, seed, device=device, fill=not scramble, shuffle_seed=10 * rank + (7 if scramble else 0))
            if scramble:
                st.scramble()
            sts[g.group] = st
            ctx.register(g.group, g.policy, members, st.table(), keepalive=st)
            ctx.mark(g.group, 33, J.CLEAN)
        else:
            ctx.declare_group(g.group, g.policy, members)
    if comm:
        init_comm(ctx, comm_dir, world, rank)
    return ctx, sts


def check(ctx, sts, gids):
    torch.cuda.synchronize()
    for g in groups:
        if g.group not in gids or g.group not in sts:
            continue
        ctx.verify(g.group)
        for i, t in enumerate(g.tensors):
            assert np.array_equal(sts[g.group].tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, seed, g.group)), \
                (g.group, t.name)


if phase == "host":
    ctx, sts = make_ctx(shm + "/comm1", scramble=False)
    blob = ctx.fingerprint()
    allb = ctx.exchange_records(blob)
    st_, sel = J.select_consistent_replica(allb, list(range(world)))
    assert st_ == J.OK, J.parse_selection(sel)
    g0 = J.parse_selection(sel)["groups"][0]
    assert g0["writers"] == list(range(world))
    cap = ctx.capture(sel)                              # 1/k of every group this rank writes
    ctx.commit(sel)
    for st in sts.values():
        st.scramble()
    res = ctx.restore(J.ALL_GROUPS, J.HOST)             # 1/n H2D + peers' slices over IPC, fused into K3
    check(ctx, sts, {{0, 1, 2}})
    print("host ok", cap["image_bytes"], res["h2d_bytes"], res["p2p_bytes"], flush=True)
elif phase in ("w0", "repl", "dirty"):
    # rank 0 healthy; rank 1 replaced; rank 2 alive but DIRTY with a half-applied
    # update: both non-writers are repaired from rank 0 (SURVEY O8 destinations)
    ctx, sts = make_ctx(shm + "/comm3", scramble=(phase == "repl"))
    if phase == "dirty":
        g0 = groups[0]
        for i in range(0, len(g0.tensors), 2):
            t = g0.tensors[i]
            J.inject_update(sts[0].ptrs[i], 0, t.nbytes // 4, t.gen_id, 34)
        torch.cuda.synchronize()
        ctx.mark(0, 33, J.DIRTY)
    if phase != "repl":
        open(f"{{shm}}/blob3.{{rank}}", "wb").write(ctx.fingerprint())
    t0 = time.time()
    while not all(os.path.exists(f"{{shm}}/blob3.{{r}}") for r in (0, 2)) and time.time() - t0 < 120:
        time.sleep(0.02)
    time.sleep(0.2)
    blobs = b"".join(open(f"{{shm}}/blob3.{{r}}", "rb").read() for r in (0, 2))
    st_, sel = J.select_consistent_replica(blobs, [0, 2])
    assert st_ == J.OK, J.parse_selection(sel)
    gsel = {{g["group"]: g for g in J.parse_selection(sel)["groups"]}}
    assert gsel[0]["writers"] == [0] and gsel[0]["excluded"] == [(2, J.DIRTY)], gsel[0]
    ctx.restore(J.ALL_GROUPS, J.PEER, sel)
    if phase == "repl":
        check(ctx, sts, {{0, 1, 2}})
    elif phase == "dirty":                       # repaired in group 0; a writer of group 1
        assert gsel[1]["writers"] == [0, 2]
        check(ctx, sts, {{0}})
    print(phase, "ok", flush=True)
elif phase in ("w_nosel", "repl_nosel"):
    # rank 1 died; the survivors 0 and 2 fingerprint, exchange and select over
    # their own (shrunk) communicator; then a fresh replacement joins a new
    # communicator and restores in PEER mode WITHOUT any selection or blob: it
    # receives the selection and the writers' digests over the communicator
    # (SURVEY.md §8(b); PAPER.md:174 copy from a healthy replica)
    ctx, sts = make_ctx(None, scramble=(phase == "repl_nosel"), comm=False)
    sel = None
    if phase == "w_nosel":
        init_comm(ctx, shm + "/comm4a", 2, {{0: 0, 2: 1}}[rank], [0, 2])
        allb = ctx.exchange_records(ctx.fingerprint())
        st_, sel = J.select_consistent_replica(allb, [0, 2])
        assert st_ == J.OK, J.parse_selection(sel)
    init_comm(ctx, shm + "/comm4b", world, rank)
    res = ctx.restore(J.ALL_GROUPS, J.PEER, sel)
    if phase == "repl_nosel":
        check(ctx, sts, {{0, 1, 2}})
        assert res["groups_done"] == 3, res
    print(phase, "ok", flush=True)
elif phase in ("writer", "replacement"):
    # rank 1 died; ranks 0 and 2 keep their state, a replacement process joins
    ctx, sts = make_ctx(shm + "/comm2", scramble=(phase == "replacement"))
    if phase == "writer":
        blob = ctx.fingerprint()
        open(f"{{shm}}/blob.{{rank}}", "wb").write(blob)
    # the healthy ranks' blobs reach everyone (the harness plays the broadcast)
    t0 = time.time()
    while not all(os.path.exists(f"{{shm}}/blob.{{r}}") for r in (0, 2)) and time.time() - t0 < 120:
        time.sleep(0.02)
    time.sleep(0.2)
    blobs = b"".join(open(f"{{shm}}/blob.{{r}}", "rb").read() for r in (0, 2))
    st_, sel = J.select_consistent_replica(blobs, [0, 2])
    assert st_ == J.OK, J.parse_selection(sel)
    res = ctx.restore(J.ALL_GROUPS, J.PEER, sel)
    if phase == "replacement":
        gsel = {{g["group"]: g for g in J.parse_selection(sel)["groups"]}}
        assert gsel[0]["writers"] == [0, 2] and gsel[2]["writers"] == [0]
        check(ctx, sts, {{0, 1, 2}})
        print("peer ok", res["p2p_bytes"], flush=True)
    else:
        print("writer ok", flush=True)
ctx.close()
"""


def _env(transport, rank):
    from tests.mp_util import nccl_env
    return dict(os.environ) if transport == "ipc" else nccl_env("test", rank)


def _spawn(shm, world, phases, transport):
    procs = []
    for r, ph in phases.items():
        code = textwrap.dedent(RANK.format(root=ROOT, rank=r, world=world, shm=shm, phase=ph, transport=transport))
        procs.append(subprocess.Popen([sys.executable, "-c", code], cwd=ROOT, stdout=subprocess.PIPE,
                                      stderr=subprocess.STDOUT, text=True, env=_env(transport, r)))
    outs = [p.communicate(timeout=600)[0] for p in procs]
    for p, o in zip(procs, outs):
        assert p.returncode == 0, "\n=====\n".join(outs)
    return outs


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_multirank_capture_and_host_restore(transport):
    shm = f"/dev/shm/jitc-ipc-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        outs = _spawn(shm, 3, {0: "host", 1: "host", 2: "host"}, transport)
        assert all("host ok" in o for o in outs), outs
    finally:
        shutil.rmtree(shm, ignore_errors=True)


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_multirank_peer_restore_of_replacement(transport):
    shm = f"/dev/shm/jitc-ipc-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        outs = _spawn(shm, 3, {0: "writer", 1: "replacement", 2: "writer"}, transport)
        assert "peer ok" in outs[1] and "writer ok" in outs[0] and "writer ok" in outs[2], outs
    finally:
        shutil.rmtree(shm, ignore_errors=True)


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_peer_restore_replacement_without_selection(transport):
    """The replacement passes no selection and no blobs to jitc_restore(PEER):
    the selection comes from the writers over the new communicator."""
    shm = f"/dev/shm/jitc-ipc-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        outs = _spawn(shm, 3, {0: "w_nosel", 1: "repl_nosel", 2: "w_nosel"}, transport)
        assert "repl_nosel ok" in outs[1] and "w_nosel ok" in outs[0] and "w_nosel ok" in outs[2], outs
    finally:
        shutil.rmtree(shm, ignore_errors=True)


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_peer_repairs_replacement_and_dirty_member(transport):
    shm = f"/dev/shm/jitc-ipc-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        outs = _spawn(shm, 3, {0: "w0", 1: "repl", 2: "dirty"}, transport)
        assert "w0 ok" in outs[0] and "repl ok" in outs[1] and "dirty ok" in outs[2], outs
    finally:
        shutil.rmtree(shm, ignore_errors=True)
