"""Reading R9: a writer dies during the
capture -> the survivors re-run it with k - 1 writers, since HBM still holds
their state.  Real processes on one B200 over both transports:

  3 ranks select writers {0, 1, 2} and capture their 1/3 shards; rank 1 dies
  (os._exit) before the commit -> the survivors' commit barrier fails with
  JITC_EPEER once rank 1's heartbeat is stale (instead of hanging) ->
  jitc_comm_dead == [1] -> jitc_comm_shrink -> fingerprint -> exchange ->
  select (writers {0, 2}) -> capture -> commit -> a replacement for rank 1
  HOST-restores bit-exact against the oracle.  The same over NCCL (socket
  transport on one GPU) with the liveness table: the commit's all-reduce
  wait polls the heartbeats (nccl_sync) and fails with JITC_EPEER; the
  survivors abort the communicator (the failed all-reduce is still in flight)
  and build a fresh one among themselves."""
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

import pytest

from tests.test_gpu_hang_collective import REPL

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

RANK = r"""
import os, sys, time
sys.path.insert(0, {root!r})
import torch
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
from workloads import configs as W
rank, shm, transport = {rank}, {shm!r}, {transport!r}
import torch as _t
device = rank % _t.cuda.device_count()
_t.cuda.set_device(device)
w = W.scaled(W.c2(), 40000, )
ctx = J.Context(device=device, rank=rank, world=3, chunk_bytes=1 << 20, image_dir=shm + "/img", staging_bytes=48 << 20,
                slot_bytes=8 << 20)
keep = []
for g in w.groups:
    st = GroupState(g, w.seed, device=device, shuffle_seed=rank); keep.append(st)
    ctx.register(g.group, g.policy, [0, 1, 2], st.table(), keepalive=st)
    ctx.mark(g.group, 50, J.CLEAN)
torch.cuda.synchronize()
def uid(name, me):                                 # NCCL unique ids through the shared directory
    p = shm + "/" + name
    if me == 0:
        open(p + ".tmp", "wb").write(J.get_unique_id())
        os.rename(p + ".tmp", p)
    while not os.path.exists(p):
        time.sleep(0.01)
    return open(p, "rb").read()
if transport == "ipc":
    ctx.comm_init_ipc(shm + "/comm", 3, rank)
else:                                              # NCCL + the liveness table (jitc_liveness_init)
    ctx.liveness_init(shm + "/live")
    ctx.comm_init(uid("uid", rank), 3, rank)
allb = ctx.exchange_records(ctx.fingerprint())
s_, sel = J.select_consistent_replica(allb, [0, 1, 2])
assert s_ == J.OK and J.parse_selection(sel)["groups"][0]["writers"] == [0, 1, 2]
ctx.capture(sel)                                   # every writer's 1/3 shard
if rank == 1:
    os._exit(1)                                    # dies before the commit: no complete checkpoint exists
t0 = time.time()
try:
    ctx.commit(sel)
    raise SystemExit("commit succeeded without rank 1")
except J.JitcError as e:
    # NCCL's socket transport may report the closed connection first (ENCCL)
    assert e.status == J.EPEER or (transport == "nccl" and e.status == J.ENCCL), e
detect = time.time() - t0
dead = ctx.comm_dead()
while not dead and time.time() - t0 < 10:          # (ENCCL can precede the stale heartbeat)
    time.sleep(0.05)
    dead = ctx.comm_dead()
assert dead == [1], dead
if transport == "ipc":
    ctx.comm_shrink(dead)
else:     # the failed all-reduce is still in flight: abort, then a fresh communicator among the survivors
    ctx.comm_destroy()
    ctx.comm_init(uid("uid2", 0 if rank == 0 else 1), 2, 0 if rank == 0 else 1, job_ranks=[0, 2])
allb = ctx.exchange_records(ctx.fingerprint())     # HBM still holds the state: re-run with k = 2
s_, sel2 = J.select_consistent_replica(allb, [0, 2])
assert s_ == J.OK and J.parse_selection(sel2)["groups"][0]["writers"] == [0, 2]
cap = ctx.capture(sel2)
ctx.commit(sel2)
print("survivor", rank, "detected in %.2f s, recaptured" % detect, cap["image_bytes"], flush=True)
ctx.close()
"""


def _env(transport, r):
    from tests.mp_util import nccl_env
    env = dict(os.environ, JITC_PEER_DEAD_MS="500")
    return env if transport != "nccl" else nccl_env("wd", r, env)


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_writer_dies_before_commit_survivors_recapture(transport):
    shm = f"/dev/shm/jitc-wdeath-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        procs = [subprocess.Popen([sys.executable, "-c", textwrap.dedent(RANK.format(root=ROOT, rank=r, shm=shm,
                                                                                     transport=transport))],
                                  cwd=ROOT, stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True,
                                  env=_env(transport, r))
                 for r in range(3)]
        try:
            outs = [p.communicate(timeout=300)[0] for p in procs]
        finally:
            for p in procs:
                if p.poll() is None:
                    p.kill()
        assert procs[1].returncode == 1
        for i in (0, 2):
            assert procs[i].returncode == 0 and "recaptured" in outs[i], "\n=====\n".join(outs)
        r = subprocess.run([sys.executable, "-c", textwrap.dedent(REPL.format(root=ROOT, shm=shm))], cwd=ROOT,
                           capture_output=True, text=True, timeout=300)
        assert r.returncode == 0 and "bit-exact" in r.stdout, r.stdout + r.stderr
    finally:
        shutil.rmtree(shm, ignore_errors=True)


PEER_RANK = RANK.split("ctx.capture(sel)")[0].replace(
    'assert s_ == J.OK and J.parse_selection(sel)["groups"][0]["writers"] == [0, 1, 2]\n', "") + r"""
# PEER restore: writers 0 and 1 rebuild rank 2 from live HBM; writer 1 dies first
s_, sel = J.select_consistent_replica(allb, [0, 1])
assert s_ == J.OK and J.parse_selection(sel)["groups"][0]["writers"] == [0, 1]
if rank == 1:
    os._exit(1)
t0 = time.time()
try:
    ctx.restore(J.ALL_GROUPS, J.PEER, sel)
    out = "completed"
except J.JitcError as e:
    assert e.status == J.EPEER or (transport == "nccl" and e.status == J.ENCCL), e
    out = "EPEER" if e.status == J.EPEER else "ENCCL"
print("rank", rank, out, "after %.2f s" % (time.time() - t0), flush=True)
os._exit(0)                      # a failed survivor leaves (its heartbeat stops)
"""


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_writer_dies_during_peer_restore_no_hang(transport):
    """A writer dies before a PEER restore: the replacement's restore fails
    with JITC_EPEER (NCCL's socket transport may report ENCCL first) within
    seconds instead of hanging, and the other writer finishes or fails the
    same way once the replacement has left."""
    shm = f"/dev/shm/jitc-wdeathp-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        procs = [subprocess.Popen([sys.executable, "-c", textwrap.dedent(PEER_RANK.format(
            root=ROOT, rank=r, shm=shm, transport=transport))], cwd=ROOT, stdout=subprocess.PIPE,
            stderr=subprocess.STDOUT, text=True, env=_env(transport, r)) for r in range(3)]
        try:
            outs = [p.communicate(timeout=240)[0] for p in procs]
        finally:
            for p in procs:
                if p.poll() is None:
                    p.kill()
        assert procs[1].returncode == 1
        assert procs[2].returncode == 0 and ("rank 2 EPEER" in outs[2] or "rank 2 ENCCL" in outs[2]), \
            "\n=====\n".join(outs)
        assert procs[0].returncode == 0 and "rank 0 " in outs[0], "\n=====\n".join(outs)
    finally:
        shutil.rmtree(shm, ignore_errors=True)


RETRY_RANK = RANK.split("allb = ctx.exchange_records(ctx.fingerprint())")[0] + r"""
import numpy as np
from oracle import oracle as O
allb = ctx.exchange_records(ctx.fingerprint())
s_, sel = J.select_consistent_replica(allb, [0, 1, 2])
assert s_ == J.OK
ctx.capture(sel)
ctx.commit(sel)                                    # a complete 3-way checkpoint
for st in keep:
    st.scramble()
t0 = time.time()
try:                                               # rank 2 exits part-way through (JITC_DEBUG_EXIT_AFTER_ROUND)
    ctx.restore(J.ALL_GROUPS, J.HOST)
    raise SystemExit("restore completed without rank 2")
except J.JitcError as e:
    assert e.status == J.EPEER, e
dead = ctx.comm_dead()
while not dead and time.time() - t0 < 10:
    time.sleep(0.05)
    dead = ctx.comm_dead()
assert dead == [2], dead
ctx.comm_shrink(dead)
res = ctx.restore(J.ALL_GROUPS, J.HOST)            # retry: 2-way slices, fresh round generation
for g in w.groups:
    ctx.verify(g.group)
torch.cuda.synchronize()
for st, g in zip(keep, w.groups):
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, w.seed, g.group)), t.name
print("survivor", rank, "retried restore bit-exact in", res["rounds"], "rounds", flush=True)
ctx.close()
"""


def test_restore_aborted_part_way_then_retried():
    """ADVICE r01 (IPC restore rounds): a rank dies after posting its first
    rounds of a 3-way HOST restore, so the survivors' restore aborts with
    JITC_EPEER part-way, with the shared round counters already advanced.  The
    survivors shrink and retry the restore 2-way: every call has its own round
    generation, so no wait can pass on a stale counter of the aborted call, and
    the retry is bit-exact against the oracle."""
    shm = f"/dev/shm/jitc-rretry-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    os.makedirs(shm)
    try:
        procs = []
        for r in range(3):
            env = _env("ipc", r)
            if r == 2:
                env["JITC_DEBUG_EXIT_AFTER_ROUND"] = "2"
            procs.append(subprocess.Popen([sys.executable, "-c", textwrap.dedent(RETRY_RANK.format(
                root=ROOT, rank=r, shm=shm, transport="ipc"))], cwd=ROOT, stdout=subprocess.PIPE,
                stderr=subprocess.STDOUT, text=True, env=env))
        try:
            outs = [p.communicate(timeout=300)[0] for p in procs]
        finally:
            for p in procs:
                if p.poll() is None:
                    p.kill()
        assert procs[2].returncode == 17, "\n=====\n".join(outs)
        for i in (0, 1):
            assert procs[i].returncode == 0 and "retried restore bit-exact" in outs[i], "\n=====\n".join(outs)
    finally:
        shutil.rmtree(shm, ignore_errors=True)
