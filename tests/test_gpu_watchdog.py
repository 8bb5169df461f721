"""NEXT-1 hang detection on one B200 (§3.1-3.2).

A collective hung on a dead peer is emulated by spinning CTAs on the
training stream (jitc_inject_hang); the event recorded after it never
completes.  The library's watchdog thread must notice the stuck event, then
capture and commit the state by itself -- while the main Python thread holds
the GIL inside a blocking C call (PAPER.md:132's deadlock) and while the hung
kernel still occupies SMs (the default stream is blocked, the
copies run on other streams).  The committed image must restore bit-exact
against the oracle."""
import os
import shutil
import time
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
    return jitc


@pytest.fixture
def shm():
    d = f"/dev/shm/jitc-wd-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    yield d
    shutil.rmtree(d, ignore_errors=True)


def _setup(J, shm, phase):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    g = W.c1().groups[0]
    st = GroupState(g, 0xBEEF)
    ctx = J.Context(device=0, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=256 << 20, slot_bytes=64 << 20)
    ctx.register(0, J.REQUIRED, [0, 1], st.table(), keepalive=st)
    ctx.mark(0, 12, phase)
    torch.cuda.synchronize()
    return g, st, ctx


def test_watchdog_captures_under_hang_holding_gil(J, shm):
    g, st, ctx = _setup(J, shm, J.CLEAN)
    # the replacement's context exists before the hang: nothing below may
    # allocate or free while the emulated collective blocks (cudaFree would
    # synchronise the whole device and wait on the hung kernel)
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    st2 = GroupState(g, 0xBEEF, fill=False, shuffle_seed=5)
    st2.scramble()
    ctx2 = J.Context(device=0, rank=1, world=2, chunk_bytes=1 << 20, image_dir=shm, staging_bytes=256 << 20,
                     slot_bytes=64 << 20)
    ctx2.register(0, J.REQUIRED, [0, 1], st2.table(), keepalive=st2)
    torch.cuda.synchronize()
    train = torch.cuda.Stream()
    J.inject_hang(train.cuda_stream, 32, slot=3)          # the "all-reduce" that never finishes
    ev = torch.cuda.Event()
    ev.record(train)
    try:
        ctx.watch_event(ev.cuda_event, tag=77)
        t0 = time.perf_counter()
        ctx.watchdog_start(timeout_ms=200, action=J.ON_HANG_LOCAL_CAPTURE)
        r = ctx.watchdog_wait(30000, hold_gil=True)          # GIL held while the watchdog works
        dt = (time.perf_counter() - t0) * 1e3
        assert r["fired"] and r["tag"] == 77
        assert 200 <= r["waited_ms"] < 2000 and dt < 10000
        assert r["stats"]["image_bytes"] == 48_138_240 and r["stats"]["d2h_bytes"] == 48_138_240
        assert not ev.query(), "the emulated collective is still hung"
        # the replacement restores the committed image while the hang persists
        res = ctx2.restore(0, J.HOST)
        assert res["image_bytes"] == 48_138_240
        ctx2.verify(0)
        assert not ev.query()
    finally:
        J.inject_release(3)
    train.synchronize()
    assert ev.query()
    torch.cuda.synchronize()
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st2.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 0xBEEF, 0)), t.name
    ctx2.close()
    ctx.close()


def test_watchdog_no_false_positive(J, shm):
    g, st, ctx = _setup(J, shm, J.CLEAN)
    s = torch.cuda.Stream()
    ctx.watchdog_start(timeout_ms=300, action=J.ON_HANG_LOCAL_CAPTURE)
    for i in range(50):                                      # collectives that complete
        ev = torch.cuda.Event()
        ev.record(s)
        ctx.watch_event(ev.cuda_event, tag=i)
        time.sleep(0.01)
    r = ctx.watchdog_wait(600)
    assert not r["fired"]
    ctx.watchdog_stop()
    assert not os.path.exists(f"{shm}/g0.commit")
    ctx.close()


def test_watchdog_dirty_rank_refuses(J, shm):
    """A rank that hangs inside its own optimizer step (phase DIRTY) must not
    save a partially updated state: the local capture fails with
    ENOCONSISTENT and nothing is committed."""
    g, st, ctx = _setup(J, shm, J.DIRTY)
    train = torch.cuda.Stream()
    J.inject_hang(train.cuda_stream, 8, slot=4)
    ev = torch.cuda.Event()
    ev.record(train)
    try:
        ctx.watch_event(ev.cuda_event, tag=1)
        ctx.watchdog_start(timeout_ms=100, action=J.ON_HANG_LOCAL_CAPTURE)
        with pytest.raises(J.JitcError) as e:
            ctx.watchdog_wait(30000)
        assert e.value.status == J.ENOCONSISTENT
        assert not os.path.exists(f"{shm}/g0.commit")
    finally:
        J.inject_release(4)
    train.synchronize()
    ctx.close()
