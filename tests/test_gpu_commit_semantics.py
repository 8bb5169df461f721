"""Commit / restore semantics on B200 (round-2 fixes of ADVICE r01):

* a dropped OPTIONAL group keeps no checkpoint: its commit record from an
  earlier failure is removed, and a HOST restore without a selection only
  restores groups committed at the REQUIRED groups' v* (reading R1: grads-like
  state is kept only if consistent at v*);
* REQUIRED groups committed at different versions are refused
  (JITC_EINCOMPLETE), as is a manifest whose v* is not the selection's;
* the phase word is read as a seqlock around K1: a word that changed while K1
  ran labels the record DIRTY at the newer version (reading R6/R12).

Everything restored is compared with the oracle (bit-exact)."""
import os
import shutil
import threading
import time
import uuid

import numpy as np
import pytest
import torch

from oracle import oracle as O
from workloads import configs as W

pytestmark = pytest.mark.gpu
C = 4096


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    assert torch.cuda.is_available(), "GPU tests need a B200"
    return jitc


@pytest.fixture
def shm():
    d = f"/dev/shm/jitc-cs-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    yield d
    shutil.rmtree(d, ignore_errors=True)


def _groups():
    w = W.scaled(W.c2(world=1), 3000)
    return w.groups[0], w.groups[1], w.seed         # REQUIRED params/master/m/v, OPTIONAL grads


def _select(J, ctx, healthy=(0,)):
    blob = ctx.fingerprint()
    st, sel = J.select_consistent_replica(ctx.exchange_records(blob), list(healthy))
    assert st == J.OK, J.parse_selection(sel)
    return blob, sel


def _same_as_oracle(st, g, seed, v_updates=()):
    torch.cuda.synchronize()
    L = O.lib()
    for i, t in enumerate(g.tensors):
        want = O.gen_tensor_bytes(t, seed, g.group)
        for (idx, v) in v_updates:
            if idx == i:
                w32 = want.view(np.uint32).copy()
                L.orc_update_fp32(O._ptr(w32), 0, t.numel, t.gen_id, v)
                want = w32.view(np.uint8)
        assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), want), t.name


def test_dropped_optional_group_loses_old_commit(J, shm):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    greq, gopt, seed = _groups()
    sr, so = GroupState(greq, seed), GroupState(gopt, seed)
    ctx = J.Context(device=0, chunk_bytes=C, image_dir=shm, staging_bytes=8 << 20, slot_bytes=1 << 20)
    ctx.register(0, J.REQUIRED, [0], sr.table(), keepalive=sr)
    ctx.register(1, J.OPTIONAL, [0], so.table(), keepalive=so)
    # failure 1 at v = 5: both groups CLEAN -> both committed
    ctx.mark(0, 5, J.CLEAN)
    ctx.mark(1, 5, J.CLEAN)
    _, sel5 = _select(J, ctx)
    ctx.capture(sel5)
    ctx.commit(sel5)
    assert os.path.exists(f"{shm}/g1.commit")
    # training goes on: a master tensor changes (step 6); the grads are mid-update
    # (DIRTY) at failure 2, so the selection drops the OPTIONAL group
    i_master = next(i for i, t in enumerate(greq.tensors) if t.name.startswith("master/"))
    tm = greq.tensors[i_master]
    J.inject_update(sr.tensor_bytes(i_master).data_ptr(), 0, tm.numel, tm.gen_id, 6)
    torch.cuda.synchronize()
    ctx.mark(0, 6, J.CLEAN)
    ctx.mark(1, 6, J.DIRTY)
    _, sel6 = _select(J, ctx)
    gsel = {g["group"]: g for g in J.parse_selection(sel6)["groups"]}
    assert gsel[1]["status"] == J.G_DROPPED and gsel[1]["writers"] == []
    ctx.capture(sel6)
    assert not os.path.exists(f"{shm}/g1.commit"), "capture must remove the dropped group's old commit record"
    ctx.commit(sel6)
    assert not os.path.exists(f"{shm}/g1.commit") and not os.path.exists(f"{shm}/g1.manifest")
    # a replacement restores without a selection: only the REQUIRED group, at v* = 6
    sr.scramble()
    so.scramble()
    res = ctx.restore(J.ALL_GROUPS, J.HOST)
    assert (res["groups_done"], res["groups_skipped"]) == (1, 1)   # g1 has no checkpoint: left out
    _same_as_oracle(sr, greq, seed, [(i_master, 6)])


def test_stale_optional_commit_is_skipped_and_required_mismatch_refused(J, shm):
    """A crash between capture and commit could still leave an old commit
    record of the dropped group (before this round's fix it survived every
    later commit).  HOST restore without a selection then takes the REQUIRED
    groups' v* and skips the OPTIONAL group committed at another version; with
    the selection, the dropped group is skipped outright.  REQUIRED groups at
    different versions are refused."""
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    greq, gopt, seed = _groups()
    sr, so = GroupState(greq, seed), GroupState(gopt, seed)
    ctx = J.Context(device=0, chunk_bytes=C, image_dir=shm, staging_bytes=8 << 20, slot_bytes=1 << 20)
    ctx.register(0, J.REQUIRED, [0], sr.table(), keepalive=sr)
    ctx.register(1, J.OPTIONAL, [0], so.table(), keepalive=so)
    ctx.mark(0, 5, J.CLEAN)
    ctx.mark(1, 5, J.CLEAN)
    _, sel5 = _select(J, ctx)
    ctx.capture(sel5)
    ctx.commit(sel5)
    old1 = {ext: open(f"{shm}/g1{ext}", "rb").read() for ext in (".commit", ".manifest")}
    old0 = {ext: open(f"{shm}/g0{ext}", "rb").read() for ext in (".commit", ".manifest")}
    ctx.mark(0, 6, J.CLEAN)
    ctx.mark(1, 6, J.DIRTY)
    _, sel6 = _select(J, ctx)
    ctx.capture(sel6)
    ctx.commit(sel6)
    for ext, b in old1.items():            # the stale v=5 checkpoint of the grads reappears
        open(f"{shm}/g1{ext}", "wb").write(b)
    so.scramble()
    res = ctx.restore(J.ALL_GROUPS, J.HOST)
    assert (res["groups_done"], res["groups_skipped"]) == (1, 1)
    assert int(so.arena[0].item()) == 0xA5, "the stale OPTIONAL group must not be restored"
    res = ctx.restore(J.ALL_GROUPS, J.HOST, sel6)
    assert (res["groups_done"], res["groups_skipped"]) == (1, 1)
    # the same stale manifest against a selection at v* = 5 -> g0 (v* 6) refused
    with pytest.raises(J.JitcError) as e:
        ctx.restore(J.ALL_GROUPS, J.HOST, sel5)
    assert e.value.status == J.EINCOMPLETE
    # REQUIRED groups at different versions: g0 back at v = 5, a second REQUIRED group at 6
    for ext, b in old0.items():
        open(f"{shm}/g0{ext}", "wb").write(b)
    g2 = W.random_table(3, 20, group=2)
    s2 = GroupState(g2, 1)
    ctx.register(2, J.REQUIRED, [0], s2.table(), keepalive=s2)
    ctx.mark(2, 6, J.CLEAN)
    _, sel2 = _select(J, ctx)
    ctx.capture(sel2)
    ctx.commit(sel2)          # g0 and g2 committed at 6; g1 dropped again
    for ext, b in old0.items():
        open(f"{shm}/g0{ext}", "wb").write(b)
    with pytest.raises(J.JitcError) as e:
        ctx.restore(J.ALL_GROUPS, J.HOST)
    assert e.value.status == J.EINCOMPLETE and "different versions" in str(e.value)
    ctx.close()


def test_phase_word_seqlock_marks_torn_fingerprint_dirty(J, shm, monkeypatch):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    greq, _, seed = _groups()
    monkeypatch.setenv("JITC_DEBUG_FP_PAUSE_US", "300000")   # 300 ms between K1's end and the 2nd read
    sr = GroupState(greq, seed)
    ctx = J.Context(device=0, chunk_bytes=C, image_dir=shm, staging_bytes=8 << 20, slot_bytes=1 << 20)
    ctx.register(0, J.REQUIRED, [0], sr.table(), keepalive=sr)
    ctx.mark(0, 9, J.CLEAN)
    [(_, _, _, [rec])] = O.decode_blobs(ctx.fingerprint())
    assert (rec.version, rec.phase) == (9, O.CLEAN)          # unchanged word: CLEAN
    out = {}
    th = threading.Thread(target=lambda: out.setdefault("blob", ctx.fingerprint()))
    th.start()
    time.sleep(0.1)
    ctx.mark(0, 9, J.DIRTY)          # the optimizer step begins while the fingerprint is in flight
    th.join()
    [(_, _, _, [rec])] = O.decode_blobs(out["blob"])
    assert (rec.version, rec.phase) == (9, O.DIRTY)
    st, sel = J.select_consistent_replica(out["blob"], [0])
    assert st != J.OK                                           # a torn lone replica is never selected
    ctx.mark(0, 10, J.CLEAN)
    th = threading.Thread(target=lambda: out.update(blob=ctx.fingerprint()))
    th.start()
    time.sleep(0.1)
    ctx.mark(0, 11, J.CLEAN)         # a whole step completed during K1: also torn
    th.join()
    [(_, _, _, [rec])] = O.decode_blobs(out["blob"])
    assert (rec.version, rec.phase) == (11, O.DIRTY)
    ctx.close()
