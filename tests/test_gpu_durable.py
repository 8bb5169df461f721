"""NEXT-4, durable tier (§6.3): a committed JIT image is
persisted to disk (O_DIRECT, manifest, commit record last), survives the loss
of the host image, is staged back and restored bit-exact against the oracle;
a corrupted or uncommitted durable copy is refused."""
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
    return jitc


@pytest.fixture
def dirs():
    tag = f"{os.getpid()}-{uuid.uuid4().hex[:8]}"
    d = (f"/dev/shm/jitc-dur-a-{tag}", f"/dev/shm/jitc-dur-b-{tag}", f"/tmp/jitc-durable-{tag}")
    yield d
    for x in d:
        shutil.rmtree(x, ignore_errors=True)


def test_persist_stage_in_restore(J, dirs):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    shm_a, shm_b, disk = dirs
    w = W.scaled(W.c2(), 200000)
    kw = dict(device=0, chunk_bytes=1 << 20, staging_bytes=256 << 20, slot_bytes=64 << 20)
    ctx = J.Context(image_dir=shm_a, **kw)
    sts = {}
    for g in w.groups:
        sts[g.group] = GroupState(g, w.seed)
        ctx.register(g.group, g.policy, [0], sts[g.group].table(), keepalive=sts[g.group])
        ctx.mark(g.group, 3, J.CLEAN)
    with pytest.raises(J.JitcError) as e:          # nothing committed yet
        ctx.persist(0, disk)
    assert e.value.status == J.EINCOMPLETE
    ctx.capture_local()
    for g in w.groups:
        s = ctx.persist(g.group, disk)
        assert s["image_bytes"] >= O.layout_of_group(g, 1 << 20).L
    ctx.close()
    shutil.rmtree(shm_a)                            # every host image is lost
    ctx2 = J.Context(image_dir=shm_b, **kw)
    sts2 = {}
    for g in w.groups:
        sts2[g.group] = GroupState(g, w.seed, fill=False, shuffle_seed=3)
        sts2[g.group].scramble()
        ctx2.register(g.group, g.policy, [0], sts2[g.group].table(), keepalive=sts2[g.group])
    with pytest.raises(J.JitcError) as e:           # nothing staged yet
        ctx2.restore(0, J.HOST)
    assert e.value.status == J.EINCOMPLETE
    for g in w.groups:
        ctx2.stage_in(g.group, disk)
    ctx2.restore(J.ALL_GROUPS, J.HOST)
    torch.cuda.synchronize()
    for g in w.groups:
        ctx2.verify(g.group)
        for i, t in enumerate(g.tensors):
            assert np.array_equal(sts2[g.group].tensor_bytes(i).cpu().numpy(),
                                  O.gen_tensor_bytes(t, w.seed, g.group)), t.name
    # a flipped byte in the durable image is caught by K3 at the exact chunk
    lay = O.layout_of_group(w.groups[0], 1 << 20)
    pos = lay.L - 1000
    with open(f"{disk}/g0.img", "r+b") as f:
        f.seek(pos); b = f.read(1); f.seek(pos); f.write(bytes([b[0] ^ 1]))
    ctx2.stage_in(0, disk)
    with pytest.raises(J.JitcError) as e:
        ctx2.restore(0, J.HOST)
    assert e.value.status == J.ECORRUPT and e.value.first_bad == pos >> 20
    # a torn commit record is refused before any byte is read
    with open(f"{disk}/g1.commit", "r+b") as f:
        f.seek(20); f.write(b"\xff")
    with pytest.raises(J.JitcError) as e:
        ctx2.stage_in(1, disk)
    assert e.value.status == J.EINCOMPLETE
    ctx2.close()
