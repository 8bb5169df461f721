"""Multi-rank scenarios of SURVEY.md §8(d) (C4 ZeRO-1, C5 TP4xDP2) on one
B200: 8 job ranks run as 8 library contexts in one process, sharing one
/dev/shm image directory like the ranks of a box.  Blobs are concatenated in
rank order (what jitc_exchange_records returns; only the NCCL transport is
bypassed, it needs 8 GPUs).  Every writer captures its own 1/k shard into the
shared image, the lowest writer commits, a replacement restores, and the
restored bytes are compared with the oracle's expected state -- including a
half-applied optimizer step, DIRTY phases, bit flips in HBM and in the image.
Shapes are the configs' tensor tables clipped to a few thousand elements."""
import copy
import os
import shutil
import uuid

import numpy as np
import pytest
import torch

from oracle import oracle as O
from workloads import configs as W

pytestmark = pytest.mark.gpu
V = 40          # minibatch index at failure
C = 4096


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    return jitc


@pytest.fixture
def shm():
    d = f"/dev/shm/jitc-scn-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    yield d
    shutil.rmtree(d, ignore_errors=True)


class Job:
    """world contexts on one GPU; rank r holds w.groups_of(r)."""

    def __init__(self, J, w, shm, dead=()):
        from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
        self.J, self.w, self.shm = J, w, shm
        self.ctx, self.states = {}, {}
        for r in range(w.world):
            if r in dead:
                continue
            ctx = J.Context(device=0, rank=r, world=w.world, chunk_bytes=C, staging_bytes=8 << 20,
                            slot_bytes=1 << 20, image_dir=shm)
            for g in w.groups:
                if r in g.members:
                    st = GroupState(g, w.seed, shuffle_seed=100 + r)
                    self.states[(r, g.group)] = st
                    ctx.register(g.group, g.policy, g.members, st.table(), keepalive=st)
                    ctx.mark(g.group, V, J.CLEAN)
                else:
                    ctx.declare_group(g.group, g.policy, g.members)
            self.ctx[r] = ctx
        torch.cuda.synchronize()

    def select(self, healthy=None):
        healthy = sorted(self.ctx) if healthy is None else healthy
        blobs = b"".join(self.ctx[r].fingerprint() for r in sorted(self.ctx))
        st, sel = self.J.select_consistent_replica(blobs, healthy)
        ref = O.select(blobs, healthy)
        assert st == ref.status
        got = self.J.parse_selection(sel)
        if st == 0:
            assert got["v_star"] == ref.v_star
            for a, b in zip(got["groups"], ref.groups):
                assert (a["group"], a["writers"], sorted(a["excluded"]), a["status"]) == \
                       (b.group, b.writers, sorted(b.excluded), b.status)
        return st, sel, got

    def capture_commit(self, sel):
        caps = {r: self.ctx[r].capture(sel) for r in sorted(self.ctx)}   # non-writers return at once
        for r in sorted(self.ctx):
            self.ctx[r].commit(sel)
        return caps

    def close(self):
        for c in self.ctx.values():
            c.close()


def _expected(g, seed, updates):
    """Oracle state of group g after the given U_v updates:
    updates = list of (v, [tensor indices])."""
    L = O.lib()
    out = []
    for i, t in enumerate(g.tensors):
        b = O.gen_tensor_bytes(t, seed, g.group).copy()
        for v, idx in updates:
            if i in idx:
                x = b.view(np.uint32)
                L.orc_update_fp32(O._ptr(x), 0, len(x), t.gen_id, v)
        out.append(b)
    return out


def _restore_into_fresh(J, w, shm, rank, groups, expect):
    """A replacement process for `rank`: fresh tensors, HOST restore from the
    committed shared image, byte comparison with the oracle."""
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    ctx = J.Context(device=0, rank=rank, world=w.world, chunk_bytes=C, staging_bytes=8 << 20, slot_bytes=1 << 20,
                    image_dir=shm)
    sts = {}
    for g in w.groups:
        if rank in g.members:
            st = GroupState(g, w.seed, fill=False, shuffle_seed=999)
            st.scramble()
            sts[g.group] = st
            ctx.register(g.group, g.policy, g.members, st.table(), keepalive=st)
        else:
            ctx.declare_group(g.group, g.policy, g.members)
    for gid in groups:
        ctx.restore(gid, J.HOST)
        ctx.verify(gid)
    torch.cuda.synchronize()
    for gid in groups:
        g = next(x for x in w.groups if x.group == gid)
        for i, t in enumerate(g.tensors):
            assert np.array_equal(sts[gid].tensor_bytes(i).cpu().numpy(), expect[gid][i]), (gid, t.name)
    ctx.close()


def _small(w, n=3000):
    w = W.scaled(w, n)
    for g in w.groups:
        for t in g.tensors:
            if t.dtype == "bf16" and t.numel % 2:
                t.numel += 1          # keep bf16 tensors a whole number of u32 words (U_v is per u32)
    return w


def test_c5_tp4_dp2_sharded_capture_and_replacement(J, shm):
    """C5: TP partition p on ranks {p, p+4}; rank 5 dies.  Partition 1 has a
    single (unverified) replica, the others two writers each capturing half
    of the shared image; the replacement for rank 5 restores partition 1."""
    w = _small(W.c5(n_layer=2))
    job = Job(J, w, shm, dead=(5,))
    st, sel, got = job.select()
    assert st == 0 and got["v_star"] == V
    g = {x["group"]: x for x in got["groups"]}
    assert g[1]["writers"] == [1] and g[1]["status"] == J.parse_selection(sel)["groups"][1]["status"] == 1
    assert g[0]["writers"] == [0, 4] and g[2]["writers"] == [2, 6] and g[5]["writers"] == [1]
    caps = job.capture_commit(sel)
    for gid in (0, 2):                     # two writers: each wrote about half of the image
        lay = O.layout_of_group(w.groups[gid], C)
        img = np.fromfile(f"{shm}/g{gid}.img", dtype=np.uint8)[:lay.L]
        assert np.array_equal(img, O.pack(_expected(w.groups[gid], w.seed, []), lay))
    assert caps[0]["image_bytes"] + caps[4]["image_bytes"] >= O.layout_of_group(w.groups[0], C).L
    assert caps[0]["image_bytes"] < O.layout_of_group(w.groups[0], C).L
    expect = {gid: _expected(w.groups[gid], w.seed, []) for gid in (1, 5)}
    _restore_into_fresh(J, w, shm, 5, [1, 5], expect)
    job.close()


def test_manifest_and_commit_record_bytes_equal_oracle(J, shm):
    """A8 parity (byte work => bit-exact): the manifest and commit record the
    library writes for every C5 group -- k = 2 writers, a lone writer after
    rank 5 died, the user's CPU-state aux bytes -- equal the
    oracle's O4b encoding of the oracle's own selection,
    layout and digests, byte for byte."""
    w = _small(W.c5(n_layer=2))
    job = Job(J, w, shm, dead=(5,))
    aux = b"iteration=40;rng=" + bytes(range(29))
    for c in job.ctx.values():
        c.set_aux(aux)
    healthy = sorted(job.ctx)
    blobs = b"".join(job.ctx[r].fingerprint() for r in healthy)
    ref = O.select(blobs, healthy)
    st, sel, got = job.select()
    assert st == 0
    job.capture_commit(sel)
    n_checked = 0
    for gs in ref.groups:
        if not gs.writers:
            continue
        g = next(x for x in w.groups if x.group == gs.group)
        lay = O.layout_of_group(g, C)
        d = O.jf64(O.pack(_expected(g, w.seed, []), lay), C, 0, lay.n_c)
        want_man = O.encode_manifest(gs, ref.v_star, lay, d, aux)
        got_man = open(f"{shm}/g{gs.group}.manifest", "rb").read()
        assert got_man == want_man, gs.group
        assert open(f"{shm}/g{gs.group}.commit", "rb").read() == O.commit_record(gs.group, ref.v_star, want_man)
        n_checked += 1
    assert n_checked == len(w.groups)
    job.close()


def test_fingerprint_blobs_bytes_equal_oracle(J, shm):
    """A3/A4 parity: every rank's fingerprint blob -- header, job topology
    (including groups it only declares) and one O4 record per held group with
    the K1 digests and root -- equals the oracle's encoding of the oracle's
    layout, digests and phase word, byte for byte (C5, TP4 x DP2, 8 ranks;
    one rank DIRTY at the next version to cover the phase/version fields)."""
    w = _small(W.c5(n_layer=2))
    job = Job(J, w, shm)
    job.ctx[3].mark(3, V + 1, J.DIRTY)
    torch.cuda.synchronize()
    topo = [O.TopoEntry(g.group, g.policy, list(g.members)) for g in w.groups]
    digests = {}
    for g in w.groups:
        lay = O.layout_of_group(g, C)
        d = O.jf64(O.pack(_expected(g, w.seed, []), lay), C, 0, lay.n_c)
        digests[g.group] = (lay, d)
    for r in sorted(job.ctx):
        recs = []
        for g in w.groups:
            if r not in g.members:
                continue
            lay, d = digests[g.group]
            version, phase = (V + 1, O.DIRTY) if (r, g.group) == (3, 3) else (V, O.CLEAN)
            recs.append(O.Record(r, g.group, g.policy, phase, version, lay.layout_hash, C, lay.L, d,
                                 O.root(lay.layout_hash, d)))
        assert job.ctx[r].fingerprint() == O.encode_blob(r, topo, recs), r
    job.close()


def test_c5_bitflip_conflict_and_image_corruption(J, shm):
    """C5 injections: a flip in rank 2's master (HBM) makes partition 2 a 1-1
    tie (ECONFLICT, the flipped chunk listed); after a clean capture, a flip
    in partition 1's committed image is caught at the exact chunk."""
    w = _small(W.c5(n_layer=2))
    job = Job(J, w, shm)
    gi = next(i for i, t in enumerate(w.groups[2].tensors) if t.name.startswith("master/"))
    lay2 = O.layout_of_group(w.groups[2], C)
    J.inject_bitflip(job.states[(2, 2)].ptrs[gi], 10, 3)
    torch.cuda.synchronize()
    st, sel, got = job.select()
    assert st == J.ECONFLICT
    g2 = next(x for x in got["groups"] if x["group"] == 2)
    assert g2["conflict_chunks"] == [(lay2.offsets[gi] + 10) // C]
    J.inject_bitflip(job.states[(2, 2)].ptrs[gi], 10, 3)   # undo
    torch.cuda.synchronize()
    st, sel, got = job.select()
    assert st == 0
    job.capture_commit(sel)
    lay1 = O.layout_of_group(w.groups[1], C)
    pos = lay1.L // 2 + 7
    with open(f"{shm}/g1.img", "r+b") as f:
        f.seek(pos); b = f.read(1); f.seek(pos); f.write(bytes([b[0] ^ 0x80]))
    with pytest.raises(J.JitcError) as e:
        job.ctx[1].restore(1, J.HOST)
    assert e.value.status == J.ECORRUPT and e.value.first_bad == pos // C
    job.close()


def _zero_step(J, job, w, dead, params_done, half):
    """One synthetic ZeRO-1 optimizer step to version V+1 (SURVEY d.1 C4):
    mark(opt, DIRTY) -> U_{V+1} on the shard -> mark(opt, V+1);
    mark(params, DIRTY) -> param gather -> mark(params, V+1) on ranks whose
    gather completed.  The dead rank stops after updating `half` of its shard."""
    for r, ctx in job.ctx.items():
        for g in w.groups:
            if r not in g.members or g.group < 2:
                continue
            st = job.states[(r, g.group)]
            ctx.mark(g.group, V, J.DIRTY)
            n = len(g.tensors) if r != dead else half
            for i in range(n):
                J.inject_update(st.ptrs[i], 0, g.tensors[i].nbytes // 4, g.tensors[i].gen_id, V + 1)
            if r != dead:
                ctx.mark(g.group, V + 1, J.CLEAN)
        pst = job.states[(r, 0)]
        ctx.mark(0, V, J.DIRTY)
        if r in params_done:
            for i, t in enumerate(w.groups[0].tensors):
                J.inject_update(pst.ptrs[i], 0, t.nbytes // 4, t.gen_id, V + 1)
            ctx.mark(0, V + 1, J.CLEAN)
    torch.cuda.synchronize()


def test_c4_hybrid_zero_mid_update_failure(J, shm):
    """S8 on real state: hybrid ZeRO S=4 x R=2, rank 2 dies halfway through
    its optimizer shard; params gathered inside {0-3} and {4-7}, so {4..7}
    complete.  v* = V+1, params from {4..7}, shard 2 from rank 6 alone, grads
    (still at V) dropped; the replacement for rank 2 restores the post-step
    state, which equals the oracle's U_{V+1} applied to every tensor."""
    w = _small(W.c4(shards=4), 2000)
    job = Job(J, w, shm)
    _zero_step(J, job, w, dead=2, params_done={4, 5, 6, 7}, half=1)
    healthy = [r for r in range(8) if r != 2]
    st, sel, got = job.select(healthy)
    assert st == 0 and got["v_star"] == V + 1
    g = {x["group"]: x for x in got["groups"]}
    assert g[0]["writers"] == [4, 5, 6, 7] and sorted(g[0]["excluded"]) == [(0, 1), (1, 1), (3, 1)]
    assert g[4]["writers"] == [6] and g[1]["status"] == 3 and g[1]["writers"] == []
    job.capture_commit(sel)
    all_idx = lambda gid: list(range(len(w.groups[gid].tensors)))
    expect = {0: _expected(w.groups[0], w.seed, [(V + 1, all_idx(0))]),
              4: _expected(w.groups[4], w.seed, [(V + 1, all_idx(4))])}
    _restore_into_fresh(J, w, shm, 2, [0, 4], expect)
    job.close()


def test_c4_global_gather_inconsistent_and_pure_zero(J, shm):
    """S9: with a global param gather nobody finishes the params, the shards
    are only at V+1 -> ENOCONSISTENT (a partial update is detected and the
    library refuses).  S7: pure ZeRO (S=8), a dead rank's shard has no replica
    -> ENOREPLICA."""
    w = _small(W.c4(shards=4), 1500)
    job = Job(J, w, shm)
    _zero_step(J, job, w, dead=2, params_done=set(), half=1)
    st, sel, got = job.select([r for r in range(8) if r != 2])
    assert st == J.ENOCONSISTENT
    job.close()
    shutil.rmtree(shm, ignore_errors=True)
    w8 = _small(W.c4(shards=8), 800)
    job = Job(J, w8, shm, dead=(3,))
    st, sel, got = job.select()
    assert st == J.ENOREPLICA
    job.close()
