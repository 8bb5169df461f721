"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  All of this is integer / byte work, so the bar is
bit-exact (BASELINE.json north_star)."""
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


@pytest.fixture
def shm():
    d = f"/dev/shm/jitc-test-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    yield d
    shutil.rmtree(d, ignore_errors=True)


def _state(g, seed, **kw):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    return GroupState(g, seed, **kw)


def _ctx(J, C, image_dir=None, flags=0, staging=64 << 20, slot=8 << 20, rank=0, world=1):
    return J.Context(device=0, rank=rank, world=world, chunk_bytes=C, staging_bytes=staging, slot_bytes=slot,
                     image_dir=image_dir, flags=flags | J.F_TIME_KERNELS)


def _records(blob):
    [(rank, topo, th, recs)] = O.decode_blobs(blob)
    return {r.group: r for r in recs}


def _small_groups():
    gs = [W.random_table(s, 60, max_bytes=20000, group=s) for s in range(3)]
    gs.append(W.scaled(W.c2(), 40000).groups[0])
    gs[-1].group = 7
    return gs


# ------------------------------------------------------------------ K4 generator
def test_k4_generator_matches_oracle(J):
    for g in _small_groups()[:2] + [W.c1().groups[0]]:
        st = _state(g, 0x1234)
        torch.cuda.synchronize()
        for i, t in enumerate(g.tensors):
            got = st.tensor_bytes(i).cpu().numpy()
            want = O.gen_tensor_bytes(t, 0x1234, g.group)
            assert np.array_equal(got, want), t.name


def test_k4_update_and_rne_match_oracle(J):
    g = W.c1().groups[0]
    st = _state(g, 7)
    L = O.lib()
    for i in (0, 5, 60):
        t = g.tensors[i]
        x = st.tensor_bytes(i)
        J.inject_update(x.data_ptr(), 3, t.numel - 3, t.gen_id, 11)
        torch.cuda.synchronize()
        want = O.gen_tensor_bytes(t, 7, g.group).view(np.uint32).copy()
        L.orc_update_fp32(O._ptr(want[3:]), 3, t.numel - 3, t.gen_id, 11)
        assert np.array_equal(x.cpu().numpy().view(np.uint32), want)
        p = torch.empty(t.numel, dtype=torch.int16, device="cuda")
        J.inject_rne(x.data_ptr(), p.data_ptr(), t.numel)
        torch.cuda.synchronize()
        ref = torch.from_numpy(want.view(np.float32).copy()).to(torch.bfloat16).view(torch.int16)
        assert torch.equal(p.cpu(), ref)


# ------------------------------------------------------------------ K1 fingerprint
@pytest.mark.parametrize("C", [4096, 1 << 20])
@pytest.mark.parametrize("misalign", [0, 1, 2, 8])
def test_k1_digests_match_oracle(J, C, misalign):
    for g in _small_groups():
        st = _state(g, 99, misalign=misalign)
        ctx = _ctx(J, C)
        lh, L = ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
        lay = O.layout_of_group(g, C)
        assert (lh, L) == (lay.layout_hash, lay.L)
        ctx.mark(g.group, 5, J.CLEAN)
        rec = _records(ctx.fingerprint(g.group))[g.group]
        img = O.pack(O.gen_group(g, 99), lay)
        d = O.jf64(img, C, 0, lay.n_c)
        assert np.array_equal(rec.d, d)
        assert rec.root == O.root(lay.layout_hash, d) and rec.version == 5 and rec.phase == O.CLEAN
        ctx.close()


def test_k1_c1_full(J):
    w = W.c1()
    g = w.groups[0]
    st = _state(g, w.seed)
    ctx = _ctx(J, 1 << 20)
    ctx.register(0, J.REQUIRED, [0, 1], st.table(), keepalive=st)
    rec = _records(ctx.fingerprint())[0]
    lay = O.layout_of_group(g, 1 << 20)
    d = O.jf64(O.pack(O.gen_group(g, w.seed), lay), lay.C, 0, lay.n_c)
    assert lay.L == 48_138_240 and np.array_equal(rec.d, d)


def test_phase_word_stream_ordered(J):
    g = W.random_table(1, 4)
    st = _state(g, 1)
    ctx = _ctx(J, 4096)
    ctx.register(0, J.REQUIRED, [0], st.table(), keepalive=st)
    s = torch.cuda.Stream()
    ctx.mark(0, 41, J.DIRTY, s.cuda_stream)
    s.synchronize()
    assert ctx.phase(0) == (41, J.DIRTY)
    ctx.mark(0, 42, J.CLEAN, s.cuda_stream)
    s.synchronize()
    assert ctx.phase(0) == (42, J.CLEAN)
    ctx.mark(0, 43, J.DIRTY)          # host write
    assert ctx.phase(0) == (43, J.DIRTY)
    rec = _records(ctx.fingerprint())[0]
    assert (rec.version, rec.phase) == (43, O.DIRTY)


# ------------------------------------------------------------------ capture / restore
def _pipeline(J, ctx, healthy=(0,)):
    blob = ctx.fingerprint()
    allb = ctx.exchange_records(blob)
    st, sel = J.select_consistent_replica(allb, list(healthy))
    assert st == J.OK, J.parse_selection(sel)
    cap = ctx.capture(sel)
    ctx.commit(sel)
    return blob, sel, cap


@pytest.mark.parametrize("flags", [0, 1, 2, 3])     # staging+CE / zero-copy D2H / zero-copy H2D / both
@pytest.mark.parametrize("C", [4096, 1 << 20])
def test_capture_restore_bit_exact(J, shm, flags, C):
    for g in _small_groups():
        st = _state(g, 5, misalign=2 if g.group == 1 else 0)
        ctx = _ctx(J, C, image_dir=shm, flags=flags, staging=4 * C * 4, slot=4 * C)
        ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
        ctx.mark(g.group, 3, J.CLEAN)
        blob, sel, cap = _pipeline(J, ctx)
        lay = O.layout_of_group(g, C)
        want = O.pack(O.gen_group(g, 5), lay)
        img = np.fromfile(f"{shm}/g{g.group}.img", dtype=np.uint8)[:lay.L]
        assert np.array_equal(img, want)                       # K2 image == oracle pack
        assert cap["image_bytes"] == lay.L and cap["kernel_launches"] >= 1
        st.scramble()
        res = ctx.restore(g.group, J.HOST)
        torch.cuda.synchronize()
        for i, t in enumerate(g.tensors):                      # K3 restore == original state
            assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 5, g.group)), t.name
        assert ctx.verify(g.group) == 2**64 - 1
        assert ctx.verify(g.group, blob) == 2**64 - 1
        ctx.close()


def _segment_edge_table():
    """Tensors whose sizes straddle the kernels' 128 KiB segment (work unit)
    and the 64 KiB / 1 MiB chunks: every piece shape K1/K2/K3 cut a tensor
    into (whole segments, a ragged last segment, a < 16-B data tail, pieces
    ended by a chunk edge), with vector and scalar paths via misalignment."""
    K = 1 << 17
    g = W.GroupSpec(11, W.REQUIRED, [0])
    sizes = [K - 16, K - 1, K, K + 1, K + 8, K + 16, K + 17, 2 * K + 3, (1 << 20) - 1, (1 << 20) + 5,
             3 * (1 << 20) + 7, 40000, 5]
    for i, b in enumerate(sizes):
        g.tensors.append(W.TensorSpec(f"u{i}", "u8", b, "bytes", i))
    g.tensors.append(W.TensorSpec("f", "f32", 300_001, "master", 100))
    g.tensors.append(W.TensorSpec("h", "bf16", 200_001, "grad", 101))
    g.tensors.append(W.TensorSpec("z", "zeros", K + 3, "bytes", 102))
    return g


@pytest.mark.parametrize("C", [1 << 16, 1 << 20])
@pytest.mark.parametrize("misalign", [0, 1, 2, 8])
def test_segment_boundaries_bit_exact(J, shm, C, misalign):
    """K1 digests, the K2 image, the K3 restore and A12 verify equal the oracle
    on tensors cut at every kind of segment / chunk boundary (round-2 128 KiB
    segments, 512-thread read+write CTAs, 8-load K1)."""
    g = _segment_edge_table()
    st = _state(g, 77, misalign=misalign)
    ctx = _ctx(J, C, image_dir=shm, staging=8 * C * 4, slot=4 * C)
    lh, L = ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    lay = O.layout_of_group(g, C)
    assert (lh, L) == (lay.layout_hash, lay.L)
    ctx.mark(g.group, 9, J.CLEAN)
    blob, sel, cap = _pipeline(J, ctx)
    want = O.pack(O.gen_group(g, 77), lay)
    assert np.array_equal(_records(blob)[g.group].d, O.jf64(want, C, 0, lay.n_c))
    img = np.fromfile(f"{shm}/g{g.group}.img", dtype=np.uint8)[:lay.L]
    assert np.array_equal(img, want)
    st.scramble()
    ctx.restore(g.group, J.HOST)
    torch.cuda.synchronize()
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 77, g.group)), t.name
    assert ctx.verify(g.group, blob) == 2**64 - 1
    ctx.close()


@pytest.mark.parametrize("flags", [0, 3])
@pytest.mark.parametrize("piece_mb", [1, 3])
def test_capture_restore_image_pinned_in_pieces(J, shm, monkeypatch, flags, piece_mb):
    """The shared host image is pinned as separate registrations (1 GiB
    pieces in production; 1 and 3 MiB here so that small images span many):
    copy-engine transfers must split at every piece boundary, and the
    zero-copy kernels must see the pieces as one contiguous mapping.  Image and
    restored tensors bit-exact vs the oracle."""
    monkeypatch.setenv("JITC_PIN_PIECE_MB", str(piece_mb))
    g = _small_groups()[-1]                       # C2 table clipped: ~20 MB image
    C = 1 << 20
    st = _state(g, 6, misalign=2)
    ctx = _ctx(J, C, image_dir=shm, flags=flags, staging=8 * C * 2, slot=8 * C)
    ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    ctx.mark(g.group, 3, J.CLEAN)
    lay = O.layout_of_group(g, C)
    assert lay.L > 4 * (piece_mb << 20)
    blob, sel, cap = _pipeline(J, ctx)
    want = O.pack(O.gen_group(g, 6), lay)
    assert np.array_equal(np.fromfile(f"{shm}/g{g.group}.img", dtype=np.uint8)[:lay.L], want)
    st.scramble()
    ctx.restore(g.group, J.HOST)
    torch.cuda.synchronize()
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 6, g.group)), t.name
    ctx.close()


def test_restore_in_fresh_context_from_shm(J, shm):
    """A replacement process registers the same tensors and restores from the
    committed shared image (HOST mode, selection from the manifest)."""
    g = W.scaled(W.c1(), 5000).groups[0]
    st = _state(g, 8)
    ctx = _ctx(J, 4096, image_dir=shm)
    ctx.register(0, J.REQUIRED, [0, 1], st.table(), keepalive=st)
    ctx.mark(0, 9, J.CLEAN)
    _pipeline(J, ctx)
    ctx.close()
    st2 = _state(g, 8, fill=False, shuffle_seed=9)
    st2.scramble()
    ctx2 = _ctx(J, 4096, image_dir=shm, rank=1, world=2)
    ctx2.register(0, J.REQUIRED, [0, 1], st2.table(), keepalive=st2)
    ctx2.restore(0, J.HOST)
    torch.cuda.synchronize()
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st2.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 8, 0))


def test_corrupt_host_image_exact_chunk(J, shm):
    g = _small_groups()[3]
    C = 4096
    st = _state(g, 6)
    ctx = _ctx(J, C, image_dir=shm)
    ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    _pipeline(J, ctx)
    lay = O.layout_of_group(g, C)
    rng = np.random.default_rng(1)
    for _ in range(5):
        pos = int(rng.integers(0, lay.L))
        with open(f"{shm}/g{g.group}.img", "r+b") as f:
            f.seek(pos); b = f.read(1); f.seek(pos); f.write(bytes([b[0] ^ 0x10]))
        with pytest.raises(J.JitcError) as e:
            ctx.restore(g.group, J.HOST)
        assert e.value.status == J.ECORRUPT and e.value.first_bad == pos // C
        with open(f"{shm}/g{g.group}.img", "r+b") as f:
            f.seek(pos); f.write(b)
    ctx.restore(g.group, J.HOST)


def test_fuzzed_manifest_and_commit_record_refused(J, shm):
    """Robustness of the metadata path (PAPER.md:136, :140 -- a checkpoint
    whose metadata is incomplete or corrupted is discarded): 300 random
    single-byte changes and truncations of the committed manifest and commit
    record.  Every one must be refused with EINCOMPLETE or ELAYOUT -- never
    accepted, never a crash -- and the intact files then restore bit-exact."""
    g = _small_groups()[3]
    C = 4096
    st = _state(g, 6)
    ctx = _ctx(J, C, image_dir=shm)
    ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    _pipeline(J, ctx)
    paths = {k: f"{shm}/g{g.group}.{k}" for k in ("manifest", "commit")}
    orig = {k: open(p, "rb").read() for k, p in paths.items()}
    rng = np.random.default_rng(11)
    seen = set()
    for it in range(300):
        which = "manifest" if it % 3 else "commit"
        b = bytearray(orig[which])
        if it % 10 == 9:
            b = b[:int(rng.integers(0, len(b)))]                 # torn write
        else:
            pos = int(rng.integers(0, len(b)))
            b[pos] ^= int(rng.integers(1, 256))                  # any change to one byte
        with open(paths[which], "wb") as f:
            f.write(bytes(b))
        with pytest.raises(J.JitcError) as e:
            ctx.restore(g.group, J.HOST)
        assert e.value.status in (J.EINCOMPLETE, J.ELAYOUT), (which, it, e.value)
        seen.add(e.value.status)
        with open(paths[which], "wb") as f:
            f.write(orig[which])
    assert J.EINCOMPLETE in seen
    st.scramble()
    ctx.restore(g.group, J.HOST)
    ctx.verify(g.group)
    torch.cuda.synchronize()
    for i, t in enumerate(g.tensors):
        assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 6, g.group)), t.name
    ctx.close()


def test_uncommitted_refused(J, shm):
    g = W.random_table(4, 10)
    st = _state(g, 6)
    ctx = _ctx(J, 4096, image_dir=shm)
    ctx.register(0, J.REQUIRED, [0], st.table(), keepalive=st)
    _pipeline(J, ctx)
    os.unlink(f"{shm}/g0.commit")
    with pytest.raises(J.JitcError) as e:
        ctx.restore(0, J.HOST)
    assert e.value.status == J.EINCOMPLETE


def test_hbm_bitflip_detected_by_verify(J):
    g = _small_groups()[3]
    C = 4096
    st = _state(g, 2)
    ctx = _ctx(J, C)
    ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    blob = ctx.fingerprint()
    lay = O.layout_of_group(g, C)
    for i in (0, 3, len(g.tensors) - 1):
        nb = g.tensors[i].nbytes
        byte = nb // 2
        J.inject_bitflip(st.ptrs[i], byte, 5)
        with pytest.raises(J.JitcError) as e:
            ctx.verify(g.group, blob)
        assert e.value.status == J.ECORRUPT and e.value.first_bad == (lay.offsets[i] + byte) // C
        J.inject_bitflip(st.ptrs[i], byte, 5)
    ctx.verify(g.group, blob)


def test_unstable_between_fingerprint_and_capture(J, shm):
    g = _small_groups()[0]
    st = _state(g, 2)
    ctx = _ctx(J, 4096, image_dir=shm)
    ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
    blob = ctx.fingerprint()
    st_, sel = J.select_consistent_replica(blob, [0])
    J.inject_bitflip(st.ptrs[2], 0, 0)
    with pytest.raises(J.JitcError) as e:
        ctx.capture(sel)
    assert e.value.status == J.EUNSTABLE


def test_capture_pipeline_across_groups(J, shm):
    """jitc_capture runs the rounds of all groups as one pipeline (short first
    round, slots carried across groups): every group's image == the oracle's
    pack; a change in the SECOND group between fingerprint and capture is
    EUNSTABLE naming that group, after which commit refuses before writing
    anything (the group is not captured; no group gets a commit record) and a
    fresh fingerprint -> capture -> commit -> restore works."""
    C = 4096
    gs = [W.random_table(40 + i, 50, max_bytes=30000, group=i) for i in range(3)]
    sts = [_state(g, 8 + g.group) for g in gs]
    ctx = _ctx(J, C, image_dir=shm, staging=8 * C * 4, slot=4 * C)   # rounds of 4 chunks, 8 slots
    for g, st in zip(gs, sts):
        ctx.register(g.group, J.REQUIRED, [0], st.table(), keepalive=st)
        ctx.mark(g.group, 4, J.CLEAN)
    blob = ctx.fingerprint()
    st_, sel = J.select_consistent_replica(blob, [0])
    J.inject_bitflip(sts[1].ptrs[3], 0, 1)
    with pytest.raises(J.JitcError) as e:
        ctx.capture(sel)
    assert e.value.status == J.EUNSTABLE and "group 1" in str(e.value)
    with pytest.raises(J.JitcError) as e:
        ctx.commit(sel)
    assert e.value.status == J.ESTATE
    assert not any(os.path.exists(f"{shm}/g{g.group}.commit") for g in gs), "no partial commit"
    J.inject_bitflip(sts[1].ptrs[3], 0, 1)                    # undo: the state is the oracle's again
    blob, sel, cap = _pipeline(J, ctx)
    assert cap["rounds"] >= 3
    for g in gs:
        lay = O.layout_of_group(g, C)
        img = np.fromfile(f"{shm}/g{g.group}.img", dtype=np.uint8)[:lay.L]
        assert np.array_equal(img, O.pack(O.gen_group(g, 8 + g.group), lay)), g.group
    for st in sts:
        st.scramble()
    ctx.restore(J.ALL_GROUPS, J.HOST)
    torch.cuda.synchronize()
    for g, st in zip(gs, sts):
        for i, t in enumerate(g.tensors):
            assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 8 + g.group, g.group))
        assert ctx.verify(g.group, blob) == 2**64 - 1
    ctx.close()


def test_half_step_detected(J):
    """A half-applied optimizer step (U_v on tensors [0, split)) changes exactly
    the chunks the oracle predicts, and the replica class splits."""
    g = W.scaled(W.c1(), 20000).groups[0]
    C = 4096
    a, b = _state(g, 3), _state(g, 3)
    ctxa, ctxb = _ctx(J, C, rank=0, world=2), _ctx(J, C, rank=1, world=2)
    ctxa.register(0, J.REQUIRED, [0, 1], a.table(), keepalive=a)
    ctxb.register(0, J.REQUIRED, [0, 1], b.table(), keepalive=b)
    split = 40
    for i in range(split):
        t = g.tensors[i]
        J.inject_update(b.ptrs[i], 0, t.numel, t.gen_id, 4)
    torch.cuda.synchronize()
    ra, rb = _records(ctxa.fingerprint())[0], _records(ctxb.fingerprint())[0]
    lay = O.layout_of_group(g, C)
    touched = set()
    for i in range(split):
        touched |= set(range(lay.offsets[i] // C, (lay.offsets[i] + lay.nbytes[i] - 1) // C + 1))
    assert set(np.nonzero(ra.d != rb.d)[0].tolist()) == touched
    st, sel = J.select_consistent_replica(ctxa.fingerprint() + ctxb.fingerprint(), [0, 1])
    assert st == J.ECONFLICT


# ------------------------------------------------------------------ full size (every chunk)
BENCH_STAGING, BENCH_SLOT = 16 << 30, 8 << 30     # bench.py's launch configuration (--staging / --slot)


@pytest.mark.slow
@pytest.mark.parametrize("cfg", ["C2", "C3"])
def test_full_size_every_chunk(J, shm, cfg):
    """C2 (GPT-2 1.5B, 24.9 GB) and C3 (Llama-3-8B, 128.5 GB, the BASELINE
    target shape) in the launch configuration bench.py times (1 MiB chunks,
    8 GiB rounds, 16 GiB staging), checked over the WHOLE state:
      * every chunk of the committed /dev/shm image equals the oracle's O2
        image (regenerated block by block on all host cores), so a wrong
        image offset in the host-built segment table cannot hide;
      * every one of the n_c K1 digests in this rank's record equals O3 of
        the oracle's image, and the record's root equals the oracle's root;
      * after capture -> scramble -> HOST restore, jitc_verify passes and every
        byte of every restored tensor equals the committed image (which was
        just shown equal to the oracle's)."""
    from oracle import stream as S
    w = W.CONFIGS[cfg]()
    C = 1 << 20
    states = {g.group: _state(g, w.seed) for g in w.groups}
    ctx = J.Context(device=0, chunk_bytes=C, image_dir=shm, flags=J.F_TIME_KERNELS, staging_bytes=BENCH_STAGING,
                    slot_bytes=BENCH_SLOT)
    for g in w.groups:
        ctx.register(g.group, g.policy, [0], states[g.group].table(), keepalive=states[g.group])
        ctx.mark(g.group, 100, J.CLEAN)
    blob, sel, cap = _pipeline(J, ctx)
    recs = _records(blob)
    imgs = {}
    for g in w.groups:
        lay = O.layout_of_group(g, C)
        imgs[g.group] = (lay, np.memmap(f"{shm}/g{g.group}.img", dtype=np.uint8, mode="r"))
        r = S.check_image(g, w.seed, lay, imgs[g.group][1], recs[g.group].d)
        print(f"{cfg} group {g.group}: {lay.n_c} chunks, {lay.L / 1e9:.2f} GB checked in {r.seconds:.1f} s "
              f"on {r.threads} threads")
        assert r.bad_bytes == [], f"image chunks differing from the oracle: {r.bad_bytes[:20]}"
        assert r.bad_digests == [], f"K1 digests differing from the oracle: {r.bad_digests[:20]}"
        assert recs[g.group].root == r.root and recs[g.group].n_c == lay.n_c
        states[g.group].scramble()
    ctx.restore(J.ALL_GROUPS, J.HOST)
    for g in w.groups:
        ctx.verify(g.group, blob)
    torch.cuda.synchronize()
    for g in w.groups:
        lay, img = imgs[g.group]
        st = states[g.group]
        for i, t in enumerate(g.tensors):
            off, n = lay.offsets[i], t.nbytes
            for a in range(0, n, 1 << 30):
                b = min(a + (1 << 30), n)
                want = torch.from_numpy(np.asarray(img[off + a:off + b])).cuda()
                assert torch.equal(st.tensor_bytes(i)[a:b], want), (t.name, a)
    ctx.close()
    del states
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ edge cases
def test_edge_empty_tensors_empty_group_max_chunk(J, shm):
    """Zero-byte tensors inside a table, a group with no tensors at all (L = 0,
    n_c = 0), 1-byte tensors, and the maximum chunk size (64 MiB) -- capture,
    restore and verify must all work and stay bit-exact."""
    g = W.random_table(21, 30, max_bytes=3000, group=1)
    for i in (0, 7, 29):                           # zero-byte tensors, incl. first and last
        g.tensors[i].numel = 0
    g.tensors[3].dtype, g.tensors[3].numel = "u8", 1
    empty = W.GroupSpec(2, J.REQUIRED, [0], [])
    for C in (4096, 64 << 20):
        d = f"{shm}-{C}"
        st = _state(g, 4)
        ste = _state(empty, 4)
        ctx = _ctx(J, C, image_dir=d, staging=2 * C * 2, slot=C)
        lh, L = ctx.register(1, J.REQUIRED, [0], st.table(), keepalive=st)
        lh0, L0 = ctx.register(2, J.REQUIRED, [0], ste.table(), keepalive=ste)
        lay = O.layout_of_group(g, C)
        assert (lh, L) == (lay.layout_hash, lay.L) and L0 == 0
        assert lh0 == O.layout_of_group(empty, C).layout_hash
        blob, sel, cap = _pipeline(J, ctx)
        recs = _records(blob)
        assert recs[2].n_c == 0 and recs[2].root == O.root(lh0, np.zeros(0, dtype=np.uint64))
        assert np.array_equal(recs[1].d, O.jf64(O.pack(O.gen_group(g, 4), lay), C, 0, lay.n_c))
        st.scramble()
        ctx.restore(J.ALL_GROUPS, J.HOST)
        ctx.verify(1)
        ctx.verify(2)
        torch.cuda.synchronize()
        for i, t in enumerate(g.tensors):
            assert np.array_equal(st.tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, 4, 1)), t.name
        ctx.close()
        shutil.rmtree(d, ignore_errors=True)


@pytest.mark.slow
def test_edge_tensors_over_4gib(J, shm):
    """Maximum sizes: two tensors larger than 4 GiB (a u8 one of 4 GiB + 5 B
    at a 2-byte-misaligned address, an fp32 one of 4 GiB + 12 B -- the size
    class of an unsharded 70B-model embedding in fp32), so every 32-bit
    element, byte and segment count would wrap.  1 MiB chunks, 1 GiB rounds.
    Sampled chunks around each 4 GiB boundary, the tails and the first chunk
    equal the oracle's image bytes and digests; the restore is bit-exact on
    the same samples and verify passes over the whole group."""
    big = 1 << 32
    g = W.GroupSpec(3, J.REQUIRED, [0], [
        W.TensorSpec("head", "f32", 1000, "master", 0),
        W.TensorSpec("emb.u8", "u8", big + 5, "bytes", 1),
        W.TensorSpec("emb.f32", "f32", (big + 12) // 4, "master", 2),
        W.TensorSpec("tail", "bf16", 777, "master", 3),
    ])
    C = 1 << 20
    st = _state(g, 9, misalign=2)
    assert st.ptrs[1] % 16 == 2
    ctx = _ctx(J, C, image_dir=shm, staging=2 << 30, slot=1 << 30)
    lh, L = ctx.register(3, J.REQUIRED, [0], st.table(), keepalive=st)
    lay = O.layout_of_group(g, C)
    assert (lh, L) == (lay.layout_hash, lay.L) and L > 2 * big
    blob, sel, cap = _pipeline(J, ctx)
    rec = _records(blob)[3]
    marks = [0, lay.L - 1]
    for i in (1, 2):
        marks += [lay.offsets[i], lay.offsets[i] + big - 1, lay.offsets[i] + big, lay.offsets[i] + g.tensors[i].nbytes - 1]
    chunks = sorted({m // C for m in marks} | {m // C + 1 for m in marks if m // C + 1 < lay.n_c})
    img = np.memmap(f"{shm}/g3.img", dtype=np.uint8, mode="r")
    want = {}
    for c in chunks:
        a, b = c * C, min((c + 1) * C, lay.L)
        want[c] = O.image_range(g, 9, lay, a, b)
        assert np.array_equal(np.asarray(img[a:b]), want[c]), c
        assert int(rec.d[c]) == int(O.jf64(want[c], C, a, lay.n_c)[c]), c
    st.scramble()
    ctx.restore(3, J.HOST)
    ctx.verify(3, blob)
    torch.cuda.synchronize()
    for c in chunks:
        a, b = c * C, min((c + 1) * C, lay.L)
        for i, t in enumerate(g.tensors):
            lo, hi = max(a, lay.offsets[i]), min(b, lay.offsets[i] + t.nbytes)
            if lo < hi:
                got = st.tensor_bytes(i)[lo - lay.offsets[i]:hi - lay.offsets[i]].cpu().numpy()
                assert np.array_equal(got, want[c][lo - a:hi - a]), (c, t.name)
    ctx.close()
    del st
    torch.cuda.empty_cache()


def test_layout_mismatch_between_replicas(J):
    """S10 with real fingerprints: one replica registered one tensor with a
    different size -> ELAYOUT for the whole selection."""
    import copy
    g = W.random_table(8, 12)
    g2 = copy.deepcopy(g)
    g2.tensors[5].numel += 1
    a, b = _state(g, 1), _state(g2, 1)
    ca, cb = _ctx(J, 4096, rank=0, world=2), _ctx(J, 4096, rank=1, world=2)
    ca.register(0, J.REQUIRED, [0, 1], a.table(), keepalive=a)
    cb.register(0, J.REQUIRED, [0, 1], b.table(), keepalive=b)
    st, sel = J.select_consistent_replica(ca.fingerprint() + cb.fingerprint(), [0, 1])
    assert st == J.ELAYOUT
