"""Whole-path oracle invariants (BASELINE.json north_star):
restore(capture(S)) == S bitwise, the union of shards covers every byte once,
identical replicas give equal digests, a flip in the committed image is caught
at the exact chunk, and an uncommitted checkpoint is refused (PAPER.md:136,
:140)."""
import numpy as np

from oracle import oracle as O
from workloads import configs as W


def _c1_small():
    return W.scaled(W.c1(), 3000)


def test_identical_replicas_equal_digests_and_roundtrip():
    w = _c1_small()
    g = w.groups[0]
    lay = O.layout_of_group(g, 4096)
    imgs, ds = {}, {}
    for r in range(2):               # two DP replicas generated from the same seed
        imgs[r] = O.pack(O.gen_group(g, w.seed), lay)
        ds[r] = O.jf64(imgs[r], lay.C, 0, lay.n_c)
    assert np.array_equal(ds[0], ds[1])
    for k in (1, 2):
        gs = O.GroupSel(0, O.REQUIRED, writers=list(range(k)))
        st, host, man, com = O.capture_sim(gs, 3, lay, imgs, ds)
        assert st == O.OK and np.array_equal(host, imgs[0])
        st, bad, ts = O.restore_sim(host, man, com)
        assert st == O.OK
        for a, b in zip(ts, O.gen_group(g, w.seed)):
            assert np.array_equal(a, b)


def test_corrupt_image_exact_chunk():
    w = _c1_small()
    g = w.groups[0]
    lay = O.layout_of_group(g, 4096)
    img = O.pack(O.gen_group(g, w.seed), lay)
    d = O.jf64(img, lay.C, 0, lay.n_c)
    gs = O.GroupSel(0, O.REQUIRED, writers=[0])
    st, host, man, com = O.capture_sim(gs, 3, lay, {0: img}, {0: d})
    rng = np.random.default_rng(0)
    for _ in range(20):
        pos = int(rng.integers(0, lay.L))
        h = host.copy(); h[pos] ^= 1 << int(rng.integers(0, 8))
        st, bad, _ = O.restore_sim(h, man, com)
        assert st == O.ECORRUPT and bad == pos // lay.C


def test_uncommitted_refused():
    w = _c1_small()
    g = w.groups[0]
    lay = O.layout_of_group(g, 4096)
    img = O.pack(O.gen_group(g, w.seed), lay)
    d = O.jf64(img, lay.C, 0, lay.n_c)
    gs = O.GroupSel(0, O.REQUIRED, writers=[0])
    _, host, man, com = O.capture_sim(gs, 3, lay, {0: img}, {0: d})
    assert O.restore_sim(host, man, None)[0] == O.EINCOMPLETE
    assert O.restore_sim(host, None, com)[0] == O.EINCOMPLETE
    bad = bytearray(man); bad[100] ^= 1            # a torn / altered manifest
    assert O.restore_sim(host, bytes(bad), com)[0] == O.EINCOMPLETE


def test_half_step_detected():
    """A half-applied optimizer step (U_v on tensors [0, split)) changes the
    digests of exactly the chunks those tensors touch -- at
    every split point, built incrementally: split s+1
    is split s plus the update of tensor s."""
    w = _c1_small()
    g = w.groups[0]
    lay = O.layout_of_group(g, 4096)
    ts = O.gen_group(g, w.seed)
    d0 = O.jf64(O.pack(ts, lay), lay.C, 0, lay.n_c)
    L = O.lib()
    t2 = [t.copy() for t in ts]
    touched = set()
    n_split = 0
    for split in range(1, len(ts) + 1):
        i = split - 1
        if g.tensors[i].dtype == "f32":
            x = t2[i].view(np.uint32)
            L.orc_update_fp32(O._ptr(x), 0, len(x), g.tensors[i].gen_id, 4)
            touched |= set(range(lay.offsets[i] // lay.C, (lay.offsets[i] + lay.nbytes[i] - 1) // lay.C + 1))
        if split == len(ts):
            break                       # the whole step applied: not a half step
        d1 = O.jf64(O.pack(t2, lay), lay.C, 0, lay.n_c)
        changed = set(np.nonzero(d0 != d1)[0].tolist())
        assert changed == touched, split
        assert (O.root(lay.layout_hash, d0) != O.root(lay.layout_hash, d1)) == bool(touched), split
        n_split += 1
    assert n_split == len(ts) - 1


def test_manifest_roundtrip_aux_and_every_byte_covered():
    """O4b + the aux section (PAPER.md:132 CPU state carried
    opaque; PAPER.md:136 metadata last): decode(encode(x)) == x, the shard
    table is O5's, and changing ANY single byte of the manifest body is caught
    by the trailer (fold_fmix64 is a chain of bijections over LE words, so a
    change confined to one word always changes it) -> EINCOMPLETE."""
    g = W.random_table(5, 7, max_bytes=3000)
    lay = O.layout_of_group(g, 4096)
    img = O.pack(O.gen_group(g, 2), lay)
    d = O.jf64(img, lay.C, 0, lay.n_c)
    gs = O.GroupSel(0, O.REQUIRED, writers=[1, 4, 6])
    for aux in (b"", b"x", b"iteration=17;rng=" + bytes(range(40))):
        man = O.encode_manifest(gs, 9, lay, d, aux)
        assert len(man) % 8 == 0
        m = O.decode_manifest(man)
        assert m["aux"] == aux and m["writers"] == [1, 4, 6] and m["v_star"] == 9
        assert np.array_equal(m["d"], d) and m["root"] == O.root(lay.layout_hash, d)
        assert m["shards"] == [(w, *O.shard(lay.n_c, 3, s)) for s, w in enumerate([1, 4, 6])]
        assert m["layout"].offsets == lay.offsets and m["layout"].names == lay.names
        com = O.commit_record(0, 9, man)
        assert O.restore_sim(img, man, com)[0] == O.OK
    for pos in range(len(man) - 8):
        bad = bytearray(man)
        bad[pos] ^= 0x5A
        assert O.restore_sim(img, bytes(bad), com)[0] == O.EINCOMPLETE, pos
