"""oracle/stream.py: the block-wise, multi-threaded oracle passes used for
every-chunk parity at bench size and for the d.7 committed-image JF64 must
equal the one-shot oracle (O2 pack, O3 jf64) and must localise a difference
to the exact chunk."""
import numpy as np

from oracle import oracle as O
from oracle import stream as S
from workloads import configs as W


def _case(C=4096):
    g = W.scaled(W.c1(), 3000).groups[0]
    lay = O.layout_of_group(g, C)
    img = O.pack(O.gen_group(g, 77), lay)
    return g, lay, img


def test_jf64_image_equals_one_shot():
    g, lay, img = _case()
    want = O.jf64(img, lay.C, 0, lay.n_c)
    for threads, block in ((1, 1 << 30), (3, 3 * lay.C), (8, lay.C)):
        assert np.array_equal(S.jf64_image(img, lay.C, lay.L, threads, block), want)


def test_check_image_clean_and_root():
    g, lay, img = _case()
    d = O.jf64(img, lay.C, 0, lay.n_c)
    r = S.check_image(g, 77, lay, img, d, threads=4, block=5 * lay.C)
    assert r.bad_bytes == [] and r.bad_digests == [] and r.chunks == lay.n_c
    assert r.root == O.root(lay.layout_hash, d)


def test_check_image_localises_byte_and_digest_faults():
    g, lay, img = _case()
    d = O.jf64(img, lay.C, 0, lay.n_c)
    bad_img = img.copy()
    bad_img[7 * lay.C + 13] ^= 0x10           # one bit in chunk 7
    bad_img[lay.L - 1] ^= 0x01                # last byte (padding or data) of the last chunk
    bad_d = d.copy()
    bad_d[3] ^= np.uint64(1)
    r = S.check_image(g, 77, lay, bad_img, bad_d, threads=3, block=4 * lay.C)
    assert sorted(r.bad_bytes) == [7, lay.n_c - 1]
    assert r.bad_digests == [3]               # digests are checked against O3 of the ORACLE image
    # a wrong seed (every byte differs) is caught everywhere
    r2 = S.check_image(g, 78, lay, img, d, threads=2, block=8 * lay.C)
    assert len(r2.bad_bytes) == lay.n_c or len(r2.bad_bytes) >= lay.n_c - 1


def test_chunk_sample_pack_unpack_digests_equal_full_image():
    """The d.7 sample: packing the sampled pieces gives exactly the sampled
    chunks of the full O2 image (zero padding included), their sampled-JF64
    digests equal the full digests at those chunks, and O8 unpack returns the
    pieces.  Ragged last chunk included (L not a multiple of C)."""
    g = W.scaled(W.c2(), 2500).groups[0]
    for C, every, th in ((4096, 3, 1), (4096, 16, 4), (1 << 16, 1, 2)):
        lay = O.layout_of_group(g, C)
        full = O.pack(O.gen_group(g, 5), lay)
        dfull = O.jf64(full, C, 0, lay.n_c)
        cs = S.chunk_sample(g, 5, lay, every, threads=th)
        assert cs.chunks == list(range(0, lay.n_c, every))
        img = O.pack(cs.pieces, cs.lay, threads=th)
        for i, c in enumerate(cs.chunks):
            n = min((c + 1) * C, lay.L) - c * C
            assert np.array_equal(img[i * C:i * C + n], full[c * C:c * C + n]), (C, every, c)
        d = S.jf64_sample(img, cs, lay.n_c, threads=th)
        assert np.array_equal(d[cs.chunks], dfull[cs.chunks])
        back = O.unpack(img, cs.lay, threads=th)
        assert all(np.array_equal(a, b) for a, b in zip(back, cs.pieces))
