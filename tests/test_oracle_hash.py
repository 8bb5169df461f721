"""Pins for the oracle's hash primitives (fmix64, splitmix64, FNV-1a, fold,
JF64, root) against published vectors and mathematical invariants -- never
against a re-typed copy of the oracle's own formula."""
import os

import numpy as np
import pytest

from oracle import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")
M = (1 << 64) - 1


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return [l.rstrip("\n") for l in f if l.strip() and not l.startswith("#")]


def _rotl(x, r):
    return ((x << r) | (x >> (64 - r))) & M


def _murmur3_x64_128(key: bytes, seed: int) -> bytes:
    """MurmurHash3_x64_128 body written in the test; its finalizer is the
    ORACLE's fmix64, so the SMHasher verification value pins that function."""
    c1, c2 = 0x87C37B91114253D5, 0x4CF5AD432745937F
    h1 = h2 = seed
    n = len(key)
    nb = n // 16
    for i in range(nb):
        k1 = int.from_bytes(key[16 * i:16 * i + 8], "little")
        k2 = int.from_bytes(key[16 * i + 8:16 * i + 16], "little")
        k1 = (_rotl((k1 * c1) & M, 31) * c2) & M
        h1 ^= k1
        h1 = (_rotl(h1, 27) + h2) & M
        h1 = (h1 * 5 + 0x52DCE729) & M
        k2 = (_rotl((k2 * c2) & M, 33) * c1) & M
        h2 ^= k2
        h2 = (_rotl(h2, 31) + h1) & M
        h2 = (h2 * 5 + 0x38495AB5) & M
    tail = key[16 * nb:]
    if len(tail) > 8:
        k2 = int.from_bytes(tail[8:], "little")
        h2 ^= (_rotl((k2 * c2) & M, 33) * c1) & M
    if len(tail) > 0:
        k1 = int.from_bytes(tail[:8], "little")
        h1 ^= (_rotl((k1 * c1) & M, 31) * c2) & M
    h1 ^= n
    h2 ^= n
    h1 = (h1 + h2) & M
    h2 = (h2 + h1) & M
    h1 = O.fmix64(h1)
    h2 = O.fmix64(h2)
    h1 = (h1 + h2) & M
    h2 = (h2 + h1) & M
    return h1.to_bytes(8, "little") + h2.to_bytes(8, "little")


def test_fmix64_smhasher_verification():
    want = int(_gold("smhasher_verification.txt")[0], 16)
    hashes = b"".join(_murmur3_x64_128(bytes(range(i)), 256 - i) for i in range(256))
    got = int.from_bytes(_murmur3_x64_128(hashes, 0)[:4], "little")
    assert got == want


def _unxorshift33(x):
    return x ^ (x >> 33)     # 33 >= 32, so one application inverts x ^= x >> 33


def test_fmix64_inverse_roundtrip():
    """fmix64 is a bijection (the JF64 single-word-detection guarantee rests on
    it): undo it with the published inverse multipliers."""
    (c1, i1), (c2, i2) = [tuple(int(t, 16) for t in l.split()) for l in _gold("fmix64_inverse.txt")]
    assert (c1 * i1) & M == 1 and (c2 * i2) & M == 1
    rng = np.random.default_rng(1)
    xs = [int(v) for v in rng.integers(0, 2**63, 20000, dtype=np.int64)] + [0, 1, M, 1 << 63]
    xs += [x | (1 << 63) for x in xs[:5000]]
    for x in xs:
        y = O.fmix64(x)
        y = _unxorshift33(y)
        y = (y * i2) & M
        y = _unxorshift33(y)
        y = (y * i1) & M
        y = _unxorshift33(y)
        assert y == x
    assert O.fmix64(0) == 0


def test_splitmix64_vigna_vector():
    want = [int(v) for v in _gold("splitmix64_vigna.txt")]
    x = 1234567
    got = []
    for _ in range(5):
        got.append(O.splitmix64(x))     # output for state x is splitmix64(x) (pre-increment form)
        x = (x + O.PHI) & M
    assert got == want


def test_fnv1a64_vectors():
    for line in _gold("fnv1a64.txt"):
        inp, h = line.split("\t")
        assert O.fnv1a64(inp.encode()) == int(h, 16)


def test_fold_fmix64_unwinds_with_inverse():
    (c1, i1), (c2, i2) = [tuple(int(t, 16) for t in l.split()) for l in _gold("fmix64_inverse.txt")]

    def inv(y):
        y = _unxorshift33(y); y = (y * i2) & M; y = _unxorshift33(y); y = (y * i1) & M
        return _unxorshift33(y)
    xs = [5, 0, M, 12345678901234567, 42]
    h = O.fold_fmix64(xs)
    for x in reversed(xs):
        h = inv(h) ^ x
    assert h == 0


# ------------------------------------------------------------------- JF64
def test_jf64_closed_form_zero_terms():
    """If word g holds (g+1)*PHI every term is fmix64(0) = 0, so every chunk
    digest is 0.  Pins the key formula, the global word index (not byte index,
    not per-chunk index), and the little-endian word read."""
    C = 4096
    n_words = 5 * C // 8 + 24          # 5 chunks + a ragged 192-byte tail
    g = np.arange(n_words, dtype=np.uint64)
    words = (g + np.uint64(1)) * np.uint64(O.PHI)
    img = words.astype("<u8").view(np.uint8)
    d = O.jf64(img, C)
    assert len(d) == 6 and not d.any()
    # a fragment starting at byte 3*C gives the same (zero) digests for its chunks
    d2 = O.jf64(img[3 * C:], C, byte0=3 * C)
    assert not d2.any()
    # off by one in the key (g instead of g+1) would make them all nonzero
    img2 = (g * np.uint64(O.PHI)).astype("<u8").view(np.uint8)
    assert O.jf64(img2, C).all()


def test_jf64_single_word_special_case():
    """One-word image: d[0] = fmix64(w ^ PHI); with w = 0 this is fmix64(PHI),
    a value fixed independently by the SMHasher-pinned fmix64."""
    img = np.zeros(8, dtype=np.uint8)
    assert int(O.jf64(img, 4096)[0]) == O.fmix64(O.PHI)


def test_jf64_every_single_bit_flip_detected():
    """Brute force: all 32,768 single-bit flips of a 4 KiB state change d[c]
    (a guarantee from bijectivity)."""
    rng = np.random.default_rng(7)
    img = rng.integers(0, 256, 4096, dtype=np.uint8)
    C = 1024
    base = O.jf64(img, C)
    for byte in range(4096):
        for bit in range(8):
            img[byte] ^= 1 << bit
            d = O.jf64(img[(byte // C) * C:(byte // C + 1) * C], C, byte0=(byte // C) * C)
            img[byte] ^= 1 << bit
            assert d[byte // C] != base[byte // C]


def test_jf64_chunk_merge_linearity():
    """Digests at chunk size 4C are sums of the 4C/C sub-chunk digests: the key
    depends only on the global word index (catches per-chunk indexing)."""
    rng = np.random.default_rng(3)
    img = rng.integers(0, 256, 64 * 1024 + 256, dtype=np.uint8)
    a = O.jf64(img, 4096)
    b = O.jf64(img, 16384)
    for c in range(len(b)):
        assert int(b[c]) == int(np.sum(a[4 * c:4 * c + 4], dtype=np.uint64))


def test_jf64_position_sensitive():
    """Swapping two different words changes the digest (the key is not dropped)."""
    rng = np.random.default_rng(4)
    img = rng.integers(0, 256, 4096, dtype=np.uint8)
    w = img.view("<u8").copy()
    d0 = O.jf64(img, 4096)
    w[[3, 100]] = w[[100, 3]]
    assert O.jf64(w.view(np.uint8), 4096)[0] != d0[0]


def test_jf64_random_multiword_corruptions():
    rng = np.random.default_rng(5)
    img = rng.integers(0, 256, 8192, dtype=np.uint8)
    d0 = O.jf64(img, 8192)[0]
    for _ in range(2000):
        x = img.copy()
        idx = rng.integers(0, 8192, rng.integers(2, 20))
        x[idx] ^= rng.integers(1, 256, len(idx), dtype=np.uint8)
        assert O.jf64(x, 8192)[0] != d0


def test_root_chain():
    rng = np.random.default_rng(6)
    d = rng.integers(0, 2**63, 50, dtype=np.int64).astype(np.uint64)
    r = O.root(0x1234, d)
    # n_c = 0: root = fmix64(layout_hash ^ 0)
    assert O.root(0x1234, np.zeros(0, dtype=np.uint64)) == O.fmix64(0x1234)
    # one element: fmix64(fmix64(lh ^ 1) ^ d0)
    assert O.root(7, d[:1]) == O.fmix64(O.fmix64(7 ^ 1) ^ int(d[0]))
    # any single change or transposition changes the root
    for i in range(50):
        e = d.copy(); e[i] ^= np.uint64(1)
        assert O.root(0x1234, e) != r
    e = d.copy(); e[[1, 2]] = e[[2, 1]]
    assert O.root(0x1234, e) != r


def test_oracle_threads_agree():
    """digests (and pack/unpack) are identical with 1 or
    N oracle threads -- each thread owns whole chunks / whole tensors."""
    from workloads import configs as W
    g = W.random_table(77, 300, max_bytes=9000)
    for C in (4096, 1 << 16):
        lay = O.layout_of_group(g, C)
        ts = O.gen_group(g, 3)
        img1 = O.pack(ts, lay)
        for th in (2, 3, 8, 1000):
            assert np.array_equal(O.pack(ts, lay, threads=th), img1)
            for a, b in ((0, lay.L), (8 * 37, lay.L - 8 * 5), (C + 8, 3 * C + 16)):
                assert np.array_equal(O.jf64(img1[a:b], C, a, lay.n_c, threads=th),
                                      O.jf64(img1[a:b], C, a, lay.n_c)), (th, a, b)
            for x, y in zip(O.unpack(img1, lay, threads=th), ts):
                assert np.array_equal(x, y.view(np.uint8).reshape(-1))
