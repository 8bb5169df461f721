"""Pins for the oracle's layout (O1), pack/unpack (O2/O8), shard rule (O5) and
generator (O9)."""
import numpy as np
import pytest
import torch

from oracle import oracle as O
from workloads import configs as W


def _tables():
    for seed in range(6):
        yield W.random_table(seed, 40)


def test_layout_alignment_padding_and_roundtrip():
    for g in _tables():
        lay = O.layout_of_group(g, 4096)
        ts = O.gen_group(g, 99)
        # offsets 256-aligned, non-overlapping, in registration order; L multiple of 256
        for i, (off, nb) in enumerate(zip(lay.offsets, lay.nbytes)):
            assert off % 256 == 0
            if i + 1 < len(lay.offsets):
                assert off + nb <= lay.offsets[i + 1] < off + nb + 256
        assert lay.L % 256 == 0 and lay.L >= sum(lay.nbytes)
        img = O.pack(ts, lay)
        # padding bytes are zero
        mask = np.ones(lay.L, dtype=bool)
        for off, nb in zip(lay.offsets, lay.nbytes):
            mask[off:off + nb] = False
        assert not img[mask].any()
        back = O.unpack(img, lay)
        for a, b in zip(ts, back):
            assert np.array_equal(a, b)


def test_layout_hash_sensitivity():
    g = W.random_table(1, 10)
    base = O.layout_of_group(g, 4096).layout_hash
    import copy
    for mut in range(4):
        g2 = copy.deepcopy(g)
        if mut == 0:
            g2.tensors[3].name += "x"
        elif mut == 1:
            g2.tensors[3].numel += 1
        elif mut == 2:
            g2.tensors[3].dtype = "f32" if g2.tensors[3].dtype != "f32" else "u8"
        else:
            g2.tensors[2], g2.tensors[3] = g2.tensors[3], g2.tensors[2]
        assert O.layout_of_group(g2, 4096).layout_hash != base
    assert O.layout_of_group(g, 8192).layout_hash != base


def test_config_sizes_match_survey():
    """SURVEY.md §8(a) A1 / §8(d) d.1 image sizes and tensor counts."""
    def L(w, rank=0):
        return sum(O.layout_of_group(g, 1 << 20).L for g in w.groups_of(rank))
    assert L(W.c1()) == 48_138_240 and len(W.c1().groups[0].tensors) == 156
    assert L(W.c2()) == 24_921_865_984 and sum(len(g.tensors) for g in W.c2().groups) == 2900
    assert L(W.c3()) == 128_484_179_968 and sum(len(g.tensors) for g in W.c3().groups) == 1455
    c5 = W.c5()
    assert O.layout_of_group(c5.groups[0], 1 << 20).L + O.layout_of_group(c5.groups[4], 1 << 20).L \
        == 117_935_570_944
    assert (L(W.c3()) + (1 << 20) - 1) // (1 << 20) == 122_533


def test_shard_exact_cover_bruteforce():
    """O5: the union of shards covers every chunk exactly once, sizes differ by <= 1."""
    for n_c in list(range(0, 300)) + [1999, 2000, 23768, 122533]:
        for k in range(1, 17):
            seen = np.zeros(n_c, dtype=np.int32)
            sizes = []
            prev_end = 0
            for s in range(k):
                c0, c1 = O.shard(n_c, k, s)
                assert c0 == prev_end and c1 >= c0
                prev_end = c1
                seen[c0:c1] += 1
                sizes.append(c1 - c0)
            assert prev_end == n_c and (seen == 1).all()
            assert max(sizes) - min(sizes) <= 1


def test_shard_bytes_clip():
    L, C = 10 * 4096 + 512, 4096
    n_c = (L + C - 1) // C
    got = [O.shard_bytes(n_c, 3, s, C, L) for s in range(3)]
    assert got[0][0] == 0 and got[-1][1] == L
    assert all(a[1] == b[0] for a, b in zip(got, got[1:]))


def test_generator_ranges_and_signs():
    w = W.c1()
    g = w.groups[0]
    for t in g.tensors[::7]:
        x = O.gen_tensor_bytes(t, w.seed, g.group, 0, min(t.numel, 5000)).view(np.uint32)
        e = (x >> 23) & 0xFF
        lo, hi, pos = t.range
        assert e.min() >= lo and e.max() <= hi
        if pos:
            assert not (x >> 31).any()
        else:
            assert (x >> 31).any() and not (x >> 31).all()
        assert len(np.unique(e)) == min(hi - lo + 1, len(np.unique(e)))


def test_generator_bf16_is_rne_of_fp32():
    """bf16 params == RNE(master): compare with torch's float32 -> bfloat16
    conversion (round-to-nearest-even), a library routine."""
    w = W.c2()
    g = w.groups[0]
    n = len(g.tensors) // 4
    for i in [0, 1, 5, 17, n - 1]:
        p, m = g.tensors[i], g.tensors[n + i]
        assert p.gen_id == m.gen_id
        k = min(p.numel, 20000)
        pb = O.gen_tensor_bytes(p, w.seed, g.group, 0, k).view(np.uint16)
        mb = O.gen_tensor_bytes(m, w.seed, g.group, 0, k).view(np.float32)
        ref = torch.from_numpy(mb.copy()).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
        assert np.array_equal(pb, ref)


def test_generator_slices_agree():
    """Element-range generation (used for sampled full-size parity) equals the
    slice of the whole-tensor generation, for every dtype incl. u8 tails."""
    g = W.random_table(11, 30, max_bytes=9000)
    for t in g.tensors:
        full = O.gen_tensor_bytes(t, 5, 0)
        eb = W.ELEM_BYTES[t.dtype]
        for e0 in [0, 1, 3, t.numel // 2]:
            cnt = max(0, min(t.numel - e0, 17))
            part = O.gen_tensor_bytes(t, 5, 0, e0, cnt)
            assert np.array_equal(part, full[e0 * eb:(e0 + cnt) * eb])


def test_image_range_matches_pack():
    g = W.random_table(12, 25)
    lay = O.layout_of_group(g, 4096)
    img = O.pack(O.gen_group(g, 77), lay)
    for a, b in [(0, lay.L), (4096, 8192), (13, 999), (lay.L - 300, lay.L)]:
        assert np.array_equal(O.image_range(g, 77, lay, a, b), img[a:b])


def test_update_changes_low_mantissa_only():
    L = O.lib()
    x = (np.arange(1000, dtype=np.uint64) * np.uint64(2654435761)).astype(np.uint32)
    y = x.copy()
    L.orc_update_fp32(O._ptr(y), 0, len(y), 3, 9)
    assert ((x ^ y) >> 16 == 0).all() and (x != y).mean() > 0.99
    z = y.copy()
    L.orc_update_fp32(O._ptr(z), 0, len(z), 3, 9)   # XOR update is an involution
    assert np.array_equal(z, x)
