"""Oracle passes over a whole full-size image, block by block on all host
cores -- TEST INFRASTRUCTURE ONLY (tests/, bench.py's cpu_baseline leg).

Nothing here adds arithmetic: every byte and digest comes from the oracle's
own O2 (image_range: the generator O9 placed by the layout O1) and O3 (jf64)
routines, called on disjoint chunk-aligned blocks.  JF64 digests are per
chunk and blocks never split a chunk, so the block-wise result equals the
single-pass one (tests/test_oracle_hash.py pins chunk-merge linearity and
1-vs-N-thread equality).

Used for
  * every-chunk parity at bench size (VERDICT r01 "what's weak" #1): the
    committed /dev/shm image of C2 / C3 against O2, and the GPU's K1
    digests against O3 of O2, chunk by chunk over the whole image;
  * JF64 over the committed image (the bytes the GPU
    digested), which doubles as a bit-exact check of the manifest digests.
"""
from __future__ import annotations

import bisect
import os
import time
from concurrent.futures import ThreadPoolExecutor
from dataclasses import dataclass, field
from typing import List, Optional

import numpy as np

from . import oracle as O


def host_threads() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def _blocks(L: int, C: int, block: int):
    """[0, L) cut into chunk-aligned blocks of about `block` bytes."""
    step = max(C, block // C * C)
    return [(a, min(a + step, L)) for a in range(0, L, step)]


def _diff_chunks(x: np.ndarray, y: np.ndarray, a: int, C: int) -> List[int]:
    """Global chunk ids (block starting at image byte a) where x and y differ."""
    out = []
    for o in range(0, len(x), C):
        if not np.array_equal(x[o:o + C], y[o:o + C]):
            out.append((a + o) // C)
    return out


@dataclass
class ImageCheck:
    bytes_checked: int = 0
    chunks: int = 0
    bad_bytes: List[int] = field(default_factory=list)     # chunks whose image bytes differ from O2
    bad_digests: List[int] = field(default_factory=list)   # chunks whose digest differs from O3(O2)
    root: int = 0                                          # O3 root of the oracle's image
    seconds: float = 0.0
    threads: int = 1


def check_image(g, seed: int, lay: "O.Layout", img: np.ndarray, digests: Optional[np.ndarray],
                threads: int = 0, block: int = 64 << 20) -> ImageCheck:
    """Every chunk of a group's image: the image bytes `img[0:L]` against the
    oracle's O2 image (generated block by block with image_range), and, when
    given, `digests[c]` against O3 of the oracle's image.  Returns the lists of
    differing chunks (empty == bit-exact) and the oracle's root."""
    threads = threads or host_threads()
    C, L, n_c = lay.C, lay.L, lay.n_c
    d_all = np.zeros(n_c, dtype=np.uint64)
    res = ImageCheck(bytes_checked=L, chunks=n_c, threads=threads)
    t0 = time.perf_counter()

    def run(ab):
        a, b = ab
        want = O.image_range(g, seed, lay, a, b)
        got = np.asarray(img[a:b])
        bad = [] if np.array_equal(got, want) else _diff_chunks(got, want, a, C)
        d = O.jf64(want, C, a, n_c)
        c0, c1 = a // C, (b + C - 1) // C
        d_all[c0:c1] = d[c0:c1]          # disjoint chunk ranges per block
        bad_d = []
        if digests is not None:
            bad_d = [int(c0 + i) for i in np.nonzero(d[c0:c1] != digests[c0:c1])[0]]
        return bad, bad_d

    with ThreadPoolExecutor(threads) as ex:
        for bad, bad_d in ex.map(run, _blocks(L, C, block)):
            res.bad_bytes += bad
            res.bad_digests += bad_d
    res.root = O.root(lay.layout_hash, d_all)
    res.seconds = time.perf_counter() - t0
    return res


def jf64_image(img: np.ndarray, C: int, L: int, threads: int = 0, block: int = 256 << 20) -> np.ndarray:
    """O3 digests d[0..n_c) of image bytes img[0:L] (e.g. the committed
    /dev/shm image), block by block on `threads` host threads."""
    threads = threads or host_threads()
    n_c = (L + C - 1) // C
    d_all = np.zeros(n_c, dtype=np.uint64)

    def run(ab):
        a, b = ab
        d = O.jf64(np.asarray(img[a:b]), C, a, n_c)
        c0, c1 = a // C, (b + C - 1) // C
        d_all[c0:c1] = d[c0:c1]

    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(run, _blocks(L, C, block)))
    return d_all


# ----------------------------------------------------------------------------
# Evenly spaced chunk samples ("pack/unpack run on 1/16
# of the chunks, evenly spaced, extrapolated and labelled sampled")
# ----------------------------------------------------------------------------
@dataclass
class ChunkSample:
    """Chunks c = 0, every, 2*every, ... of one group's image.  Sample chunk i
    (global chunk chunks[i]) sits at sample offset i*C; `lay` is the O1-style
    layout of the sample (one entry per tensor piece that falls in a sampled
    chunk), so O2 pack / O8 unpack run on it unchanged; `pieces` holds the
    pieces' bytes from the O9 generator (state generation is not timed)."""
    group: int
    every: int
    chunks: List[int]
    lens: List[int]                 # data bytes of each sampled chunk (the last chunk may be short)
    lay: "O.Layout"
    pieces: List[np.ndarray]

    @property
    def nbytes(self) -> int:
        return sum(self.lens)


def chunk_sample(g, seed: int, lay: "O.Layout", every: int, threads: int = 0) -> ChunkSample:
    from workloads.configs import ELEM_BYTES
    C = lay.C
    chunks = list(range(0, lay.n_c, max(1, every)))
    spans = []                       # (sample offset, tensor, image lo, image hi)
    for i, c in enumerate(chunks):
        a, b = c * C, min((c + 1) * C, lay.L)
        # tensors overlapping [a, b): offsets are sorted
        k = max(0, bisect.bisect_right(lay.offsets, a) - 1)
        while k < len(g.tensors) and lay.offsets[k] < b:
            t, off = g.tensors[k], lay.offsets[k]
            lo, hi = max(a, off), min(b, off + t.nbytes)
            if lo < hi:
                spans.append((i * C + (lo - a), k, lo, hi))
            k += 1

    def gen(sp):
        so, k, lo, hi = sp
        t, off = g.tensors[k], lay.offsets[k]
        eb = ELEM_BYTES[t.dtype]
        e0, e1 = (lo - off) // eb, (hi - off + eb - 1) // eb
        raw = O.gen_tensor_bytes(t, seed, g.group, e0, e1 - e0)
        s = (lo - off) - e0 * eb
        return np.ascontiguousarray(raw[s:s + (hi - lo)])

    with ThreadPoolExecutor(threads or host_threads()) as ex:
        pieces = list(ex.map(gen, spans))
    sub = O.Layout([f"s{j}" for j in range(len(spans))], [hi - lo for (_, _, lo, hi) in spans],
                   [0] * len(spans), [so for (so, _, _, _) in spans], len(chunks) * C, C, 0)
    lens = [min((c + 1) * C, lay.L) - c * C for c in chunks]
    return ChunkSample(g.group, every, chunks, lens, sub, pieces)


def jf64_sample(img: np.ndarray, cs: ChunkSample, n_c: int, threads: int = 1) -> np.ndarray:
    """O3 digests of the sampled chunks of a sample image (chunk i at offset
    i*C), keyed by their GLOBAL word indices; returns d[0..n_c) with only the
    sampled chunks filled."""
    C = cs.lay.C
    d = np.zeros(n_c, dtype=np.uint64)
    L = O.lib()
    base = O._ptr(img)

    def run(ab):
        for i in range(*ab):
            c, n = cs.chunks[i], cs.lens[i]
            L.orc_jf64_accumulate(base + i * C, c * C // 8, n // 8, C // 8, O._ptr(d))

    parts = O._parts(len(cs.chunks), threads)
    if len(parts) == 1:
        run(parts[0])
    else:
        with ThreadPoolExecutor(len(parts)) as ex:
            list(ex.map(run, parts))
    return d
