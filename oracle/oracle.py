"""CPU oracle for the JIT-checkpointing data path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and
`--impl reference`) may import this module.  It shares no code with the CUDA
path (paper_conf_eurosys_guptakkvgkrs24_b200/, include/): the byte and hash
arithmetic lives in oracle/jitc_oracle.c, the decision procedures below are
written step by step from the paper and SURVEY.md §8(c) (O1..O10).

Each function names the passage it follows.  "Reading Rn" refers to the table
of readings in DESIGN.md (where PAPER.md is silent or ambiguous).

Parity status: every function here is pinned by a `-m "not gpu"` test
(tests/test_oracle_*.py) against something other than itself -- published
vectors (SMHasher, Vigna's splitmix64, FNV), bijectivity, brute force, or the
selection truth table S1..S11 written from PAPER.md:140-188.  No stored value
comes from the CUDA path.
"""
from __future__ import annotations

import ctypes
import os
import struct
import subprocess
from dataclasses import dataclass, field
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
MASK = (1 << 64) - 1
PHI = 0x9E3779B97F4A7C15
ALIGN = 256                                   # reading R4

# status codes (include/jitc.h mirrors these names; values are the contract)
OK, EINVAL, ESTATE, ENOMEM, ECUDA, ENCCL = 0, -1, -2, -3, -4, -5
ELAYOUT, ENOREPLICA, ECONFLICT, ENOCONSISTENT = -6, -7, -8, -9
EUNSTABLE, ECORRUPT, EINCOMPLETE, EIO = -10, -11, -12, -13
CLEAN, DIRTY = 0, 1
REQUIRED, OPTIONAL = 0, 1
# per-group selection status
G_OK, G_UNVERIFIED_SINGLE, G_NOREPLICA, G_DROPPED, G_CONFLICT, G_NOCANDIDATE = 0, 1, 2, 3, 4, 5
# exclusion reasons (O6 step 10)
R_DIRTY, R_STALE_VERSION, R_MINORITY = 1, 2, 3


# ----------------------------------------------------------------------------
# C part
# ----------------------------------------------------------------------------
def build(force: bool = False) -> str:
    """Compile oracle/jitc_oracle.c with plain gcc -O2 (no vector intrinsics)."""
    src = os.path.join(_HERE, "jitc_oracle.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-shared", "-fPIC", "-o", _SO, src])
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        u64, u32, vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        L.orc_fmix64.restype = u64; L.orc_fmix64.argtypes = [u64]
        L.orc_splitmix64.restype = u64; L.orc_splitmix64.argtypes = [u64]
        L.orc_jf64_term.restype = u64; L.orc_jf64_term.argtypes = [u64, u64]
        L.orc_jf64_accumulate.restype = None
        L.orc_jf64_accumulate.argtypes = [vp, u64, u64, u64, vp]
        L.orc_root.restype = u64; L.orc_root.argtypes = [u64, vp, u64]
        L.orc_fold_fmix64.restype = u64; L.orc_fold_fmix64.argtypes = [vp, u64]
        L.orc_pack.restype = None; L.orc_pack.argtypes = [vp, vp, vp, u64, vp, u64]
        L.orc_unpack.restype = None; L.orc_unpack.argtypes = [vp, vp, vp, vp, u64]
        for f in (L.orc_gen_fp32, L.orc_gen_bf16):
            f.restype = None
            f.argtypes = [vp, u64, u64, u64, u32, u32, u32, u32, ctypes.c_int]
        L.orc_update_fp32.restype = None; L.orc_update_fp32.argtypes = [vp, u64, u64, u32, u64]
        L.orc_rne_bf16.restype = None; L.orc_rne_bf16.argtypes = [vp, vp, u64]
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def fmix64(x: int) -> int:
    return lib().orc_fmix64(x & MASK)


def splitmix64(z: int) -> int:
    return lib().orc_splitmix64(z & MASK)


def fold_fmix64(xs: Sequence[int]) -> int:
    """O1: h = 0; for x in xs: h = fmix64(h ^ x)."""
    a = np.array([x & MASK for x in xs], dtype=np.uint64)
    return lib().orc_fold_fmix64(_ptr(a), len(a))


def fnv1a64(data: bytes) -> int:
    """FNV-1a 64-bit (Fowler/Noll/Vo): offset 0xcbf29ce484222325, prime 0x100000001b3."""
    h = 0xCBF29CE484222325
    for b in data:
        h ^= b
        h = (h * 0x100000001B3) & MASK
    return h


# ----------------------------------------------------------------------------
# O1 layout  (image order / alignment: reading R4; tensor identity: R5)
# ----------------------------------------------------------------------------
@dataclass
class Layout:
    names: List[str]
    nbytes: List[int]
    dtypes: List[int]
    offsets: List[int]
    L: int
    C: int
    layout_hash: int

    @property
    def n_c(self) -> int:
        return (self.L + self.C - 1) // self.C


def align_up(x: int, a: int = ALIGN) -> int:
    return (x + a - 1) // a * a


def layout(names: Sequence[str], nbytes: Sequence[int], dtypes: Sequence[int], C: int) -> Layout:
    """off[0] = 0; off[i+1] = align_up(off[i] + nbytes[i], 256); L = off[n].
    layout_hash = fold_fmix64([n, C, for each tensor: fnv1a64(name), nbytes, dtype])."""
    offs, off = [], 0
    for nb in nbytes:
        offs.append(off)
        off = align_up(off + nb)
    xs = [len(names), C]
    for nm, nb, dt in zip(names, nbytes, dtypes):
        xs += [fnv1a64(nm.encode()), nb, dt]
    return Layout(list(names), list(nbytes), list(dtypes), offs, off, C, fold_fmix64(xs))


def layout_of_group(g, C: int) -> Layout:
    from workloads.configs import DTYPE_CODE
    return layout([t.name for t in g.tensors], [t.nbytes for t in g.tensors],
                  [DTYPE_CODE[t.dtype] for t in g.tensors], C)


# ----------------------------------------------------------------------------
# O9 generator (host side; the K4 kernel implements the same formula itself)
# ----------------------------------------------------------------------------
def gen_tensor_bytes(t, seed: int, group: int, e0: int = 0, count: Optional[int] = None) -> np.ndarray:
    """Elements [e0, e0+count) of tensor spec t as raw little-endian bytes."""
    L = lib()
    if count is None:
        count = t.numel - e0
    lo, hi, pos = t.range
    if t.dtype == "f32":
        out = np.empty(count, dtype=np.uint32)
        L.orc_gen_fp32(_ptr(out), e0, count, seed, group, t.gen_id, lo, hi, int(pos))
        return out.view(np.uint8)
    if t.dtype == "bf16":
        out = np.empty(count, dtype=np.uint16)
        L.orc_gen_bf16(_ptr(out), e0, count, seed, group, t.gen_id, lo, hi, int(pos))
        return out.view(np.uint8)
    if t.dtype == "u8":      # byte b = byte (b % 4) of fp32 word (b // 4), little-endian
        w0, w1 = e0 // 4, (e0 + count + 3) // 4
        words = np.empty(max(w1 - w0, 0), dtype=np.uint32)
        L.orc_gen_fp32(_ptr(words), w0, w1 - w0, seed, group, t.gen_id, lo, hi, int(pos))
        b = words.view(np.uint8)
        return b[e0 - 4 * w0: e0 - 4 * w0 + count].copy()
    if t.dtype == "zeros":
        return np.zeros(count, dtype=np.uint8)
    if t.dtype == "ones":
        return np.full(count, 0xFF, dtype=np.uint8)
    raise ValueError(t.dtype)


def gen_group(g, seed: int) -> List[np.ndarray]:
    return [gen_tensor_bytes(t, seed, g.group) for t in g.tensors]


def image_range(g, seed: int, lay: Layout, a: int, b: int) -> np.ndarray:
    """Image bytes [a, b) of group g, generated tensor slice by tensor slice
    (used for sampled parity at full size, where the whole image is too big)."""
    out = np.zeros(b - a, dtype=np.uint8)
    from workloads.configs import ELEM_BYTES
    for t, off in zip(g.tensors, lay.offsets):
        lo, hi = max(a, off), min(b, off + t.nbytes)
        if lo >= hi:
            continue
        eb = ELEM_BYTES[t.dtype]
        e0, e1 = (lo - off) // eb, (hi - off + eb - 1) // eb
        raw = gen_tensor_bytes(t, seed, g.group, e0, e1 - e0)
        s = (lo - off) - e0 * eb
        out[lo - a: hi - a] = raw[s: s + (hi - lo)]
    return out


# ----------------------------------------------------------------------------
# O2 pack / O8 unpack
# ----------------------------------------------------------------------------
def _parts(n: int, threads: int) -> List[Tuple[int, int]]:
    """[0, n) cut into `threads` contiguous, nearly equal parts (O5's rule)."""
    t = max(1, min(threads, n)) if n else 1
    return [(s * n // t, (s + 1) * n // t) for s in range(t)]


def _run_parts(fn, parts):
    """Runs fn(a, b) for every part; with more than one part, on threads
    (ctypes releases the GIL inside the C calls).  The parts touch disjoint
    bytes, so the result is the single-threaded one."""
    if len(parts) == 1:
        fn(*parts[0])
        return
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(len(parts)) as ex:
        list(ex.map(lambda ab: fn(*ab), parts))


def pack(tensors: Sequence[np.ndarray], lay: Layout, threads: int = 1) -> np.ndarray:
    """O2.  threads > 1 (oracle timing): tensors are cut
    into contiguous runs and each run is packed into its own image span
    [off[first], off[last+1]) -- the spans partition [0, L)."""
    img = np.empty(lay.L, dtype=np.uint8)
    ts = [np.ascontiguousarray(t) for t in tensors]
    src = (ctypes.c_void_p * max(1, len(ts)))(*[_ptr(t) for t in ts])
    nb = np.array(lay.nbytes, dtype=np.uint64)
    off = np.array(lay.offsets, dtype=np.uint64)
    ends = list(lay.offsets[1:]) + [lay.L]

    def run(a, b):
        if a == b:
            return
        base = lay.offsets[a]
        rel = off[a:b] - np.uint64(base)
        sub = (ctypes.c_void_p * (b - a))(*[src[i] for i in range(a, b)])
        lib().orc_pack(sub, _ptr(nb[a:b]), _ptr(rel), b - a, _ptr(img) + base, ends[b - 1] - base)

    if not ts:
        img[:] = 0
    else:
        _run_parts(run, _parts(len(ts), threads))
    return img


def unpack(img: np.ndarray, lay: Layout, threads: int = 1) -> List[np.ndarray]:
    """O8 unpack; threads > 1 splits the tensor list (disjoint destinations)."""
    outs = [np.empty(nb, dtype=np.uint8) for nb in lay.nbytes]
    dst = (ctypes.c_void_p * max(1, len(outs)))(*[_ptr(t) for t in outs])
    nb = np.array(lay.nbytes, dtype=np.uint64)
    off = np.array(lay.offsets, dtype=np.uint64)

    def run(a, b):
        if a == b:
            return
        sub = (ctypes.c_void_p * (b - a))(*[dst[i] for i in range(a, b)])
        lib().orc_unpack(_ptr(img), sub, _ptr(nb[a:b]), _ptr(off[a:b]), b - a)

    if outs:
        _run_parts(run, _parts(len(outs), threads))
    return outs


# ----------------------------------------------------------------------------
# O3 JF64
# ----------------------------------------------------------------------------
def jf64(img: np.ndarray, C: int, byte0: int = 0, n_c: Optional[int] = None, threads: int = 1) -> np.ndarray:
    """Chunk digests of an image fragment starting at image byte byte0 (a
    multiple of 8); returns d indexed by global chunk id (length n_c).
    threads > 1 (oracle timing): the fragment is cut at
    chunk boundaries, so every thread owns whole digests d[c]."""
    assert img.dtype == np.uint8 and len(img) % 8 == 0 and byte0 % 8 == 0
    if n_c is None:
        n_c = (byte0 + len(img) + C - 1) // C
    d = np.zeros(n_c, dtype=np.uint64)
    img = np.ascontiguousarray(img)
    g0, nw, cw = byte0 // 8, len(img) // 8, C // 8
    c_first, c_end = g0 // cw, (g0 + nw + cw - 1) // cw if nw else g0 // cw

    def run(ca, cb):
        wa, wb = max(g0, ca * cw), min(g0 + nw, cb * cw)
        if wb > wa:
            lib().orc_jf64_accumulate(_ptr(img) + 8 * (wa - g0), wa, wb - wa, cw, _ptr(d))

    parts = [(c_first + a, c_first + b) for a, b in _parts(c_end - c_first, threads)]
    _run_parts(run, parts)
    return d


def root(layout_hash: int, d: np.ndarray) -> int:
    d = np.ascontiguousarray(d, dtype=np.uint64)
    return lib().orc_root(layout_hash & MASK, _ptr(d), len(d))


# ----------------------------------------------------------------------------
# O4 record and per-rank blob
# ----------------------------------------------------------------------------
MAGIC_R = int.from_bytes(b"JITR", "little")
MAGIC_B = int.from_bytes(b"JITB", "little")
MAGIC_S = int.from_bytes(b"JITS", "little")
MAGIC_M = int.from_bytes(b"JITM", "little")
MAGIC_C = int.from_bytes(b"JITC", "little")


@dataclass
class Record:
    rank: int
    group: int
    policy: int
    phase: int
    version: int
    layout_hash: int
    C: int
    L: int
    d: np.ndarray
    root: int = 0

    @property
    def n_c(self) -> int:
        return len(self.d)


def encode_record(r: Record) -> bytes:
    """O4: 64-B header then d[0..n_c), little-endian."""
    hdr = struct.pack("<IHBBiIQQQQQQ", MAGIC_R, 1, r.policy, r.phase, r.rank, r.group,
                      r.version, r.layout_hash, r.n_c, r.C, r.root, r.L)
    return hdr + np.asarray(r.d, dtype="<u8").tobytes()


def decode_record(buf: bytes, pos: int = 0) -> Tuple[Record, int]:
    (magic, fmt, policy, phase, rank, group, version, lh, n_c, C, rt, L) = \
        struct.unpack_from("<IHBBiIQQQQQQ", buf, pos)
    if magic != MAGIC_R or fmt != 1:
        raise ValueError("bad record")
    d = np.frombuffer(buf, dtype="<u8", count=n_c, offset=pos + 64).astype(np.uint64)
    return Record(rank, group, policy, phase, version, lh, C, L, d, rt), pos + 64 + 8 * n_c


@dataclass
class TopoEntry:
    group: int
    policy: int
    members: List[int]


def topo_hash(topo: Sequence[TopoEntry]) -> int:
    xs = [len(topo)]
    for e in sorted(topo, key=lambda e: e.group):
        xs += [e.group, e.policy, len(e.members)] + sorted(e.members)
    return fold_fmix64(xs)


def encode_blob(rank: int, topo: Sequence[TopoEntry], recs: Sequence[Record]) -> bytes:
    """Per-rank blob: 32-B header, topology table, then the group records.
    header: u32 'JITB', u16 fmt=1, u16 n_topo, i32 rank, u32 n_recs,
            u64 blob_bytes, u64 topo_hash."""
    topo = sorted(topo, key=lambda e: e.group)
    tb = b""
    for e in topo:
        ms = sorted(e.members)
        ent = struct.pack("<IBBH", e.group, e.policy, 0, len(ms)) + struct.pack(f"<{len(ms)}i", *ms)
        ent += b"\0" * ((-len(ent)) % 8)
        tb += ent
    rb = b"".join(encode_record(r) for r in recs)
    total = 32 + len(tb) + len(rb)
    hdr = struct.pack("<IHHiIQQ", MAGIC_B, 1, len(topo), rank, len(recs), total, topo_hash(topo))
    return hdr + tb + rb


def decode_blobs(buf: bytes):
    """Concatenated blobs -> list of (rank, topo, topo_hash, [Record])."""
    out, pos = [], 0
    while pos < len(buf):
        magic, fmt, n_topo, rank, n_recs, total, th = struct.unpack_from("<IHHiIQQ", buf, pos)
        if magic != MAGIC_B or fmt != 1:
            raise ValueError("bad blob")
        p = pos + 32
        topo = []
        for _ in range(n_topo):
            g, pol, _pad, nm = struct.unpack_from("<IBBH", buf, p)
            ms = list(struct.unpack_from(f"<{nm}i", buf, p + 8))
            p += 8 + 4 * nm + ((-(8 + 4 * nm)) % 8)
            topo.append(TopoEntry(g, pol, ms))
        recs = []
        for _ in range(n_recs):
            r, p = decode_record(buf, p)
            recs.append(r)
        out.append((rank, topo, th, recs))
        pos += total
    return out


# ----------------------------------------------------------------------------
# O5 shard rule (reading R9: sharded 1/k save instead of PAPER.md:136's
# every-rank-writes-everything)
# ----------------------------------------------------------------------------
def shard(n_c: int, k: int, s: int) -> Tuple[int, int]:
    """Writer s of k gets chunks [floor(s*n_c/k), floor((s+1)*n_c/k))."""
    return (s * n_c) // k, ((s + 1) * n_c) // k


def shard_bytes(n_c: int, k: int, s: int, C: int, L: int) -> Tuple[int, int]:
    c0, c1 = shard(n_c, k, s)
    return min(c0 * C, L), min(c1 * C, L)


# ----------------------------------------------------------------------------
# O6 select  (PAPER.md:140 §3.3 any replica / discard corrupted; :148 i vs i+1;
# :176-178 barrier invariant; :184-188 optimizer-step failure + hooks;
# :491 pure ZeRO has no replica)
# ----------------------------------------------------------------------------
@dataclass
class GroupSel:
    group: int
    policy: int
    status: int = G_OK
    layout_hash: int = 0
    C: int = 0
    n_c: int = 0
    L: int = 0
    root: int = 0
    writers: List[int] = field(default_factory=list)
    members: List[int] = field(default_factory=list)
    excluded: List[Tuple[int, int]] = field(default_factory=list)
    conflict_chunks: List[int] = field(default_factory=list)


@dataclass
class Selection:
    status: int
    v_star: int = 0
    topo_hash: int = 0
    groups: List[GroupSel] = field(default_factory=list)
    bad_group: int = -1


def select(blobs_buf: bytes, healthy: Sequence[int]) -> Selection:
    """O6, step by step."""
    blobs = decode_blobs(blobs_buf)
    healthy = set(healthy)
    blobs = [b for b in blobs if b[0] in healthy]
    if not blobs:
        return Selection(ENOREPLICA)
    # every rank must declare the same job topology (group -> policy, members)
    ths = {b[2] for b in blobs}
    if len(ths) != 1:
        return Selection(ELAYOUT)
    topo = sorted(blobs[0][1], key=lambda e: e.group)
    th = blobs[0][2]
    recs = sorted([r for b in blobs for r in b[3]], key=lambda r: (r.group, r.rank))

    gsel: Dict[int, GroupSel] = {}
    cand: Dict[int, Dict[int, List[Record]]] = {}     # group -> version -> class
    conflict: Dict[int, Dict[int, List[int]]] = {}    # group -> version -> differing chunks
    no_record: List[int] = []
    for e in topo:
        G = e.group
        gs = GroupSel(G, e.policy, members=sorted(e.members))
        gsel[G] = gs
        # 1. records of the healthy members
        RG = [r for r in recs if r.group == G and r.rank in healthy and r.rank in e.members]
        # 2. layout mismatch is a hard error
        if len({(r.layout_hash, r.C, r.n_c, r.L) for r in RG}) > 1:
            return Selection(ELAYOUT, topo_hash=th, bad_group=G)
        # 3. no records -> no replica
        if not RG:
            gs.status = G_NOREPLICA
            no_record.append(G)
            cand[G], conflict[G] = {}, {}
            continue
        gs.layout_hash, gs.C, gs.n_c, gs.L = RG[0].layout_hash, RG[0].C, RG[0].n_c, RG[0].L
        # 4. CLEAN records
        CG = [r for r in RG if r.phase == CLEAN]
        # 5. per version: unique largest class of identical roots
        cand[G], conflict[G] = {}, {}
        for v in sorted({r.version for r in CG}):
            classes: Dict[int, List[Record]] = {}
            for r in CG:
                if r.version == v:
                    classes.setdefault(r.root, []).append(r)
            sizes = sorted((len(c) for c in classes.values()), reverse=True)
            if len(sizes) > 1 and sizes[0] == sizes[1]:
                tied = [c for c in classes.values() if len(c) == sizes[0]]
                ds = [c[0].d for c in tied]
                diff = sorted({int(i) for a in ds for b in ds for i in np.nonzero(a != b)[0]})
                conflict[G][v] = diff
            else:
                cand[G][v] = max(classes.values(), key=len)
    # 6. V = intersection over REQUIRED groups of versions with a candidate
    req = [e.group for e in topo if e.policy == REQUIRED]
    if req:
        V = None
        for G in req:
            s = set(cand[G].keys())
            V = s if V is None else V & s
    else:
        V = set().union(*[set(cand[G].keys()) for G in gsel]) if gsel else set()
    if not V:
        if any(G in no_record for G in req) or (not req and not V):
            st = ENOREPLICA
        else:
            # reading R8b: the failure is a conflict if some version would have
            # been common to all REQUIRED groups had the tied classes counted
            Vp = None
            for G in req:
                s = set(cand[G].keys()) | set(conflict[G].keys())
                Vp = s if Vp is None else Vp & s
            st = ECONFLICT if Vp else ENOCONSISTENT
        sel = Selection(st, topo_hash=th)
        for G, gs in gsel.items():
            if gs.status == G_OK:
                if conflict[G]:
                    gs.status = G_CONFLICT
                    gs.conflict_chunks = conflict[G][max(conflict[G])]
                elif not cand[G]:
                    gs.status = G_NOCANDIDATE
            sel.groups.append(gs)
        return sel
    # 7. v* = max V
    vs = max(V)
    sel = Selection(OK, v_star=vs, topo_hash=th)
    for e in topo:
        G = e.group
        gs = gsel[G]
        if gs.status == G_NOREPLICA:          # only possible for OPTIONAL here
            gs.status = G_DROPPED
            sel.groups.append(gs)
            continue
        c = cand[G].get(vs)
        if c is not None:
            # 8./9. writers = members of the candidate class, sorted by rank
            gs.writers = sorted(r.rank for r in c)
            gs.root = c[0].root
            gs.status = G_UNVERIFIED_SINGLE if len(c) == 1 else G_OK
        else:
            gs.status = G_DROPPED             # OPTIONAL without a candidate at v*
            if vs in conflict[G]:
                gs.conflict_chunks = conflict[G][vs]
        # 10. every other healthy member, with a reason
        for r in recs:
            if r.group != G or r.rank not in healthy or r.rank in gs.writers:
                continue
            if r.phase == DIRTY:
                gs.excluded.append((r.rank, R_DIRTY))
            elif r.version != vs:
                gs.excluded.append((r.rank, R_STALE_VERSION))
            else:
                gs.excluded.append((r.rank, R_MINORITY))
        sel.groups.append(gs)
    return sel


# ----------------------------------------------------------------------------
# O4b manifest, O7 capture_sim, O8 restore_sim  (metadata last: PAPER.md:136;
# discard corrupted via metadata: PAPER.md:140)
# ----------------------------------------------------------------------------
def manifest_trailer(body: bytes) -> int:
    pad = body + b"\0" * ((-len(body)) % 8)
    return fold_fmix64(np.frombuffer(pad, dtype="<u8").tolist())


def encode_manifest(gs: GroupSel, v_star: int, lay: Layout, d: np.ndarray, aux: bytes = b"") -> bytes:
    """O4b, plus the aux section of DESIGN.md §5 (the user's opaque CPU state,
    PAPER.md:132: u64 aux_len, the bytes, zero padding to 8) after the shard
    table; the trailer covers every preceding byte."""
    k = len(gs.writers)
    h = struct.pack("<IHHIIQQQQQII", MAGIC_M, 1, 0, gs.group, len(lay.names), v_star,
                    lay.layout_hash, lay.C, lay.n_c, lay.L, k, 0)
    h += struct.pack(f"<{k}i", *gs.writers) + b"\0" * ((-4 * k) % 8)
    tt = b""
    for nm, dt, nb, off in zip(lay.names, lay.dtypes, lay.nbytes, lay.offsets):
        e = nm.encode()
        tt += struct.pack("<H", len(e)) + e + struct.pack("<IQQ", dt, nb, off)
    tt += b"\0" * ((-len(tt)) % 8)
    dd = np.asarray(d, dtype="<u8").tobytes() + struct.pack("<Q", root(lay.layout_hash, d))
    st = b""
    for s, w in enumerate(gs.writers):
        c0, c1 = shard(lay.n_c, k, s)
        st += struct.pack("<iIQQ", w, 0, c0, c1)
    ax = struct.pack("<Q", len(aux)) + bytes(aux) + b"\0" * ((-len(aux)) % 8)
    body = h + tt + dd + st + ax
    return body + struct.pack("<Q", manifest_trailer(body))


def commit_record(group: int, v_star: int, manifest: bytes) -> bytes:
    tr = struct.unpack_from("<Q", manifest, len(manifest) - 8)[0]
    return struct.pack("<IIQQQ", MAGIC_C, group, v_star, tr, len(manifest))


def capture_sim(gs: GroupSel, v_star: int, lay: Layout, images: Dict[int, np.ndarray],
                digests: Dict[int, np.ndarray]):
    """O7: writer s contributes image_of(writer s)[range_s], re-digested and
    checked against the writer's fingerprint (else EUNSTABLE).  Returns
    (status, host_image, manifest, commit)."""
    k = len(gs.writers)
    host = np.zeros(lay.L, dtype=np.uint8)
    for s, w in enumerate(gs.writers):
        c0, c1 = shard(lay.n_c, k, s)
        b0, b1 = min(c0 * lay.C, lay.L), min(c1 * lay.C, lay.L)
        sl = images[w][b0:b1]
        if b1 > b0:
            dd = jf64(sl, lay.C, b0, lay.n_c)[c0:c1]
            if not np.array_equal(dd, digests[w][c0:c1]):
                return EUNSTABLE, None, None, None
        host[b0:b1] = sl
    man = encode_manifest(gs, v_star, lay, digests[gs.writers[0]])
    return OK, host, man, commit_record(gs.group, v_star, man)


def decode_manifest(man: bytes):
    (magic, fmt, _p, group, n_t, v_star, lh, C, n_c, L, k, _p2) = \
        struct.unpack_from("<IHHIIQQQQQII", man, 0)
    if magic != MAGIC_M:
        raise ValueError("bad manifest")
    p = 64
    writers = list(struct.unpack_from(f"<{k}i", man, p)); p += 4 * k + ((-4 * k) % 8)
    names, dts, nbs, offs = [], [], [], []
    p0 = p
    for _ in range(n_t):
        (ln,) = struct.unpack_from("<H", man, p); p += 2
        names.append(man[p:p + ln].decode()); p += ln
        dt, nb, off = struct.unpack_from("<IQQ", man, p); p += 20
        dts.append(dt); nbs.append(nb); offs.append(off)
    p += (-(p - p0)) % 8
    d = np.frombuffer(man, dtype="<u8", count=n_c, offset=p).astype(np.uint64); p += 8 * n_c
    (rt,) = struct.unpack_from("<Q", man, p); p += 8
    shards = [struct.unpack_from("<iIQQ", man, p + 24 * s) for s in range(k)]; p += 24 * k
    (aux_len,) = struct.unpack_from("<Q", man, p); p += 8
    aux = man[p:p + aux_len]
    lay = Layout(names, nbs, dts, offs, L, C, lh)
    return dict(group=group, v_star=v_star, layout=lay, d=d, root=rt, writers=writers,
                shards=[(w, c0, c1) for w, _, c0, c1 in shards], aux=aux)


def restore_sim(host: np.ndarray, man: Optional[bytes], commit: Optional[bytes]):
    """O8: refuse if uncommitted (EINCOMPLETE); check every chunk digest
    (ECORRUPT + first bad chunk); then unpack.  Returns (status, first_bad, tensors)."""
    if man is None or commit is None:
        return EINCOMPLETE, -1, None
    magic, group, v, tr, mlen = struct.unpack("<IIQQQ", commit)
    body = man[:-8]
    if magic != MAGIC_C or mlen != len(man) or tr != manifest_trailer(body) or \
            tr != struct.unpack_from("<Q", man, len(man) - 8)[0]:
        return EINCOMPLETE, -1, None
    m = decode_manifest(man)
    lay = m["layout"]
    d = jf64(host, lay.C, 0, lay.n_c)
    bad = np.nonzero(d != m["d"])[0]
    if len(bad):
        return ECORRUPT, int(bad[0]), None
    return OK, -1, unpack(host, lay)
