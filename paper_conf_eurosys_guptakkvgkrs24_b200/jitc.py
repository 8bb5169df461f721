"""Thin Python binding of libjitc.so (include/jitc.h): argument marshalling
only -- every step of the path runs in the library's C++/CUDA code.

The binding never falls back to anything: if libjitc.so is missing or the GPU
is not an sm_100 part, the calls raise.  PyTorch is used by callers only for
device memory, streams and process groups.
"""
from __future__ import annotations

import ctypes
import os
import struct
from typing import Dict, List, Optional, Sequence, Tuple

_PKG = os.path.dirname(os.path.abspath(__file__))
# JITC_SO overrides the library path (used only by tests/test_asan.py to load
# the sanitizer build of the same sources).
SO_PATH = os.environ.get("JITC_SO", os.path.join(_PKG, "libjitc.so"))

OK, EINVAL, ESTATE, ENOMEM, ECUDA, ENCCL = 0, -1, -2, -3, -4, -5
ELAYOUT, ENOREPLICA, ECONFLICT, ENOCONSISTENT = -6, -7, -8, -9
EUNSTABLE, ECORRUPT, EINCOMPLETE, EIO, EPEER = -10, -11, -12, -13, -14
STATUS_NAMES = {v: k for k, v in dict(
    OK=OK, EINVAL=EINVAL, ESTATE=ESTATE, ENOMEM=ENOMEM, ECUDA=ECUDA, ENCCL=ENCCL, ELAYOUT=ELAYOUT,
    ENOREPLICA=ENOREPLICA, ECONFLICT=ECONFLICT, ENOCONSISTENT=ENOCONSISTENT, EUNSTABLE=EUNSTABLE,
    ECORRUPT=ECORRUPT, EINCOMPLETE=EINCOMPLETE, EIO=EIO, EPEER=EPEER).items()}
CLEAN, DIRTY = 0, 1
REQUIRED, OPTIONAL = 0, 1
HOST, PEER = 0, 1
# per-group selection status (jitc_sel_group.status) and exclusion reasons (include/jitc.h)
G_OK, G_UNVERIFIED_SINGLE, G_NOREPLICA, G_DROPPED, G_CONFLICT, G_NOCANDIDATE = 0, 1, 2, 3, 4, 5
X_DIRTY, X_STALE_VERSION, X_MINORITY = 1, 2, 3
ALL_GROUPS = 0xFFFFFFFF
F_ZERO_COPY_D2H, F_ZERO_COPY_H2D, F_TIME_KERNELS = 1, 2, 4   # bit 3 is reserved (no effect)
K_DIGEST, K_PACK, K_UNPACK, K_PULL = 1, 2, 3, 4


class JitcError(RuntimeError):
    def __init__(self, status: int, msg: str, first_bad: int = -1):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status
        self.first_bad = first_bad


class Config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("flags", ctypes.c_uint32), ("chunk_bytes", ctypes.c_uint64), ("staging", ctypes.c_void_p),
                ("staging_bytes", ctypes.c_uint64), ("slot_bytes", ctypes.c_uint64),
                ("image_dir", ctypes.c_char_p), ("streams", ctypes.c_void_p * 2)]


class Tensor(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char_p), ("ptr", ctypes.c_void_p), ("nbytes", ctypes.c_uint64),
                ("dtype", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [("ms_host", ctypes.c_double), ("ms_device", ctypes.c_double), ("ms_kernel", ctypes.c_double),
                ("image_bytes", ctypes.c_uint64), ("d2h_bytes", ctypes.c_uint64), ("h2d_bytes", ctypes.c_uint64),
                ("p2p_bytes", ctypes.c_uint64), ("kernel_launches", ctypes.c_uint64), ("rounds", ctypes.c_uint32),
                ("first_bad_chunk", ctypes.c_int32), ("groups_done", ctypes.c_uint32),
                ("groups_skipped", ctypes.c_uint32)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class Span(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("stream", ctypes.c_int32), ("group", ctypes.c_uint32),
                ("round", ctypes.c_uint32), ("t0_ms", ctypes.c_double), ("t1_ms", ctypes.c_double),
                ("bytes", ctypes.c_uint64)]


SPAN_KIND = {1: "K1", 2: "K2", 3: "K3", 4: "K5", 10: "D2H", 11: "H2D", 12: "P2P"}


class KernelCounter(ctypes.Structure):
    _fields_ = [("launches", ctypes.c_uint64), ("bytes", ctypes.c_uint64), ("ms", ctypes.c_double),
                ("span_ms", ctypes.c_double)]


_lib = None
ABI_VERSION = 2   # include/jitc.h JITC_ABI_VERSION


def lib() -> ctypes.CDLL:
    """Loads the in-tree libjitc.so; raises if it has not been built."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise RuntimeError(f"{SO_PATH} not built: run `python -m paper_conf_eurosys_guptakkvgkrs24_b200.build` "
                           "(there is no CPU fallback)")
    L = ctypes.CDLL(SO_PATH)
    if L.jitc_abi_version() != ABI_VERSION:
        raise RuntimeError(f"{SO_PATH} has ABI {L.jitc_abi_version()}, this binding expects {ABI_VERSION}: rebuild it")
    i32, u32, u64, vp, sz = ctypes.c_int32, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_size_t
    P = ctypes.POINTER
    sig = {
        "jitc_create": ([P(Config), P(vp)], i32),
        "jitc_destroy": ([vp], None),
        "jitc_last_error": ([vp], ctypes.c_char_p),
        "jitc_abi_version": ([], ctypes.c_int),
        "jitc_register": ([vp, u32, i32, P(i32), i32, P(Tensor), sz, P(u64), P(u64)], i32),
        "jitc_declare_group": ([vp, u32, i32, P(i32), i32], i32),
        "jitc_mark": ([vp, u32, u64, i32, vp], i32),
        "jitc_phase": ([vp, u32, P(u64), P(i32)], i32),
        "jitc_get_unique_id": ([vp], i32),
        "jitc_comm_init": ([vp, vp, i32, i32, P(i32)], i32),
        "jitc_comm_shrink": ([vp, P(i32), i32], i32),
        "jitc_comm_destroy": ([vp], i32),
        "jitc_comm_init_ipc": ([vp, ctypes.c_char_p, i32, i32, P(i32)], i32),
        "jitc_liveness_init": ([vp, ctypes.c_char_p], i32),
        "jitc_comm_dead": ([vp, P(i32), i32, P(i32)], i32),
        "jitc_fingerprint": ([vp, u32, vp, sz, P(sz)], i32),
        "jitc_exchange_records": ([vp, vp, sz, vp, sz, P(sz)], i32),
        "jitc_select_consistent_replica": ([vp, sz, P(i32), i32, vp, sz, P(sz)], i32),
        "jitc_capture": ([vp, vp, sz, u32, P(Stats)], i32),
        "jitc_commit": ([vp, vp, sz], i32),
        "jitc_restore": ([vp, u32, i32, vp, sz, P(Stats)], i32),
        "jitc_verify": ([vp, u32, vp, sz, P(u64)], i32),
        "jitc_layout": ([P(Tensor), sz, u64, P(u64), P(u64), P(u64)], i32),
        "jitc_shard_range": ([u64, u32, u32, P(u64), P(u64)], i32),
        "jitc_restore_plan": ([vp, sz, u32, i32, P(i32), i32, i32, u64, u64, vp, sz, P(sz)], i32),
        "jitc_capture_plan": ([vp, sz, u32, P(i32), i32, P(i32), i32, i32, u64, u64, vp, sz, P(sz)], i32),
        "jitc_capture_fanout": ([vp, vp, sz, u32, P(i32), i32, P(Stats)], i32),
        "jitc_attach_image": ([vp, u32, u64], i32),
        "jitc_kernel_counters": ([vp, i32, P(KernelCounter)], i32),
        "jitc_reset_counters": ([vp], i32),
        "jitc_timeline_start": ([vp, u32], i32),
        "jitc_timeline_read": ([vp, P(Span), sz, P(sz)], i32),
        "jitc_gen_fill": ([vp, u32, u64, u64, u32, u32, u32, u32, i32, vp], i32),
        "jitc_inject_update": ([vp, u64, u64, u32, u64, vp], i32),
        "jitc_inject_rne": ([vp, vp, u64, vp], i32),
        "jitc_inject_bitflip": ([vp, u64, u32, vp], i32),
        "jitc_inject_hang": ([vp, i32, u32], i32),
        "jitc_inject_release": ([u32], i32),
        "jitc_watch_event": ([vp, vp, u64], i32),
        "jitc_capture_local": ([vp, P(Stats)], i32),
        "jitc_set_aux": ([vp, vp, sz], i32),
        "jitc_get_aux": ([vp, u32, vp, sz, P(sz)], i32),
        "jitc_peer_export": ([vp, u32], i32),
        "jitc_restore_pull": ([vp, u32, vp, sz, P(Stats)], i32),
        "jitc_persist": ([vp, u32, ctypes.c_char_p, P(Stats)], i32),
        "jitc_stage_in": ([vp, u32, ctypes.c_char_p, P(Stats)], i32),
        "jitc_waste_model": ([i32] + [ctypes.c_double] * 7 + [P(ctypes.c_double)] * 3, i32),
        "jitc_watchdog_start": ([vp, u32, i32, vp, vp], i32),
        "jitc_watchdog_wait": ([vp, u32, P(i32), P(u64), P(ctypes.c_double), P(ctypes.c_double), P(Stats)], i32),
        "jitc_watchdog_stop": ([vp], i32),
        "jitc_watchdog_failed": ([vp, P(i32), i32, P(i32)], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


EXPORTED = ["jitc_create", "jitc_destroy", "jitc_last_error", "jitc_abi_version", "jitc_register",
            "jitc_declare_group", "jitc_mark", "jitc_phase", "jitc_get_unique_id", "jitc_comm_init",
            "jitc_comm_shrink", "jitc_comm_destroy", "jitc_comm_init_ipc", "jitc_fingerprint", "jitc_exchange_records",
            "jitc_select_consistent_replica", "jitc_capture", "jitc_commit", "jitc_restore", "jitc_verify",
            "jitc_layout", "jitc_shard_range", "jitc_restore_plan", "jitc_kernel_counters", "jitc_reset_counters", "jitc_gen_fill",
            "jitc_inject_update", "jitc_inject_rne", "jitc_inject_bitflip", "jitc_inject_hang",
            "jitc_inject_release", "jitc_capture_local", "jitc_set_aux", "jitc_get_aux", "jitc_peer_export", "jitc_restore_pull", "jitc_persist", "jitc_stage_in", "jitc_waste_model", "jitc_watch_event", "jitc_watchdog_start", "jitc_watchdog_wait",
            "jitc_watchdog_stop", "jitc_watchdog_failed", "jitc_capture_plan", "jitc_capture_fanout",
            "jitc_attach_image", "jitc_liveness_init", "jitc_comm_dead", "jitc_timeline_start", "jitc_timeline_read"]
ON_HANG_NOTIFY, ON_HANG_LOCAL_CAPTURE, ON_HANG_COLLECTIVE_CAPTURE = 0, 1, 2


def last_error() -> str:
    return lib().jitc_last_error(None).decode(errors="replace")


def _check(st: int, what: str, first_bad: int = -1):
    if st != OK:
        raise JitcError(st, f"{what}: {last_error()}", first_bad)


def _i32arr(xs: Sequence[int]):
    return (ctypes.c_int32 * max(len(xs), 1))(*xs)


# ------------------------------------------------------------------ pure calls
def layout(tensors: Sequence[Tuple[str, int, int]], chunk_bytes: int) -> Tuple[List[int], int, int]:
    """O1 through the C ABI: [(name, nbytes, dtype)] -> (offsets, layout_hash, L)."""
    n = len(tensors)
    names = [t[0].encode() for t in tensors]
    arr = (Tensor * max(n, 1))(*[Tensor(nm, None, nb, dt) for nm, (_, nb, dt) in zip(names, tensors)])
    offs = (ctypes.c_uint64 * max(n, 1))()
    lh, L = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib().jitc_layout(arr, n, chunk_bytes, offs, ctypes.byref(lh), ctypes.byref(L)), "jitc_layout")
    return list(offs)[:n], lh.value, L.value


def shard_range(n_c: int, k: int, s: int) -> Tuple[int, int]:
    a, b = ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib().jitc_shard_range(n_c, k, s, ctypes.byref(a), ctypes.byref(b)), "jitc_shard_range")
    return a.value, b.value


def select_consistent_replica(blobs: bytes, healthy: Sequence[int]) -> Tuple[int, bytes]:
    """Returns (status, selection bytes); the selection is written on every status."""
    L = lib()
    n = ctypes.c_size_t()
    h = _i32arr(list(healthy))
    L.jitc_select_consistent_replica(blobs, len(blobs), h, len(healthy), None, 0, ctypes.byref(n))
    buf = ctypes.create_string_buffer(n.value)
    st = L.jitc_select_consistent_replica(blobs, len(blobs), h, len(healthy), buf, n.value, ctypes.byref(n))
    return st, buf.raw[:n.value]


def parse_selection(sel: bytes) -> dict:
    """Decodes a selection blob for inspection."""
    magic, fmt, n_groups, status, bad_group, v_star, topo_hash, sel_bytes, _ = struct.unpack_from("<IHHiiQQQQ", sel, 0)
    out = dict(status=status, bad_group=bad_group, v_star=v_star, topo_hash=topo_hash, groups=[])
    q = 48
    for _ in range(n_groups):
        (group, policy, gst, k, n_mem, n_ex, n_cf, _r, lh, C, n_c, L, root) = struct.unpack_from("<IBBHIIIIQQQQQ", sel, q)
        q += 64
        ints = struct.unpack_from(f"<{k + n_mem + 2 * n_ex}i", sel, q)
        q += 4 * len(ints)
        q += (-q) % 8
        cf = list(struct.unpack_from(f"<{n_cf}Q", sel, q))
        q += 8 * n_cf
        out["groups"].append(dict(group=group, policy=policy, status=gst, writers=list(ints[:k]),
                                  members=list(ints[k:k + n_mem]),
                                  excluded=[(ints[k + n_mem + 2 * j], ints[k + n_mem + 2 * j + 1]) for j in range(n_ex)],
                                  conflict_chunks=cf, layout_hash=lh, chunk_bytes=C, n_c=n_c, image_bytes=L, root=root))
    return out


MODEL_PERIODIC_OPTIMAL, MODEL_PERIODIC, MODEL_USER_JIT, MODEL_TRANSPARENT_JIT = 0, 1, 2, 3


def waste_model(kind: int, n_gpus: float, f: float, o: float = 0.0, r: float = 0.0, m: float = 0.0,
                o_jit: float = 0.0, c: float = 0.0) -> dict:
    """PAPER.md §5 eqs. 1-8 through the C ABI: {c_opt, w, w_f}."""
    co, w, wf = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    _check(lib().jitc_waste_model(kind, n_gpus, f, o, r, m, o_jit, c, ctypes.byref(co), ctypes.byref(w),
                                  ctypes.byref(wf)), "jitc_waste_model")
    return dict(c_opt=co.value, w=w.value, w_f=wf.value)


OP_NAMES = {1: "H2D", 2: "ALLGATHER", 3: "PACK", 4: "SEND", 5: "RECV", 6: "UNPACK", 7: "DIGEST_SEND", 9: "D2H",
            8: "DIGEST_RECV"}


def restore_plan(selection: bytes, group: int, mode: int, comm_job_ranks: Sequence[int], comm_rank: int,
                 staging_bytes: int, slot_bytes: int) -> dict:
    """The round schedule jitc_restore executes on `comm_rank` (pure; no GPU)."""
    L = lib()
    n = ctypes.c_size_t()
    jr = _i32arr(list(comm_job_ranks))
    args = (selection, len(selection), group, mode, jr, len(comm_job_ranks), comm_rank, staging_bytes, slot_bytes)
    _check(L.jitc_restore_plan(*args, None, 0, ctypes.byref(n)), "jitc_restore_plan")
    buf = ctypes.create_string_buffer(n.value)
    _check(L.jitc_restore_plan(*args, buf, n.value, ctypes.byref(n)), "jitc_restore_plan")
    return _parse_plan(buf.raw[:n.value])


def capture_plan(selection: bytes, group: int, movers: Sequence[int], comm_job_ranks: Sequence[int], comm_rank: int,
                 staging_bytes: int, slot_bytes: int) -> dict:
    """The round schedule jitc_capture_fanout executes on `comm_rank` (pure; no GPU)."""
    L = lib()
    n = ctypes.c_size_t()
    jr = _i32arr(list(comm_job_ranks))
    mv = _i32arr(list(movers))
    args = (selection, len(selection), group, mv, len(movers), jr, len(comm_job_ranks), comm_rank, staging_bytes,
            slot_bytes)
    _check(L.jitc_capture_plan(*args, None, 0, ctypes.byref(n)), "jitc_capture_plan")
    buf = ctypes.create_string_buffer(n.value)
    _check(L.jitc_capture_plan(*args, buf, n.value, ctypes.byref(n)), "jitc_capture_plan")
    return _parse_plan(buf.raw[:n.value])


def _parse_plan(raw: bytes) -> dict:
    magic, n_ops, R, S, n_rounds = struct.unpack_from("<IIQII", raw, 0)
    ops = []
    for i in range(n_ops):
        rnd, kind, slot, _p, peer, _p2, a, b, off, nb = struct.unpack_from("<IBBHiIQQQQ", raw, 24 + 48 * i)
        ops.append(dict(round=rnd, kind=OP_NAMES[kind], slot=slot, peer=peer, a=a, b=b, off=off, bytes=nb))
    return dict(round_bytes=R, slots=S, n_rounds=n_rounds, ops=ops)


def get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().jitc_get_unique_id(buf), "jitc_get_unique_id")
    return buf.raw


# ------------------------------------------------------------------ K4 harness kernels
def gen_fill(ptr: int, dtype: int, numel: int, seed: int, group: int, gen_id: int, lo: int, hi: int, pos: bool,
             stream: int = 0):
    _check(lib().jitc_gen_fill(ptr, dtype, numel, seed, group, gen_id, lo, hi, int(pos), stream or None),
           "jitc_gen_fill")


def inject_update(ptr: int, e0: int, count: int, gen_id: int, v: int, stream: int = 0):
    _check(lib().jitc_inject_update(ptr, e0, count, gen_id, v, stream or None), "jitc_inject_update")


def inject_rne(master_ptr: int, param_ptr: int, count: int, stream: int = 0):
    _check(lib().jitc_inject_rne(master_ptr, param_ptr, count, stream or None), "jitc_inject_rne")


def inject_bitflip(ptr: int, byte: int, bit: int, stream: int = 0):
    _check(lib().jitc_inject_bitflip(ptr, byte, bit, stream or None), "jitc_inject_bitflip")


def inject_hang(stream: int, n_ctas: int, slot: int = 0):
    """Spinning CTAs on `stream` that emulate a collective hung on a dead peer."""
    _check(lib().jitc_inject_hang(stream or None, n_ctas, slot), "jitc_inject_hang")


def inject_release(slot: int = 0):
    _check(lib().jitc_inject_release(slot), "jitc_inject_release")


# ------------------------------------------------------------------ context
class Context:
    """One libjitc context (one GPU, one process).  Methods map 1:1 to the C ABI."""

    def __init__(self, device: int = 0, rank: int = 0, world: int = 1, chunk_bytes: int = 1 << 20,
                 staging_bytes: int = 0, slot_bytes: int = 0, image_dir: Optional[str] = None, flags: int = 0,
                 staging_ptr: int = 0, streams: Tuple[int, int] = (0, 0)):
        self._L = lib()
        self._image_dir = image_dir.encode() if image_dir else None
        cfg = Config(device, rank, world, flags, chunk_bytes, staging_ptr or None, staging_bytes, slot_bytes,
                     self._image_dir, (ctypes.c_void_p * 2)(streams[0] or None, streams[1] or None))
        h = ctypes.c_void_p()
        _check(self._L.jitc_create(ctypes.byref(cfg), ctypes.byref(h)), "jitc_create")
        self._h = h
        self.rank, self.world = rank, world
        self._keep = []   # tensors registered (caller-owned, must stay alive)

    def close(self):
        if getattr(self, "_h", None):
            self._L.jitc_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- steady state
    def register(self, group: int, policy: int, members: Sequence[int], tensors: Sequence[Tuple[str, int, int, int]],
                 keepalive=None) -> Tuple[int, int]:
        """tensors: [(name, device_ptr, nbytes, dtype)] -> (layout_hash, image_bytes)."""
        names = [t[0].encode() for t in tensors]
        arr = (Tensor * max(len(tensors), 1))(*[Tensor(nm, p or None, nb, dt)
                                                for nm, (_, p, nb, dt) in zip(names, tensors)])
        lh, L = ctypes.c_uint64(), ctypes.c_uint64()
        m = _i32arr(list(members))
        _check(self._L.jitc_register(self._h, group, policy, m, len(members), arr, len(tensors), ctypes.byref(lh),
                                     ctypes.byref(L)), "jitc_register")
        if keepalive is not None:
            self._keep.append(keepalive)
        return lh.value, L.value

    def declare_group(self, group: int, policy: int, members: Sequence[int]):
        _check(self._L.jitc_declare_group(self._h, group, policy, _i32arr(list(members)), len(members)),
               "jitc_declare_group")

    def mark(self, group: int, version: int, phase: int, stream: int = 0):
        _check(self._L.jitc_mark(self._h, group, version, phase, stream or None), "jitc_mark")

    def phase(self, group: int) -> Tuple[int, int]:
        v, p = ctypes.c_uint64(), ctypes.c_int32()
        _check(self._L.jitc_phase(self._h, group, ctypes.byref(v), ctypes.byref(p)), "jitc_phase")
        return v.value, p.value

    # -- communicator
    def comm_init(self, uid: bytes, nranks: int, comm_rank: int, job_ranks: Optional[Sequence[int]] = None):
        jr = _i32arr(list(job_ranks)) if job_ranks is not None else None
        _check(self._L.jitc_comm_init(self._h, uid, nranks, comm_rank, jr), "jitc_comm_init")

    def comm_init_ipc(self, comm_dir: str, nranks: int, comm_rank: int, job_ranks: Optional[Sequence[int]] = None):
        """Intra-node communicator over CUDA IPC + shared memory (no NCCL)."""
        jr = _i32arr(list(job_ranks)) if job_ranks is not None else None
        _check(self._L.jitc_comm_init_ipc(self._h, comm_dir.encode(), nranks, comm_rank, jr), "jitc_comm_init_ipc")

    def liveness_init(self, live_dir: str):
        """Heartbeat table for failure localisation over an NCCL communicator
        (lets ON_HANG_COLLECTIVE_CAPTURE run with jitc_comm_init)."""
        _check(self._L.jitc_liveness_init(self._h, live_dir.encode()), "jitc_liveness_init")

    def comm_dead(self) -> List[int]:
        """Job ranks of the communicator whose heartbeat went stale."""
        buf = (ctypes.c_int32 * 1024)()
        n = ctypes.c_int32()
        _check(self._L.jitc_comm_dead(self._h, buf, 1024, ctypes.byref(n)), "jitc_comm_dead")
        return list(buf[:min(n.value, 1024)])

    def comm_shrink(self, failed: Sequence[int]):
        _check(self._L.jitc_comm_shrink(self._h, _i32arr(list(failed)), len(failed)), "jitc_comm_shrink")

    def comm_destroy(self):
        _check(self._L.jitc_comm_destroy(self._h), "jitc_comm_destroy")

    # -- capture
    def fingerprint(self, group: int = ALL_GROUPS) -> bytes:
        n = ctypes.c_size_t()
        _check(self._L.jitc_fingerprint(self._h, group, None, 0, ctypes.byref(n)), "jitc_fingerprint")
        buf = ctypes.create_string_buffer(n.value)
        _check(self._L.jitc_fingerprint(self._h, group, buf, n.value, ctypes.byref(n)), "jitc_fingerprint")
        return buf.raw[:n.value]

    def exchange_records(self, mine: bytes) -> bytes:
        n = ctypes.c_size_t()
        _check(self._L.jitc_exchange_records(self._h, mine, len(mine), None, 0, ctypes.byref(n)),
               "jitc_exchange_records")
        buf = ctypes.create_string_buffer(max(n.value, 1))
        _check(self._L.jitc_exchange_records(self._h, mine, len(mine), buf, n.value, ctypes.byref(n)),
               "jitc_exchange_records")
        return buf.raw[:n.value]

    def capture(self, selection: bytes, group: int = ALL_GROUPS) -> dict:
        st = Stats()
        _check(self._L.jitc_capture(self._h, selection, len(selection), group, ctypes.byref(st)), "jitc_capture")
        return st.as_dict()

    def capture_fanout(self, selection: bytes, movers: Sequence[int], group: int = ALL_GROUPS) -> dict:
        """Collective: capture with NVLink fan-out over `movers` (job ranks)."""
        st = Stats()
        mv = _i32arr(list(movers))
        _check(self._L.jitc_capture_fanout(self._h, selection, len(selection), group, mv, len(movers),
                                           ctypes.byref(st)), "jitc_capture_fanout")
        return st.as_dict()

    def attach_image(self, group: int, image_bytes: int):
        """Maps and pins the host image of a declared (non-held) group (fan-out mover)."""
        _check(self._L.jitc_attach_image(self._h, group, image_bytes), "jitc_attach_image")

    def capture_local(self) -> dict:
        st = Stats()
        _check(self._L.jitc_capture_local(self._h, ctypes.byref(st)), "jitc_capture_local")
        return st.as_dict()

    def persist(self, group: int, directory: str) -> dict:
        st = Stats()
        _check(self._L.jitc_persist(self._h, group, directory.encode(), ctypes.byref(st)), "jitc_persist")
        return st.as_dict()

    def stage_in(self, group: int, directory: str) -> dict:
        st = Stats()
        _check(self._L.jitc_stage_in(self._h, group, directory.encode(), ctypes.byref(st)), "jitc_stage_in")
        return st.as_dict()

    def set_aux(self, data: bytes):
        """CPU state (iteration, RNG, ...) to carry in the next commit's manifests."""
        _check(self._L.jitc_set_aux(self._h, data, len(data)), "jitc_set_aux")

    def get_aux(self, group: int) -> bytes:
        n = ctypes.c_size_t()
        _check(self._L.jitc_get_aux(self._h, group, None, 0, ctypes.byref(n)), "jitc_get_aux")
        buf = ctypes.create_string_buffer(max(n.value, 1))
        _check(self._L.jitc_get_aux(self._h, group, buf, n.value, ctypes.byref(n)), "jitc_get_aux")
        return buf.raw[:n.value]

    def commit(self, selection: bytes):
        _check(self._L.jitc_commit(self._h, selection, len(selection)), "jitc_commit")

    # -- restore
    def restore(self, group: int = ALL_GROUPS, mode: int = HOST, selection: Optional[bytes] = None) -> dict:
        st = Stats()
        r = self._L.jitc_restore(self._h, group, mode, selection, len(selection) if selection else 0, ctypes.byref(st))
        _check(r, "jitc_restore", st.first_bad_chunk)
        return st.as_dict()

    def peer_export(self, group: int):
        _check(self._L.jitc_peer_export(self._h, group), "jitc_peer_export")

    def restore_pull(self, group: int, selection: bytes) -> dict:
        st = Stats()
        r = self._L.jitc_restore_pull(self._h, group, selection, len(selection), ctypes.byref(st))
        _check(r, "jitc_restore_pull", st.first_bad_chunk)
        return st.as_dict()

    def verify(self, group: int, expected: Optional[bytes] = None) -> int:
        """Returns UINT64_MAX on success; raises JitcError(ECORRUPT) with first_bad on mismatch."""
        fb = ctypes.c_uint64()
        r = self._L.jitc_verify(self._h, group, expected, len(expected) if expected else 0, ctypes.byref(fb))
        _check(r, "jitc_verify", fb.value if r == ECORRUPT else -1)
        return fb.value

    # -- hang detection (NEXT-1)
    def watch_event(self, event_handle: int, tag: int):
        _check(self._L.jitc_watch_event(self._h, event_handle, tag), "jitc_watch_event")

    def watchdog_start(self, timeout_ms: int, action: int = ON_HANG_NOTIFY):
        _check(self._L.jitc_watchdog_start(self._h, timeout_ms, action, None, None), "jitc_watchdog_start")

    def watchdog_wait(self, max_ms: int, hold_gil: bool = False) -> dict:
        """Blocks until the on-hang action finished (or max_ms).  hold_gil=True
        calls through ctypes.PyDLL, i.e. WITHOUT releasing the GIL, to show the
        capture needs no Python thread."""
        f = ctypes.PyDLL(SO_PATH).jitc_watchdog_wait if hold_gil else self._L.jitc_watchdog_wait
        if hold_gil:
            f.argtypes = self._L.jitc_watchdog_wait.argtypes
            f.restype = ctypes.c_int32
        fired, tag = ctypes.c_int32(), ctypes.c_uint64()
        waited, act = ctypes.c_double(), ctypes.c_double()
        st = Stats()
        r = f(self._h, max_ms, ctypes.byref(fired), ctypes.byref(tag), ctypes.byref(waited), ctypes.byref(act),
              ctypes.byref(st))
        _check(r, "jitc_watchdog_wait")
        return dict(fired=bool(fired.value), tag=tag.value, waited_ms=waited.value, action_ms=act.value,
                    stats=st.as_dict())

    def watchdog_failed(self) -> List[int]:
        buf = (ctypes.c_int32 * 64)()
        n = ctypes.c_int32()
        _check(self._L.jitc_watchdog_failed(self._h, buf, 64, ctypes.byref(n)), "jitc_watchdog_failed")
        return list(buf)[:n.value]

    def watchdog_stop(self):
        _check(self._L.jitc_watchdog_stop(self._h), "jitc_watchdog_stop")

    def kernel_counters(self, kind: int) -> dict:
        kc = KernelCounter()
        _check(self._L.jitc_kernel_counters(self._h, kind, ctypes.byref(kc)), "jitc_kernel_counters")
        return dict(launches=kc.launches, bytes=kc.bytes, ms=kc.ms, span_ms=kc.span_ms)

    def timeline_start(self, max_spans: int = 4096):
        """Record the spans (kernel launches, copy batches) of the following calls."""
        _check(self._L.jitc_timeline_start(self._h, max_spans), "jitc_timeline_start")

    def timeline_read(self) -> list:
        n = ctypes.c_size_t()
        _check(self._L.jitc_timeline_read(self._h, None, 0, ctypes.byref(n)), "jitc_timeline_read")
        buf = (Span * max(n.value, 1))()
        _check(self._L.jitc_timeline_read(self._h, buf, n.value, ctypes.byref(n)), "jitc_timeline_read")
        return [dict(kind=SPAN_KIND.get(x.kind, x.kind), stream=x.stream, group=x.group, round=x.round,
                     t0_ms=x.t0_ms, t1_ms=x.t1_ms, bytes=x.bytes) for x in buf[:n.value]]

    def reset_counters(self):
        _check(self._L.jitc_reset_counters(self._h), "jitc_reset_counters")
