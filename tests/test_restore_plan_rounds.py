"""HOST and PEER restore round schedules at bench-like geometry (8 GiB
slots, 1 MiB chunks, GB-sized images): the plan jitc_restore executes
(jitc_restore_plan, pure host code) ends with a short round, so the K3 unpack
left after the last transfer is short (pipeline drain), while
the rounds still tile every slice exactly once and stay inside the staging
buffer.
tests/test_multirank_gloo.py replays the same plans byte by byte at small
geometry."""
import numpy as np
import pytest

from oracle import oracle as O
from workloads import configs as W

C = 1 << 20
LAST = 512 << 20


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc
    return jitc


def _selection(J, sizes, members, healthy=None):
    healthy = list(members) if healthy is None else list(healthy)
    g = W.GroupSpec(0, W.REQUIRED, list(members))
    for i, b in enumerate(sizes):
        g.tensors.append(W.TensorSpec(f"t{i}", "u8", b, "bytes", i))
    lay = O.layout_of_group(g, C)
    d = np.zeros(lay.n_c, dtype=np.uint64)          # the schedule does not depend on the digests
    topo = [O.TopoEntry(0, O.REQUIRED, list(members))]
    blobs = [O.encode_blob(r, topo, [O.Record(r, 0, O.REQUIRED, O.CLEAN, 3, lay.layout_hash, C, lay.L, d,
                                              O.root(lay.layout_hash, d))]) for r in healthy]
    st, sel = J.select_consistent_replica(b"".join(blobs), healthy)
    assert st == J.OK
    return sel, lay


@pytest.mark.parametrize("n", [1, 2, 3, 8])
@pytest.mark.parametrize("sizes", [[2_100_000_000] * 3 + [123_456_789], [700 << 20], [300 << 20], [5 << 30, 17]])
def test_host_rounds_end_short_and_tile(J, n, sizes):
    staging, slot = 16 << 30, 8 << 30
    sel, lay = _selection(J, sizes, range(n))
    plans = [J.restore_plan(sel, 0, J.HOST, list(range(n)), r, staging, slot) for r in range(n)]
    assert len({(p["round_bytes"], p["slots"], p["n_rounds"]) for p in plans}) == 1
    R, S, nr = plans[0]["round_bytes"], plans[0]["slots"], plans[0]["n_rounds"]
    h2d = np.zeros(lay.n_c + 1, dtype=np.int32)
    for r, p in enumerate(plans):
        unpack = np.zeros(lay.n_c + 1, dtype=np.int32)
        per_round = {}
        for op in p["ops"]:
            assert op["off"] + op["bytes"] <= staging
            assert op["bytes"] <= R
            if op["kind"] == "H2D":
                h2d[op["a"] // C: -(-op["b"] // C)] += 1
            if op["kind"] == "UNPACK":
                unpack[op["a"] // C: -(-op["b"] // C)] += 1
                per_round.setdefault(op["round"], []).append(op)
        assert (unpack[:lay.n_c] == 1).all(), "every rank unpacks every chunk exactly once"
        # blocks of one round do not overlap in the slot
        for ops in per_round.values():
            iv = sorted((op["off"], op["off"] + op["b"] - op["a"]) for op in ops)
            assert all(a1 <= b0 for (_, a1), (b0, _) in zip(iv, iv[1:]))
        # the last round of the schedule is short when the slice is longer than it
        slice_len = -(-lay.n_c // n) * C
        last = [op for op in p["ops"] if op["kind"] == "UNPACK" and op["round"] == nr - 1]
        if slice_len > LAST and last:
            assert max(op["b"] - op["a"] for op in last) <= LAST
    assert (h2d[:lay.n_c] == 1).all(), "the members' H2D slices tile the image exactly once"


@pytest.mark.parametrize("n", [2, 3, 8])
@pytest.mark.parametrize("sizes", [[2_100_000_000] * 3 + [123_456_789], [700 << 20], [5 << 30, 17]])
def test_peer_rounds_end_short_and_tile(J, n, sizes):
    """PEER: the last rank is the replacement; the n - 1 writers stream their
    O5 ranges.  The replacement unpacks every chunk exactly once, each writer
    packs exactly its own range, the last round is short."""
    staging, slot = 16 << 30, 8 << 30
    sel, lay = _selection(J, sizes, range(n), healthy=range(n - 1))
    plans = [J.restore_plan(sel, 0, J.PEER, list(range(n)), r, staging, slot) for r in range(n)]
    R, nr = plans[0]["round_bytes"], plans[0]["n_rounds"]
    k = n - 1
    unpack = np.zeros(lay.n_c + 1, dtype=np.int32)
    for r, p in enumerate(plans):
        pack = np.zeros(lay.n_c + 1, dtype=np.int32)
        for op in p["ops"]:
            if op["kind"] in ("DIGEST_SEND", "DIGEST_RECV"):
                continue
            assert op["off"] + op["bytes"] <= staging and op["bytes"] <= R
            if op["kind"] == "PACK":
                pack[op["a"] // C: -(-op["b"] // C)] += 1
            if op["kind"] == "UNPACK":
                assert r == n - 1
                unpack[op["a"] // C: -(-op["b"] // C)] += 1
        if r < k:
            c0, c1 = r * lay.n_c // k, (r + 1) * lay.n_c // k
            assert (pack[c0:c1] == 1).all() and pack[:c0].sum() == 0 and pack[c1:].sum() == 0
    assert (unpack[:lay.n_c] == 1).all()
    slice_len = -(-lay.n_c // k) * C
    last = [op for op in plans[n - 1]["ops"] if op["kind"] == "UNPACK" and op["round"] == nr - 1]
    if slice_len > LAST:
        assert last and max(op["b"] - op["a"] for op in last) <= LAST
