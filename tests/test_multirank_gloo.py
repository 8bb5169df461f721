"""N > 1 host logic, run as real multi-process jobs on CPU (torch.distributed
gloo, world size 2 and 4, 127.0.0.1): every rank fingerprints its replicas
with the oracle, the blobs are all-gathered, every rank runs the LIBRARY's
selection rule and computes the LIBRARY's restore round plan for every group
(jitc_restore_plan, the schedule jitc_restore executes).  Rank 0 then checks
that all ranks agree and replays the gathered plans byte by byte (H2D,
in-place all-gather, point-to-point send/recv, K2 pack, K3 unpack) on numpy
buffers: every destination must rebuild the committed image exactly, every
send must meet exactly one receive in the same round, and ranks outside a
group must get no operations for it (a TP group's exchange may not involve
the whole communicator).  The NCCL and CUDA calls themselves need GPUs; this
covers everything around them."""
import os
import socket
import traceback

import numpy as np
import pytest
import torch.multiprocessing as mp

GEOMS = [(8 * 4096 * 4, 4 * 4096), (2 * 4096 * 4, 4096 * 4), (64 * 4096, 64 * 4096), (6 * 4096 * 4, 3 * 4096)]
HOST, PEER = 0, 1


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _topology(scenario, world):
    if scenario.startswith("tp"):            # two TP partitions replicated over DP2
        return {0: [0, 2], 1: [1, 3]}
    return {0: list(range(world))}


def _worker(rank, world, port, scenario, q):
    try:
        import sys
        root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
        sys.path.insert(0, root)
        import torch.distributed as dist
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        from oracle import oracle as O
        from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
        from workloads import configs as W

        C = 4096
        topo = _topology(scenario, world)
        base = W.scaled(W.c1(), 3000).groups[0]
        dead = {"peer": 1, "tp_peer": 2}.get(scenario, -1)
        recs, images, lays = [], {}, {}
        for gid, members in topo.items():
            g = base
            lay = O.layout_of_group(g, C)
            img = O.pack(O.gen_group(g, 77 + gid), lay)
            images[gid], lays[gid] = img, lay
            if rank not in members:
                continue
            mine = img
            if scenario == "flip" and rank == world - 1:
                mine = img.copy()
                mine[lay.L // 3] ^= 0x20
            d = O.jf64(mine, C, 0, lay.n_c)
            recs.append(O.Record(rank, gid, O.REQUIRED, O.CLEAN, 5, lay.layout_hash, C, lay.L, d,
                                 O.root(lay.layout_hash, d)))
        tentries = [O.TopoEntry(gid, O.REQUIRED, m) for gid, m in topo.items()]
        blob = O.encode_blob(rank, tentries, recs)
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        healthy = [r for r in range(world) if r != dead]
        allb = b"".join(blobs[r] for r in healthy)
        st, sel = J.select_consistent_replica(allb, healthy)
        sels = [None] * world
        dist.all_gather_object(sels, (st, sel))
        plans = {}
        if st == J.OK:
            for gid in topo:
                for mode in (HOST, PEER):
                    for stg, slot in GEOMS:
                        plans[(gid, mode, stg, slot)] = J.restore_plan(sel, gid, mode, list(range(world)), rank, stg,
                                                                       slot)
        allplans = [None] * world
        dist.all_gather_object(allplans, plans)
        if rank == 0:
            ref = O.select(allb, healthy)
            q.put(("ok", dict(sels=sels, plans=allplans, topo=topo, lays={g: (l.n_c, l.L) for g, l in lays.items()},
                              imgs={g: i.tobytes() for g, i in images.items()}, ref_status=ref.status,
                              ref_writers={x.group: x.writers for x in ref.groups})))
        dist.barrier()
        dist.destroy_process_group()
    except Exception:
        q.put(("err", traceback.format_exc()))


def _run(world, scenario):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, scenario, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
    assert res[0] == "ok", res[1]
    assert all(p.exitcode == 0 for p in procs)
    return res[1]


def _replay(plans, n, img, L, sources):
    """Replays every rank's plan for one group, round by round.  `sources`:
    rank -> the image that rank's live HBM holds (writers, PEER) -- the host
    image is `img`.  Returns (restored images per rank, coverage per rank)."""
    ops_all = [op for p in plans for op in p["ops"]]
    size = max([op["off"] + op["bytes"] * (n if op["kind"] == "ALLGATHER" else 1)
                for op in ops_all if op["kind"] not in ("DIGEST_SEND", "DIGEST_RECV")] + [1])
    stage = [np.zeros(size, dtype=np.uint8) for _ in range(n)]
    out = [np.zeros(L, dtype=np.uint8) for _ in range(n)]
    cover = [np.zeros(L, dtype=np.int32) for _ in range(n)]
    h2d_cover = np.zeros(L, dtype=np.int32)
    pack_cover = np.zeros(L, dtype=np.int32)
    rounds = sorted({op["round"] for op in ops_all})
    for j in rounds:
        ops = [[op for op in plans[r]["ops"] if op["round"] == j and op["kind"] not in ("DIGEST_SEND", "DIGEST_RECV")]
               for r in range(n)]
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "H2D":
                    assert op["peer"] == r and op["b"] - op["a"] == op["bytes"]
                    stage[r][op["off"]:op["off"] + op["bytes"]] = img[op["a"]:op["b"]]
                    h2d_cover[op["a"]:op["b"]] += 1
                if op["kind"] == "PACK":
                    stage[r][op["off"]:op["off"] + op["bytes"]] = sources[r][op["a"]:op["b"]]
                    pack_cover[op["a"]:op["b"]] += 1
        ags = [r for r in range(n) if any(op["kind"] == "ALLGATHER" for op in ops[r])]
        if ags:
            assert ags == list(range(n)), "an all-gather is only planned when the group spans the communicator"
            (base, R), = {(op["off"], op["bytes"]) for r in range(n) for op in ops[r] if op["kind"] == "ALLGATHER"}
            blocks = [stage[q][base + q * R: base + (q + 1) * R].copy() for q in range(n)]
            for r in range(n):
                for q in range(n):
                    stage[r][base + q * R: base + (q + 1) * R] = blocks[q]
        sends = [(r, op) for r in range(n) for op in ops[r] if op["kind"] == "SEND"]
        recvs = [(r, op) for r in range(n) for op in ops[r] if op["kind"] == "RECV"]
        matched = set()
        for d, rv in recvs:
            m = [i for i, (w, sd) in enumerate(sends)
                 if w == rv["peer"] and sd["peer"] == d and (sd["a"], sd["b"], sd["bytes"]) == (rv["a"], rv["b"], rv["bytes"])]
            assert len(m) == 1, f"recv on {d} from {rv['peer']} round {j} unmatched"
            matched.add(m[0])
            w, sd = sends[m[0]]
            stage[d][rv["off"]:rv["off"] + rv["bytes"]] = stage[w][sd["off"]:sd["off"] + sd["bytes"]]
        assert len(matched) == len(sends), "every send meets exactly one receive"
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "UNPACK":
                    out[r][op["a"]:op["b"]] = stage[r][op["off"]:op["off"] + op["b"] - op["a"]]
                    cover[r][op["a"]:op["b"]] += 1
    return out, cover, h2d_cover, pack_cover


def _check_group(res, gid, healthy_writers_expected=None):
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    world = len(res["sels"])
    members = res["topo"][gid]
    n_c, L = res["lays"][gid]
    img = np.frombuffer(res["imgs"][gid], dtype=np.uint8)
    sel = res["sels"][0][1]
    gs = next(g for g in J.parse_selection(sel)["groups"] if g["group"] == gid)
    writers = gs["writers"]
    assert writers == res["ref_writers"][gid]
    if healthy_writers_expected is not None:
        assert writers == healthy_writers_expected
    for stg, slot in GEOMS:
        # HOST: every member restarts; the members split the image and exchange it
        plans = [res["plans"][r][(gid, HOST, stg, slot)] for r in range(world)]
        for r in range(world):
            if r not in members:
                assert plans[r]["ops"] == [], "a non-member takes part in another group's restore"
        out, cover, h2d, _ = _replay(plans, world, img, L, {})
        assert (h2d == 1).all(), "the members' H2D slices tile the image exactly once"
        for r in members:
            assert (cover[r] == 1).all() and np.array_equal(out[r], img)
        # PEER: writers stream from live HBM to every non-writer member
        plans = [res["plans"][r][(gid, PEER, stg, slot)] for r in range(world)]
        dests = [m for m in members if m not in writers]
        for r in range(world):
            dsend = [op for op in plans[r]["ops"] if op["kind"] == "DIGEST_SEND"]
            drecv = [op for op in plans[r]["ops"] if op["kind"] == "DIGEST_RECV"]
            if dests and r == writers[0]:
                assert sorted(op["peer"] for op in dsend) == dests
            else:
                assert not dsend
            assert [op["peer"] for op in drecv] == ([writers[0]] if r in dests else [])
            if r not in members or (r in writers and not dests):
                assert all(op["kind"] == "DIGEST_SEND" for op in plans[r]["ops"]) and (r != writers[0] or not plans[r]["ops"] or dests)
        out, cover, _, packc = _replay(plans, world, img, L, {w: img for w in writers})
        if dests:
            assert (packc == 1).all()
        for r in dests:
            assert (cover[r] == 1).all() and np.array_equal(out[r], img)
        for r in range(world):
            if r not in dests:
                assert not cover[r].any()


@pytest.mark.parametrize("world", [2, 4])
def test_dp_host_restore_plan(world):
    res = _run(world, "host")
    st0, sel0 = res["sels"][0]
    assert all(s == (st0, sel0) for s in res["sels"]), "every rank computes identical selection bytes"
    assert st0 == res["ref_status"] == 0
    _check_group(res, 0, list(range(world)))


@pytest.mark.parametrize("world", [2, 4])
def test_dp_peer_restore_plan(world):
    """Rank 1 died and was replaced: the healthy writers rebuild it over NVLink."""
    res = _run(world, "peer")
    st0, sel0 = res["sels"][0]
    assert all(s == (st0, sel0) for s in res["sels"]) and st0 == 0
    _check_group(res, 0, [r for r in range(world) if r != 1])


def test_tp_groups_only_members_take_part():
    """World 4, TP partitions {0,2} and {1,3}: each group's HOST exchange is
    point-to-point among its two members (no whole-communicator all-gather),
    and with rank 2 dead partition 0 is rebuilt from rank 0 alone."""
    res = _run(4, "tp")
    assert all(s == res["sels"][0] for s in res["sels"]) and res["sels"][0][0] == 0
    for gid in (0, 1):
        _check_group(res, gid)
        for r in range(4):
            assert all(op["kind"] != "ALLGATHER" for op in res["plans"][r][(gid, HOST) + GEOMS[0]]["ops"])
    res = _run(4, "tp_peer")
    assert res["sels"][0][0] == 0
    _check_group(res, 0, [0])
    _check_group(res, 1, [1, 3])


def test_flipped_replica_excluded():
    """World 4, rank 3's replica has a flipped bit: all ranks agree it is a
    MINORITY and that the writers are {0, 1, 2}; with world 2 it is a 1-1 tie
    (ECONFLICT) on every rank."""
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    res = _run(4, "flip")
    st0, sel0 = res["sels"][0]
    assert all(s == (st0, sel0) for s in res["sels"])
    g = J.parse_selection(sel0)["groups"][0]
    assert st0 == 0 and g["writers"] == [0, 1, 2] and g["excluded"] == [(3, 3)]
    res = _run(2, "flip")
    assert all(s[0] == J.ECONFLICT for s in res["sels"]) and res["ref_status"] == J.ECONFLICT
