"""N > 1 host logic, run as real multi-process jobs on CPU (torch.distributed
gloo, world size 2 and 4, 127.0.0.1): every rank fingerprints its replica with
the oracle, the blobs are all-gathered, every rank runs the LIBRARY's selection
rule and computes the LIBRARY's restore round plan (jitc_restore_plan, the
schedule jitc_restore executes).  Rank 0 then checks that all ranks agree and
replays the gathered plans byte by byte (H2D, in-place all-gather, K2 pack,
send/recv, K3 unpack) on numpy buffers: every destination must rebuild the
committed image exactly, every send must meet exactly one receive.  The NCCL
and CUDA calls themselves need GPUs; this covers everything around them."""
import os
import socket
import traceback

import numpy as np
import pytest
import torch.multiprocessing as mp

GEOMS = [(8 * 4096 * 4, 4 * 4096), (2 * 4096 * 4, 4096 * 4), (64 * 4096, 64 * 4096), (6 * 4096 * 4, 3 * 4096)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


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
        g = W.scaled(W.c1(), 3000).groups[0]
        lay = O.layout_of_group(g, C)
        img = O.pack(O.gen_group(g, 77), lay)
        dead = 1 if scenario == "peer" else -1
        version = 5
        if scenario == "flip" and rank == world - 1:
            img = img.copy()
            img[lay.L // 3] ^= 0x20
        d = O.jf64(img, C, 0, lay.n_c)
        rec = O.Record(rank, 0, O.REQUIRED, O.CLEAN, version, lay.layout_hash, C, lay.L, d, O.root(lay.layout_hash, d))
        blob = O.encode_blob(rank, [O.TopoEntry(0, O.REQUIRED, list(range(world)))], [rec])
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        healthy = [r for r in range(world) if r != dead]
        allb = b"".join(blobs[r] for r in healthy)
        st, sel = J.select_consistent_replica(allb, healthy)
        sels = [None] * world
        dist.all_gather_object(sels, (st, sel))
        plans = {}
        for mode in (J.HOST, J.PEER):
            for stg, slot in GEOMS:
                plans[(mode, stg, slot)] = J.restore_plan(sel, 0, mode, list(range(world)), rank, stg, slot)
        allplans = [None] * world
        dist.all_gather_object(allplans, plans)
        k = len(J.parse_selection(sel)["groups"][0]["writers"]) if st == J.OK else 0
        shards = [J.shard_range(lay.n_c, k, s) for s in range(k)] if k else []
        allshards = [None] * world
        dist.all_gather_object(allshards, shards)
        if rank == 0:
            ref = O.select(allb, healthy)
            q.put(("ok", dict(sels=sels, plans=allplans, shards=allshards, n_c=lay.n_c, L=lay.L, C=C,
                              img=img.tobytes(), ref_status=ref.status,
                              ref_writers=[x.writers for x in ref.groups])))
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


def _simulate_host(plans, n, img, L):
    R_stage = max(max(op["off"] + (op["bytes"] * (n if op["kind"] == "ALLGATHER" else 1)) for op in p["ops"]) for p in plans)
    stage = [np.zeros(R_stage, dtype=np.uint8) for _ in range(n)]
    out = [np.zeros(L, dtype=np.uint8) for _ in range(n)]
    cover = [np.zeros(L, dtype=np.int32) for _ in range(n)]
    h2d_cover = np.zeros(L, dtype=np.int32)
    rounds = sorted({op["round"] for p in plans for op in p["ops"]})
    for j in rounds:
        ops = [[op for op in plans[r]["ops"] if op["round"] == j] for r in range(n)]
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "H2D":
                    assert op["peer"] == r and op["b"] - op["a"] == op["bytes"]
                    stage[r][op["off"]:op["off"] + op["bytes"]] = img[op["a"]:op["b"]]
                    h2d_cover[op["a"]:op["b"]] += 1
        ags = [[op for op in ops[r] if op["kind"] == "ALLGATHER"] for r in range(n)]
        if n > 1:
            assert all(len(a) == 1 for a in ags), "every rank joins every round's all-gather"
            assert len({(a[0]["off"], a[0]["bytes"]) for a in ags}) == 1
            base, R = ags[0][0]["off"], ags[0][0]["bytes"]
            blocks = [stage[q][base + q * R: base + (q + 1) * R].copy() for q in range(n)]
            for r in range(n):
                for q in range(n):
                    stage[r][base + q * R: base + (q + 1) * R] = blocks[q]
        else:
            assert not ags[0]
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "UNPACK":
                    out[r][op["a"]:op["b"]] = stage[r][op["off"]:op["off"] + op["b"] - op["a"]]
                    cover[r][op["a"]:op["b"]] += 1
    assert (h2d_cover == 1).all(), "the n H2D slices tile the image exactly once"
    for r in range(n):
        assert (cover[r] == 1).all() and np.array_equal(out[r], img)


def _simulate_peer(plans, n, img, L, writers):
    size = max([op["off"] + op["bytes"] for p in plans for op in p["ops"] if op["kind"] != "BCAST_DIGESTS"] + [1])
    stage = [np.zeros(size, dtype=np.uint8) for _ in range(n)]
    out = {r: np.zeros(L, dtype=np.uint8) for r in range(n)}
    cover = {r: np.zeros(L, dtype=np.int32) for r in range(n)}
    pack_cover = np.zeros(L, dtype=np.int32)
    for r in range(n):
        b = [op for op in plans[r]["ops"] if op["kind"] == "BCAST_DIGESTS"]
        assert len(b) == 1 and b[0]["peer"] == writers[0]       # every rank joins the digest broadcast
    rounds = sorted({op["round"] for p in plans for op in p["ops"]})
    for j in rounds:
        ops = {r: [op for op in plans[r]["ops"] if op["round"] == j and op["kind"] != "BCAST_DIGESTS"] for r in range(n)}
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "PACK":
                    assert r in writers
                    stage[r][op["off"]:op["off"] + op["bytes"]] = img[op["a"]:op["b"]]
                    pack_cover[op["a"]:op["b"]] += 1
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
    assert (pack_cover == 1).all()
    dests = [r for r in range(n) if r not in writers]
    for r in dests:
        assert (cover[r] == 1).all() and np.array_equal(out[r], img)
    for r in writers:
        assert not cover[r].any()
    return dests


@pytest.mark.parametrize("world", [2, 4])
def test_multirank_host_restore_plan(world):
    res = _run(world, "host")
    st0, sel0 = res["sels"][0]
    assert all(s == (st0, sel0) for s in res["sels"]), "every rank computes identical selection bytes"
    assert st0 == res["ref_status"] == 0
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    assert J.parse_selection(sel0)["groups"][0]["writers"] == res["ref_writers"][0] == list(range(world))
    img = np.frombuffer(res["img"], dtype=np.uint8)
    # sharded capture: the k writers' chunk ranges tile [0, n_c) exactly once
    sh = res["shards"][0]
    assert sh[0][0] == 0 and sh[-1][1] == res["n_c"] and all(a[1] == b[0] for a, b in zip(sh, sh[1:]))
    for stg, slot in GEOMS:
        plans = [res["plans"][r][(J.HOST, stg, slot)] for r in range(world)]
        _simulate_host(plans, world, img, res["L"])
        plans = [res["plans"][r][(J.PEER, stg, slot)] for r in range(world)]
        # all ranks are writers: nothing to send, only the digest broadcast
        assert all(op["kind"] == "BCAST_DIGESTS" for p in plans for op in p["ops"])


@pytest.mark.parametrize("world", [2, 4])
def test_multirank_peer_restore_plan(world):
    """Rank 1 died and was replaced: the healthy writers rebuild it over NVLink."""
    res = _run(world, "peer")
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    st0, sel0 = res["sels"][0]
    assert all(s == (st0, sel0) for s in res["sels"])
    writers = J.parse_selection(sel0)["groups"][0]["writers"]
    assert st0 == 0 and writers == [r for r in range(world) if r != 1] == res["ref_writers"][0]
    img = np.frombuffer(res["img"], dtype=np.uint8)
    for stg, slot in GEOMS:
        plans = [res["plans"][r][(J.PEER, stg, slot)] for r in range(world)]
        assert _simulate_peer(plans, world, img, res["L"], writers) == [1]
        plans = [res["plans"][r][(J.HOST, stg, slot)] for r in range(world)]
        _simulate_host(plans, world, img, res["L"])


def test_multirank_flipped_replica_excluded():
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
