"""Capture with NVLink fan-out: the round
plans of jitc_capture_fanout (jitc_capture_plan, the schedule the executor
runs) for every rank of DP, TP x DP and random topologies, replayed byte by
byte on numpy buffers.  The selection comes from the LIBRARY's rule over
records the ORACLE fingerprints; the expected image is the oracle's pack.

Checked for every topology and staging geometry:
  * the movers' D2H ranges tile the image exactly once, each inside the
    mover's own lane O5(n_c, m, q), and the replayed host image equals the
    oracle image;
  * every writer packs exactly its O5(n_c, k, s) shard (the re-digest range
    of jitc_capture, so EUNSTABLE detection is unchanged) and nobody else
    packs;
  * every SEND meets exactly one RECV in the same round, data flows only
    writer -> mover, and ranks that are neither get no operations;
  * staging offsets stay inside the staging buffer and the blocks of one
    round do not overlap on a rank;
  * with movers == writers the plan has no transfer (plain sharded capture)."""
import random

import numpy as np
import pytest

from oracle import oracle as O
from workloads import configs as W

C = 4096
GEOMS = [(8 * C * 4, 4 * C), (2 * C * 4, C * 4), (64 * C, 64 * C), (6 * C * 4, 3 * C), (4 * C, C)]


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc
    return jitc


@pytest.fixture(scope="module")
def group():
    g = W.scaled(W.c1(), 3000).groups[0]
    lay = O.layout_of_group(g, C)
    img = O.pack(O.gen_group(g, 91), lay)
    return lay, img


def _selection(J, lay, img, topo, healthy, v=7):
    """topo: gid -> members.  Every healthy member fingerprints the same image."""
    blobs = []
    d = O.jf64(img, C, 0, lay.n_c)
    tentries = [O.TopoEntry(gid, O.REQUIRED, m) for gid, m in topo.items()]
    for r in healthy:
        recs = [O.Record(r, gid, O.REQUIRED, O.CLEAN, v, lay.layout_hash, C, lay.L, d, O.root(lay.layout_hash, d))
                for gid, m in topo.items() if r in m]
        blobs.append(O.encode_blob(r, tentries, recs))
    st, sel = J.select_consistent_replica(b"".join(blobs), healthy)
    assert st == J.OK, J.parse_selection(sel)
    return sel


def _o5(n_c, k, s, L):
    return min(s * n_c // k * C, L), min((s + 1) * n_c // k * C, L)


def _replay(J, sel, gid, movers, comm, lay, img, staging, slot):
    n = len(comm)
    gs = next(g for g in J.parse_selection(sel)["groups"] if g["group"] == gid)
    if staging < 2 * len(gs["writers"]) * C:      # not even one chunk per writer and slot
        with pytest.raises(J.JitcError):
            J.capture_plan(sel, gid, movers, comm, 0, staging, slot)
        return None
    plans = [J.capture_plan(sel, gid, movers, comm, r, staging, slot) for r in range(n)]
    writers = [comm.index(w) for w in gs["writers"]]
    mv = [comm.index(q) for q in sorted(movers)]
    k, m, L = len(writers), len(mv), lay.L
    assert len({(p["round_bytes"], p["slots"], p["n_rounds"]) for p in plans}) == 1, "ranks disagree on the rounds"
    S, R = plans[0]["slots"], plans[0]["round_bytes"]
    assert R % C == 0 and 0 < R <= slot and S * k * R <= staging
    stage = [np.zeros(staging, dtype=np.uint8) for _ in range(n)]
    host = np.zeros(L, dtype=np.uint8)
    d2h_cover = np.zeros(L, dtype=np.int32)
    pack_cover = [np.zeros(L, dtype=np.int32) for _ in range(n)]
    for r in range(n):
        if r not in writers and r not in mv:
            assert plans[r]["ops"] == [], "a rank that neither writes nor moves has operations"
        for op in plans[r]["ops"]:
            assert op["off"] + op["bytes"] <= staging and op["b"] - op["a"] == op["bytes"] > 0
            assert op["slot"] == op["round"] % S
            assert op["a"] % C == 0 and (op["b"] % C == 0 or op["b"] == L)
    for j in range(plans[0]["n_rounds"]):
        ops = [[op for op in plans[r]["ops"] if op["round"] == j] for r in range(n)]
        for r in range(n):
            regions = sorted({(op["off"], op["off"] + op["bytes"]) for op in ops[r]})
            for (a0, b0), (a1, b1) in zip(regions, regions[1:]):
                assert b0 <= a1, "blocks of one round overlap in staging"
            for op in ops[r]:
                if op["kind"] == "PACK":
                    assert r in writers and op["peer"] == r
                    stage[r][op["off"]:op["off"] + op["bytes"]] = img[op["a"]:op["b"]]
                    pack_cover[r][op["a"]:op["b"]] += 1
        sends = [(r, op) for r in range(n) for op in ops[r] if op["kind"] == "SEND"]
        recvs = [(r, op) for r in range(n) for op in ops[r] if op["kind"] == "RECV"]
        matched = set()
        for d, rv in recvs:
            assert d in mv and rv["peer"] in writers
            hit = [i for i, (w, sd) in enumerate(sends) if w == rv["peer"] and sd["peer"] == d and
                   (sd["a"], sd["b"], sd["off"]) == (rv["a"], rv["b"], rv["off"])]
            assert len(hit) == 1, f"recv on {d} from {rv['peer']} in round {j} unmatched"
            matched.add(hit[0])
            w, sd = sends[hit[0]]
            stage[d][rv["off"]:rv["off"] + rv["bytes"]] = stage[w][sd["off"]:sd["off"] + sd["bytes"]]
        assert len(matched) == len(sends), "every send meets exactly one receive"
        for r in range(n):
            for op in ops[r]:
                if op["kind"] == "D2H":
                    q = mv.index(r)
                    la, lb = _o5(lay.n_c, m, q, L)
                    assert la <= op["a"] and op["b"] <= lb, "a mover D2Hs outside its lane"
                    host[op["a"]:op["b"]] = stage[r][op["off"]:op["off"] + op["bytes"]]
                    d2h_cover[op["a"]:op["b"]] += 1
    assert (d2h_cover == 1).all(), "the movers' D2H ranges tile the image exactly once"
    assert np.array_equal(host, img)
    for s, w in enumerate(writers):
        a, b = _o5(lay.n_c, k, s, L)
        want = np.zeros(L, dtype=np.int32)
        want[a:b] = 1
        assert np.array_equal(pack_cover[w], want), "a writer packs exactly its O5 shard"
    for r in range(n):
        if r not in writers:
            assert not pack_cover[r].any()
    return plans


@pytest.mark.parametrize("staging,slot", GEOMS)
def test_dp_movers_equal_writers_is_plain_sharded_capture(J, group, staging, slot):
    lay, img = group
    topo = {0: [0, 1, 2, 3]}
    sel = _selection(J, lay, img, topo, [0, 1, 2, 3])
    plans = _replay(J, sel, 0, [0, 1, 2, 3], [0, 1, 2, 3], lay, img, staging, slot) or []
    assert not any(op["kind"] in ("SEND", "RECV") for p in plans for op in p["ops"])


@pytest.mark.parametrize("staging,slot", GEOMS)
def test_tp2_dp2_lone_writer_fans_out(J, group, staging, slot):
    """TP2 x DP2, rank 3 died: partition 1 has one writer (rank 1); the three
    survivors each D2H a third of it, two thirds travel over NVLink."""
    lay, img = group
    topo = {0: [0, 2], 1: [1, 3]}
    comm = [0, 1, 2]
    sel = _selection(J, lay, img, topo, comm)
    for gid in topo:
        plans = _replay(J, sel, gid, comm, comm, lay, img, staging, slot)
    if plans is None:
        return
    sent = sum(op["bytes"] for op in plans[1]["ops"] if op["kind"] == "SEND")
    lane = _o5(lay.n_c, 3, 1, lay.L)
    assert sent == lay.L - (lane[1] - lane[0]), "the lone writer ships every byte outside its own lane"


@pytest.mark.parametrize("staging,slot", GEOMS[:3])
def test_c5_shape_tp4_dp2_rank5_dead(J, group, staging, slot):
    lay, img = group
    topo = {p: [p, p + 4] for p in range(4)}
    comm = [0, 1, 2, 3, 4, 6, 7]
    sel = _selection(J, lay, img, topo, comm)
    for gid in topo:
        _replay(J, sel, gid, comm, comm, lay, img, staging, slot)


def test_random_topologies(J, group):
    lay, img = group
    rng = random.Random(1234)
    for _ in range(40):
        n = rng.randint(1, 8)
        healthy = sorted(rng.sample(range(n), rng.randint(1, n)))
        movers = sorted(rng.sample(healthy, rng.randint(1, len(healthy))))
        staging, slot = rng.choice(GEOMS)
        sel = _selection(J, lay, img, {0: list(range(n))}, healthy)
        _replay(J, sel, 0, movers, healthy, lay, img, staging, slot)


def test_plan_errors(J, group):
    lay, img = group
    sel = _selection(J, lay, img, {0: [0, 1]}, [0, 1])
    with pytest.raises(J.JitcError):
        J.capture_plan(sel, 0, [0, 5], [0, 1], 0, 1 << 20, 1 << 18)    # mover not in the communicator
    with pytest.raises(J.JitcError):
        J.capture_plan(sel, 0, [0, 1], [0, 1], 0, C, C)                 # staging below 2 * k * C
    with pytest.raises(J.JitcError):
        J.capture_plan(sel, 9, [0, 1], [0, 1], 0, 1 << 20, 1 << 18)    # group not in the selection


def test_round_robin_lanes_match_timing_model(J, group):
    """The library's fan-out plan visits the movers' lanes round-robin (each
    writer's j-th block goes to the next lane it intersects), exactly as
    tools/fanout_sim.py models it -- so that model's projections (DESIGN.md
    §8.6) describe the executed schedule -- and consecutive rounds of a lone
    writer go to different movers."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "fanout_sim", os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools", "fanout_sim.py"))
    sim = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(sim)
    sim.C = C
    lay, img = group
    for topo, healthy, gid, movers in (({0: [0, 1]}, [0], 0, [0, 1]),
                                       ({0: [0, 1, 2, 3]}, [0, 1], 0, [0, 1, 2, 3]),
                                       ({0: [0, 2], 1: [1, 3]}, [0, 1, 2], 1, [0, 1, 2])):
        sel = _selection(J, lay, img, topo, healthy)
        gs = next(g for g in J.parse_selection(sel)["groups"] if g["group"] == gid)
        writers = gs["writers"]
        for staging, slot in ((8 * C * 4, 4 * C), (6 * C * 4, 3 * C), (4 * C, C)):
            if staging < 2 * len(writers) * C:
                continue
            R = min(slot, staging // (2 * len(writers))) // C * C
            want = sim.blocks_of(lay.n_c, lay.L, len(writers), len(movers), R, "round-robin")
            for s, w in enumerate(writers):
                plan = J.capture_plan(sel, gid, movers, list(range(4)), w, staging, slot)
                packs = [(op["round"], op["a"], op["b"]) for op in plan["ops"] if op["kind"] == "PACK"]
                assert packs == [(j, a, b) for j, (a, b, q) in enumerate(want[s])]
            if len(writers) == 1:
                lanes = [q for a, b, q in want[0]]
                n_lanes = len(set(lanes))
                assert all(x != y for x, y in zip(lanes, lanes[1:])) or n_lanes == 1
