"""CPU-side checks of the C ABI (no GPU): libjitc.so loads, exports every
symbol include/jitc.h declares, the pure functions (layout, shard rule,
replica selection) agree with the oracle, and device calls fail loudly
(JITC_ECUDA) instead of falling back to the CPU."""
import os
import random
import re

import numpy as np
import pytest

from oracle import oracle as O
from workloads import configs as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    return jitc


def test_exports_every_declared_symbol(J):
    hdr = open(os.path.join(ROOT, "include", "jitc.h")).read()
    declared = set(re.findall(r"\b(jitc_[a-z0-9_]+)\s*\(", hdr))
    assert len(declared) >= 25
    L = J.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert set(J.EXPORTED) == declared
    assert L.jitc_abi_version() == 2


def test_no_cpu_fallback(J):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(J.JitcError) as e:
        J.Context(device=0)
    assert e.value.status == J.ECUDA


def test_layout_matches_oracle(J):
    for seed in range(5):
        g = W.random_table(seed, 50)
        tab = [(t.name, t.nbytes, W.DTYPE_CODE[t.dtype]) for t in g.tensors]
        for C in (4096, 1 << 20):
            offs, lh, L = J.layout(tab, C)
            ref = O.layout_of_group(g, C)
            assert offs == ref.offsets and lh == ref.layout_hash and L == ref.L
    for cfg in (W.c1(), W.c2()):
        for g in cfg.groups:
            tab = [(t.name, t.nbytes, W.DTYPE_CODE[t.dtype]) for t in g.tensors]
            offs, lh, L = J.layout(tab, 1 << 20)
            ref = O.layout_of_group(g, 1 << 20)
            assert (offs, lh, L) == (ref.offsets, ref.layout_hash, ref.L)


def test_layout_rejects_bad_chunk(J):
    with pytest.raises(J.JitcError):
        J.layout([("a", 10, 0)], 3000)


def test_shard_range_matches_oracle(J):
    for n_c in list(range(0, 70)) + [23768, 122533, 2**40 + 3]:
        for k in range(1, 17):
            for s in range(k):
                assert J.shard_range(n_c, k, s) == O.shard(n_c, k, s)


# --------------------------------------------------------------- selection parity
def _rec(rank, group, version, phase=O.CLEAN, content=0, policy=O.REQUIRED, lh=0x55, n_c=9):
    d = np.random.default_rng(content).integers(0, 2**63, n_c, dtype=np.int64).astype(np.uint64)
    return O.Record(rank, group, policy, phase, version, lh, 4096, n_c * 4096, d, O.root(lh, d))


def _compare(J, buf, healthy):
    ref = O.select(buf, healthy)
    st, sel = J.select_consistent_replica(buf, healthy)
    got = J.parse_selection(sel)
    assert st == ref.status == got["status"]
    if ref.status in (O.OK, O.ECONFLICT, O.ENOCONSISTENT, O.ENOREPLICA):
        assert got["v_star"] == ref.v_star
        gs = {g["group"]: g for g in got["groups"]}
        assert sorted(gs) == sorted(g.group for g in ref.groups)
        for rg in ref.groups:
            g = gs[rg.group]
            assert g["status"] == rg.status, (rg.group, g, rg)
            assert g["writers"] == rg.writers
            assert sorted(g["excluded"]) == sorted(rg.excluded)
            assert g["conflict_chunks"] == rg.conflict_chunks
            assert g["members"] == rg.members
            if rg.writers:
                assert g["root"] == rg.root
    return st, got


def test_select_truth_table_matches_oracle(J):
    """Re-runs the S1..S11-style scenarios through the C ABI."""
    import tests.test_oracle_select as T
    topo8 = T.dp_topo(8)
    I = 10
    cases = []
    cases.append((T.blobs(topo8, {r: [T.rec(r, 0, I)] for r in range(8) if r != 3}), [0, 1, 2, 4, 5, 6, 7]))
    cases.append((T.blobs(topo8, {r: [T.rec(r, 0, I + 1)] for r in range(8) if r != 3}), [0, 1, 2, 4, 5, 6, 7]))
    rb = {r: [T.rec(r, 0, I + 1)] for r in range(8) if r != 3}
    rb[3] = [T.rec(3, 0, I, phase=O.DIRTY, content=777)]
    cases.append((T.blobs(topo8, rb), list(range(8))))
    rb[3] = [T.rec(3, 0, I + 1, content=777)]
    cases.append((T.blobs(topo8, rb), list(range(8))))
    rb = {r: [T.rec(r, 0, I)] for r in range(8)}
    rb[5] = [T.rec(5, 0, I, content=555)]
    cases.append((T.blobs(topo8, rb), list(range(8))))
    topo2 = T.dp_topo(2)
    cases.append((T.blobs(topo2, {0: [T.rec(0, 0, I, content=9)]}), [0]))
    a, b = T.rec(0, 0, I), T.rec(1, 0, I, content=4242)
    b.d = a.d.copy(); b.d[7] ^= np.uint64(1 << 20); b.root = O.root(T.LH, b.d)
    cases.append((T.blobs(topo2, {0: [a], 1: [b]}), [0, 1]))
    for shards, mode in ((8, "pure"), (4, "s8"), (4, "s9")):
        topo = T._zero_topo(shards)
        rb = {}
        for r in range(8):
            if r == 2:
                continue
            if mode == "pure":
                rb[r] = [T.rec(r, 0, I), T.rec(r, 1, I, policy=O.OPTIONAL), T.rec(r, 2 + r, I)]
            elif mode == "s8":
                p = T.rec(r, 0, I + 1) if r >= 4 else T.rec(r, 0, I, phase=O.DIRTY, content=100 + r)
                rb[r] = [p, T.rec(r, 1, I, policy=O.OPTIONAL), T.rec(r, 2 + (r % 4), I + 1)]
            else:
                p = T.rec(r, 0, I) if r % 2 else T.rec(r, 0, I, phase=O.DIRTY, content=300 + r)
                rb[r] = [p, T.rec(r, 1, I, policy=O.OPTIONAL), T.rec(r, 2 + (r % 4), I + 1)]
        cases.append((T.blobs(topo, rb), list(rb)))
    rb = {r: [T.rec(r, 0, I)] for r in range(4)}
    rb[2] = [T.rec(2, 0, I, lh=T.LH + 1)]
    cases.append((T.blobs(T.dp_topo(4), rb), list(rb)))
    want = [O.OK, O.OK, O.OK, O.OK, O.OK, O.OK, O.ECONFLICT, O.ENOREPLICA, O.OK, O.ENOCONSISTENT, O.ELAYOUT]
    for (buf, healthy), w in zip(cases, want):
        st, _ = _compare(J, buf, healthy)
        assert st == w


def test_select_random_record_sets_match_oracle(J):
    """Library vs oracle on 3000 random multi-group record sets (versions i/i+1,
    CLEAN/DIRTY, corrupted replicas, dead ranks, OPTIONAL groups)."""
    rnd = random.Random(2024)
    for trial in range(3000):
        world = rnd.randint(1, 6)
        ngroups = rnd.randint(1, 3)
        topo = []
        for gi in range(ngroups):
            k = rnd.randint(1, world)
            members = sorted(rnd.sample(range(world), k))
            topo.append(O.TopoEntry(gi, rnd.choice([O.REQUIRED, O.REQUIRED, O.OPTIONAL]), members))
        healthy = sorted(r for r in range(world) if rnd.random() < 0.8)
        rb = {}
        for r in healthy:
            recs = []
            for e in topo:
                if r not in e.members:
                    continue
                v = 10 + rnd.randint(0, 1)
                ph = O.DIRTY if rnd.random() < 0.15 else O.CLEAN
                content = 1000 * e.group + v + (rnd.randint(1, 3) if rnd.random() < 0.2 else 0)
                recs.append(_rec(r, e.group, v, ph, content, e.policy))
            rb[r] = recs
        if not rb:
            continue
        buf = b"".join(O.encode_blob(r, topo, rb[r]) for r in sorted(rb))
        _compare(J, buf, healthy)


def test_select_rejects_garbage(J):
    st = J.lib().jitc_select_consistent_replica(b"\0" * 40, 40, None, 0, None, 0, None)
    assert st == J.EINVAL


def test_select_exhaustive_small_worlds_match_oracle(J):
    """The C ABI's selection equals the oracle's on every small-world pure-DP
    scenario of the brute-force pin (tests/test_oracle_select.py)."""
    import tests.test_oracle_select as T
    n = 0
    for states in T.small_world_scenarios():
        buf, healthy = T.scenario_buffer(states)
        if not buf:
            continue
        _compare(J, buf, healthy)
        n += 1
    assert n > 10000
