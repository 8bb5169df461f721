"""The selection rule (O6) against the truth table S1..S11 written from the
paper's cases (tests/golden/selection_truth_table.md):

  PAPER.md:140 §3.3  any DP replica; discard corrupted checkpoints via metadata
  PAPER.md:148 §3.3  state is minibatch i or i+1, both consistent
  PAPER.md:176-178   every rank enters the all-reduce before modifying state
  PAPER.md:184-188   optimizer-step failure: replicas hold i+1; pre/post hooks
  PAPER.md:128, :491 hybrid sharding required; pure ZeRO has no replica
  PAPER.md:37        single failures dominate; SDC rare -> majority of replicas
"""
import numpy as np
import pytest

from oracle import oracle as O

LH, C, NC = 0xABCDEF, 4096, 12


def _d(content: int, n_c=NC):
    return np.random.default_rng(content).integers(0, 2**63, n_c, dtype=np.int64).astype(np.uint64)


def rec(rank, group, version, phase=O.CLEAN, content=None, policy=O.REQUIRED, lh=LH, n_c=NC):
    d = _d(content if content is not None else 1000 * group + version, n_c)
    return O.Record(rank, group, policy, phase, version, lh, C, n_c * C, d, O.root(lh, d))


def blobs(topo, recs_by_rank):
    return b"".join(O.encode_blob(r, topo, recs_by_rank[r]) for r in sorted(recs_by_rank))


def dp_topo(n, groups=((0, O.REQUIRED),)):
    return [O.TopoEntry(g, p, list(range(n))) for g, p in groups]


def gsel(sel, g):
    return next(x for x in sel.groups if x.group == g)


I = 10   # minibatch index at failure


def test_S1_dies_in_fwd_bwd():
    """Pure DP n=8, rank 3 dies in fwd/bwd: seven CLEAN at v=i ⇒ v*=i, 7 writers."""
    topo = dp_topo(8)
    rb = {r: [rec(r, 0, I)] for r in range(8) if r != 3}
    sel = O.select(blobs(topo, rb), [r for r in range(8) if r != 3])
    assert sel.status == O.OK and sel.v_star == I
    g = gsel(sel, 0)
    assert g.writers == [0, 1, 2, 4, 5, 6, 7] and g.status == O.G_OK and not g.excluded


def test_S2_dies_mid_optimizer():
    """Rank 3 dies mid-optimizer; others finish the step and hang at the next
    all-reduce ⇒ seven CLEAN at i+1 ⇒ v* = i+1."""
    topo = dp_topo(8)
    rb = {r: [rec(r, 0, I + 1)] for r in range(8) if r != 3}
    sel = O.select(blobs(topo, rb), list(rb))
    assert sel.status == O.OK and sel.v_star == I + 1 and len(gsel(sel, 0).writers) == 7


@pytest.mark.parametrize("variant", ["dirty", "missed_hook"])
def test_S3_hung_partial_rank_still_readable(variant):
    topo = dp_topo(8)
    rb = {r: [rec(r, 0, I + 1)] for r in range(8) if r != 3}
    if variant == "dirty":
        rb[3] = [rec(3, 0, I, phase=O.DIRTY, content=777)]
        reason = O.R_DIRTY
    else:
        rb[3] = [rec(3, 0, I + 1, content=777)]     # CLEAN at i+1, different bytes
        reason = O.R_MINORITY
    sel = O.select(blobs(topo, rb), list(range(8)))
    g = gsel(sel, 0)
    assert sel.status == O.OK and sel.v_star == I + 1
    assert 3 not in g.writers and (3, reason) in g.excluded and len(g.writers) == 7


def test_S4_bitflip_minority():
    topo = dp_topo(8)
    rb = {r: [rec(r, 0, I)] for r in range(8) if r != 3}
    rb[5] = [rec(5, 0, I, content=555)]
    sel = O.select(blobs(topo, rb), list(rb))
    g = gsel(sel, 0)
    assert sel.status == O.OK and g.writers == [0, 1, 2, 4, 6, 7] and (5, O.R_MINORITY) in g.excluded


def test_S5_lone_survivor_unverified():
    topo = dp_topo(2)
    rb = {0: [rec(0, 0, I, content=999)]}       # flipped, but nobody to compare with
    sel = O.select(blobs(topo, rb), [0])
    g = gsel(sel, 0)
    assert sel.status == O.OK and g.writers == [0] and g.status == O.G_UNVERIFIED_SINGLE


def test_S6_tie_is_conflict():
    topo = dp_topo(2)
    a, b = rec(0, 0, I), rec(1, 0, I, content=4242)
    b.d = a.d.copy(); b.d[7] ^= np.uint64(1 << 20); b.root = O.root(LH, b.d)
    sel = O.select(blobs(topo, {0: [a], 1: [b]}), [0, 1])
    assert sel.status == O.ECONFLICT
    g = gsel(sel, 0)
    assert g.status == O.G_CONFLICT and g.conflict_chunks == [7]


def _zero_topo(shards, world=8):
    topo = [O.TopoEntry(0, O.REQUIRED, list(range(world))), O.TopoEntry(1, O.OPTIONAL, list(range(world)))]
    topo += [O.TopoEntry(2 + j, O.REQUIRED, list(range(j, world, shards))) for j in range(shards)]
    return topo


def test_S7_pure_zero_no_replica():
    """Pure ZeRO-1 (S=8): the dead rank's optimizer shard has no member ⇒
    ENOREPLICA."""
    topo = _zero_topo(8)
    rb = {}
    for r in range(8):
        if r == 2:
            continue
        rb[r] = [rec(r, 0, I), rec(r, 1, I, policy=O.OPTIONAL), rec(r, 2 + r, I)]
    sel = O.select(blobs(topo, rb), list(rb))
    assert sel.status == O.ENOREPLICA
    assert gsel(sel, 4).status == O.G_NOREPLICA


def test_S8_hybrid_zero_in_group_gather():
    """Hybrid S=4 x R=2, rank 2 dies mid-update; params gathered within {0-3}
    and {4-7}: {4..7} complete (params CLEAN at i+1), 0,1,3 hold DIRTY params;
    every optimizer shard has a CLEAN i+1 replica ⇒ v* = i+1."""
    topo = _zero_topo(4)
    rb = {}
    for r in range(8):
        if r == 2:
            continue
        p = rec(r, 0, I + 1) if r >= 4 else rec(r, 0, I, phase=O.DIRTY, content=100 + r)
        gr = rec(r, 1, I, policy=O.OPTIONAL)
        opt = rec(r, 2 + (r % 4), I + 1)
        rb[r] = [p, gr, opt]
    sel = O.select(blobs(topo, rb), list(rb))
    assert sel.status == O.OK and sel.v_star == I + 1
    g0 = gsel(sel, 0)
    assert g0.writers == [4, 5, 6, 7]
    assert sorted(x for x in g0.excluded) == [(0, O.R_DIRTY), (1, O.R_DIRTY), (3, O.R_DIRTY)]
    assert gsel(sel, 4).writers == [6] and gsel(sel, 4).status == O.G_UNVERIFIED_SINGLE
    assert gsel(sel, 2).writers == [0, 4]
    # grads are at i, not i+1: the OPTIONAL group is dropped, not an error
    assert gsel(sel, 1).status == O.G_DROPPED and gsel(sel, 1).writers == []


def test_S9_hybrid_zero_global_gather_inconsistent():
    """Global param gather: params CLEAN only at i (or DIRTY), optimizer shards
    CLEAN only at i+1 ⇒ ENOCONSISTENT (partial update detected, refuse)."""
    topo = _zero_topo(4)
    rb = {}
    for r in range(8):
        if r == 2:
            continue
        p = rec(r, 0, I) if r % 2 else rec(r, 0, I, phase=O.DIRTY, content=300 + r)
        rb[r] = [p, rec(r, 1, I, policy=O.OPTIONAL), rec(r, 2 + (r % 4), I + 1)]
    sel = O.select(blobs(topo, rb), list(rb))
    assert sel.status == O.ENOCONSISTENT


def test_S10_layout_mismatch():
    topo = dp_topo(4)
    rb = {r: [rec(r, 0, I)] for r in range(4)}
    rb[2] = [rec(2, 0, I, lh=LH + 1)]
    assert O.select(blobs(topo, rb), list(rb)).status == O.ELAYOUT
    # a different declared topology is also a layout error
    topo2 = dp_topo(4, groups=((0, O.OPTIONAL),))
    buf = blobs(topo, {0: rb[0], 1: rb[1]}) + O.encode_blob(3, topo2, [rec(3, 0, I)])
    assert O.select(buf, [0, 1, 3]).status == O.ELAYOUT


def test_S11_unstable_between_fingerprint_and_capture():
    """Bytes change between K1 and K2 ⇒ EUNSTABLE (reading R11)."""
    from workloads import configs as W
    g = W.random_table(3, 12)
    lay = O.layout_of_group(g, 4096)
    img = O.pack(O.gen_group(g, 1), lay)
    d = O.jf64(img, lay.C, 0, lay.n_c)
    gs = O.GroupSel(0, O.REQUIRED, writers=[0])
    assert O.capture_sim(gs, I, lay, {0: img}, {0: d})[0] == O.OK
    img2 = img.copy(); img2[lay.L // 2] ^= 4
    assert O.capture_sim(gs, I, lay, {0: img2}, {0: d})[0] == O.EUNSTABLE


def test_stale_version_and_optional_kept_when_consistent():
    topo = dp_topo(4, groups=((0, O.REQUIRED), (1, O.OPTIONAL)))
    rb = {r: [rec(r, 0, I + 1), rec(r, 1, I + 1, policy=O.OPTIONAL)] for r in range(4)}
    rb[1] = [rec(1, 0, I), rec(1, 1, I, policy=O.OPTIONAL)]    # one rank one step behind
    sel = O.select(blobs(topo, rb), list(rb))
    assert sel.status == O.OK and sel.v_star == I + 1
    assert gsel(sel, 0).writers == [0, 2, 3] and (1, O.R_STALE_VERSION) in gsel(sel, 0).excluded
    assert gsel(sel, 1).writers == [0, 2, 3] and gsel(sel, 1).status == O.G_OK


def test_select_is_order_independent():
    """Every rank computes the identical selection from the identical input,
    whatever order the blobs arrive in."""
    topo = dp_topo(6)
    rb = {r: [rec(r, 0, I if r < 4 else I + 1)] for r in range(6)}
    a = O.select(blobs(topo, rb), range(6))
    perm = [4, 1, 5, 0, 3, 2]
    buf = b"".join(O.encode_blob(r, topo, rb[r]) for r in perm)
    b = O.select(buf, range(6))
    assert (a.status, a.v_star, gsel(a, 0).writers) == (b.status, b.v_star, gsel(b, 0).writers)
    # both versions have a candidate; the newer one (2 replicas) wins by max V
    assert a.v_star == I + 1 and gsel(a, 0).writers == [4, 5]


def test_record_blob_roundtrip():
    topo = dp_topo(3, groups=((0, O.REQUIRED), (5, O.OPTIONAL)))
    rs = [rec(1, 0, 4), rec(1, 5, 4, policy=O.OPTIONAL, n_c=3)]
    buf = O.encode_blob(1, topo, rs)
    [(rank, t2, th, r2)] = O.decode_blobs(buf)
    assert rank == 1 and th == O.topo_hash(topo) and len(r2) == 2
    for a, b in zip(rs, r2):
        assert (a.group, a.version, a.root, a.L) == (b.group, b.version, b.root, b.L)
        assert np.array_equal(a.d, b.d)


# ----------------------------------------------------------------------------
# Brute force over small worlds: every pure-DP
# scenario with n <= 4 ranks (and every n = 5 scenario with both i and i+1
# present), each rank dead or alive x version {i, i+1} x phase {CLEAN, DIRTY}
# x corrupted {no, yes}, at most 2 corrupted ranks.  The expectation is not
# the oracle's step-by-step procedure: it is the closed-form statement of the
# rule for one group, written from the paper's cases --
#   * a state is restorable iff it is CLEAN (PAPER.md:184-188 hooks) and held
#     by a strict plurality of identical CLEAN replicas of that minibatch
#     ("discard corrupted"; reading R8: ties are conflicts);
#   * among restorable minibatches the newest wins;
#   * nothing restorable: a conflict if any CLEAN replica exists (then every
#     version present is tied), else no consistent state (all DIRTY);
#   * nobody alive: no replica.
# A dead rank contributes nothing; a corrupted rank's bytes are its own.
# ----------------------------------------------------------------------------
_DEAD = None


def _rank_states():
    yield _DEAD
    for v in (I, I + 1):
        for ph in (O.CLEAN, O.DIRTY):
            for bad in (False, True):
                yield (v, ph, bad)


def _expected_single_group(states):
    alive = {r: s for r, s in enumerate(states) if s is not _DEAD}
    if not alive:
        return O.ENOREPLICA, None, None, None
    content = {r: (v, r if bad else -1) for r, (v, ph, bad) in alive.items()}
    clean = [r for r, (v, ph, bad) in alive.items() if ph == O.CLEAN]
    best = {}
    for v in {alive[r][0] for r in clean}:
        holders = {}
        for r in clean:
            if alive[r][0] == v:
                holders.setdefault(content[r], []).append(r)
        counts = sorted((len(h) for h in holders.values()), reverse=True)
        if len(counts) == 1 or counts[0] > counts[1]:
            best[v] = sorted(max(holders.values(), key=len))
    if not best:
        return (O.ECONFLICT if clean else O.ENOCONSISTENT), None, None, None
    vs = max(best)
    writers = best[vs]
    reasons = {}
    for r, (v, ph, bad) in alive.items():
        if r in writers:
            continue
        reasons[r] = O.R_DIRTY if ph == O.DIRTY else (O.R_STALE_VERSION if v != vs else O.R_MINORITY)
    return O.OK, vs, writers, reasons


def small_world_scenarios(max_n=4, n5=True):
    import itertools
    for n in range(1, max_n + 1):
        for states in itertools.product(list(_rank_states()), repeat=n):
            if sum(1 for s in states if s is not _DEAD and s[2]) <= 2:
                yield states
    if n5:
        for states in itertools.product(list(_rank_states()), repeat=5):
            alive = [s for s in states if s is not _DEAD]
            if sum(1 for s in alive if s[2]) <= 2 and {s[0] for s in alive} == {I, I + 1} \
                    and sum(1 for s in alive if s[1] == O.DIRTY) <= 1:
                yield states


def scenario_buffer(states):
    n = len(states)
    topo = dp_topo(n)
    rb = {}
    for r, s in enumerate(states):
        if s is _DEAD:
            continue
        v, ph, bad = s
        rb[r] = [rec(r, 0, v, phase=ph, content=(5000 + 10 * r + v) if bad else v)]
    return blobs(topo, rb) if rb else b"", sorted(rb)


def test_select_exhaustive_small_worlds():
    count = 0
    for states in small_world_scenarios():
        buf, healthy = scenario_buffer(states)
        st, vs, writers, reasons = _expected_single_group(states)
        sel = O.select(buf, healthy) if buf else O.select(b"", [])
        assert sel.status == st, states
        count += 1
        if st != O.OK:
            continue
        g = gsel(sel, 0)
        assert sel.v_star == vs and g.writers == writers, states
        assert g.status == (O.G_UNVERIFIED_SINGLE if len(writers) == 1 else O.G_OK), states
        assert dict(g.excluded) == reasons, states
    assert count > 10000          # 14,430 scenarios
