"""Timing model of jitc_capture_fanout's executor: why the
order in which a writer visits the movers' lanes matters, projected for the
C5 partitions (a 1-GPU box cannot measure it: every "link" is the same PCIe
link there).

The model follows fanout_group (csrc/jitc_capture.cc) with the IPC transport,
round by round, for one group:
  * writer, round j: its host waits until every reader posted `consumed` for
    round j - S (slot reuse), then its compute stream waits for the slot's
    previous D2H (when the writer is also a mover), runs K2 over the block and
    posts `posted`; if it moves its own block, the D2H follows on its copy
    stream.
  * mover, round j with a block: its host waits for the writer's `posted`, its
    compute stream waits for the slot's previous D2H on this mover, copies the
    block peer-to-peer out of the writer's staging (NVLink; the writer's
    egress is shared FIFO) and posts `consumed`; the D2H of the block follows
    on its copy stream.
  * mover, round j without a block: posts `consumed` in stream order (after
    whatever its compute stream still waits for).
Rates: K2 6.5 TB/s (r+w), NVLink 770 GB/s out of the writer, D2H 56.5 GB/s per
GPU (round-2 measurements; the guide's NVLink figure).  Block lists are built
here exactly as build_capture_plan does, in both orders; tests/
test_capture_plan.py checks the round-robin list against the library's plan.

    python tools/fanout_sim.py
"""
import json

HBM, NVL, D2H = 6.5e12 / 2, 770e9, 56.5e9       # K2 moves 2 bytes of HBM traffic per image byte
C = 1 << 20


def o5(n_c, k, s, L):
    return min(s * n_c // k * C, L), min((s + 1) * n_c // k * C, L)


def blocks_of(n_c, L, k, m, R, order):
    """Per writer s, its blocks (a, b, lane) in round order."""
    out = []
    for s in range(k):
        a, b = o5(n_c, k, s, L)
        lanes = []
        for q in range(m):
            la, lb = o5(n_c, m, q, L)
            x, y = max(a, la), min(b, lb)
            if x < y:
                lanes.append([(u, min(u + R, y), q) for u in range(x, y, R)])
        if order == "lane-major":
            out.append([bl for lane in lanes for bl in lane])
        else:
            most = max(len(lane) for lane in lanes)
            out.append([lane[i] for i in range(most) for lane in lanes if i < len(lane)])
    return out


def simulate(n_c, L, writers, movers, staging=16 << 30, slot=8 << 30, order="round-robin", S=2):
    k, m = len(writers), len(movers)
    R = min(slot, staging // (S * k)) // C * C
    bl = blocks_of(n_c, L, k, m, R, order)
    J = max(len(x) for x in bl)
    ranks = sorted(set(writers) | set(movers))
    host = {r: 0.0 for r in ranks}
    comp = {r: 0.0 for r in ranks}
    copy = {r: 0.0 for r in ranks}
    free = {r: {} for r in ranks}                  # slot -> time its last D2H on this rank ends
    egress = {w: 0.0 for w in writers}
    consumed = {r: {} for r in ranks}              # round -> time `consumed` is posted
    posted = {w: {} for w in writers}
    readers = {w: set() for w in writers}
    for s, w in enumerate(writers):
        for a, b, q in bl[s]:
            if movers[q] != w:
                readers[w].add(movers[q])
    for j in range(J):
        sl = j % S
        # writers pack
        for s, w in enumerate(writers):
            if j >= len(bl[s]):
                continue
            a, b, q = bl[s][j]
            if j >= S:
                host[w] = max([host[w]] + [consumed[r][j - S] for r in readers[w]])
            t0 = max(host[w], comp[w], free[w].get(sl, 0.0) if movers[q] == w else 0.0)
            comp[w] = t0 + (b - a) / HBM
            posted[w][j] = comp[w]
            if movers[q] == w:
                copy[w] = max(copy[w], comp[w]) + (b - a) / D2H
                free[w][sl] = copy[w]
        # movers receive + D2H
        for r in movers:
            mine = [(s, bl[s][j]) for s, w in enumerate(writers) if j < len(bl[s]) and movers[bl[s][j][2]] == r
                    and w != r]
            slot_wait = free[r].get(sl, 0.0) if mine else 0.0
            for s, (a, b, q) in mine:
                w = writers[s]
                host[r] = max(host[r], posted[w][j])
                t0 = max(host[r], comp[r], slot_wait, egress[w])
                comp[r] = t0 + (b - a) / NVL
                egress[w] = comp[r]
            consumed[r][j] = comp[r] if mine else max(comp[r], host[r])
            for s, (a, b, q) in mine:
                copy[r] = max(copy[r], comp[r]) + (b - a) / D2H
            if mine:
                free[r][sl] = copy[r]
    return max(max(copy.values()), max(comp.values())), J, R


def main():
    # C5: TP4 x DP2 Llama-3-70B-shaped (32 layers), rank 5 dead: partition 1 has k = 1
    L = 117_935_570_944
    n_c = -(-L // C)
    surv = [0, 1, 2, 3, 4, 6, 7]
    rows = []
    for name, writers in (("partition 1 (k = 1, writer rank 1)", [1]), ("partition 0 (k = 2, writers 0, 4)", [0, 4])):
        plain = L / len(writers) / D2H
        row = {"group": name, "image_GB": round(L / 1e9, 1), "plain_sharded_s": round(plain, 3)}
        for order in ("lane-major", "round-robin"):
            t, J, R = simulate(n_c, L, writers, surv, order=order)
            row[f"fanout_{order}_s"] = round(t, 3)
            row["rounds"], row["R_GiB"] = J, R / 2**30
        row["ideal_fanout_s"] = round(L / len(surv) / D2H, 3)
        rows.append(row)
    # the whole C5 capture: fan-out handles the groups one after another (every
    # survivor moves a lane of each); plain sharded capture runs all writers at
    # once, so it takes as long as the k = 1 partition's lone writer
    k1, k2 = rows
    whole = {"plain_sharded_s": round(max(k1["plain_sharded_s"], k2["plain_sharded_s"]), 3),
             "fanout_lane-major_s": round(k1["fanout_lane-major_s"] + 3 * k2["fanout_lane-major_s"], 3),
             "fanout_round-robin_s": round(k1["fanout_round-robin_s"] + 3 * k2["fanout_round-robin_s"], 3),
             "ideal_s": round(4 * L / len(surv) / D2H, 3),
             "note": "4 partitions: partition 1 with k = 1, partitions 0, 2, 3 with k = 2"}
    print(json.dumps({"model": "tools/fanout_sim.py (IPC executor semantics, S = 2 slots)",
                      "rates": {"K2_GBps": HBM * 2 / 1e9, "nvlink_egress_GBps": NVL / 1e9, "d2h_GBps": D2H / 1e9},
                      "rows": rows, "c5_whole_capture": whole}, indent=1))


if __name__ == "__main__":
    main()
