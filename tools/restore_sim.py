"""Timing model of jitc_restore(HOST)'s executor with the IPC transport
(execute_plan in csrc/jitc_restore.cc), run on the library's own round plans
(jitc_restore_plan) for C3 at n = 1, 2, 4, 8: the projection behind DESIGN.md
§9 (a 1-GPU box cannot measure n > 1).

Per rank and round j of the plan:
  * host: before a round that writes a slot (H2D), wait until every reader
    consumed the round that last used the slot (IPC `consumed` >= j + 1 - S);
  * copy stream: wait for the slot's previous K3 on this rank, H2D the
    rank's block (host-link rate), then the compute stream posts `posted`;
  * host: wait for every peer's `posted` of round j;
  * compute stream: K3 over every block of the round -- the local block from
    HBM, the peers' blocks over NVLink (ingress-bound) -- then post `consumed`.
Rates: H2D 55.4 GB/s per GPU, K3 6.55 TB/s (r+w HBM), NVLink ingress 770 GB/s
(round-2 measurements; the guide's NVLink figure).  The fingerprint and
verify K1 passes (17.6 ms each at C3) and capture (L/n over each rank's D2H at
57.06 GB/s plus the 512 MiB first round's K2) complete the step.

    python tools/restore_sim.py
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

H2D, D2H, HBM, NVL = 55.4e9, 57.06e9, 6.55e12, 770e9
K1_S = 0.0176
C = 1 << 20


def host_restore(J, sel, n, staging=16 << 30, slot=8 << 30):
    plans = [J.restore_plan(sel, 0, J.HOST, list(range(n)), r, staging, slot) for r in range(n)]
    S, nr = plans[0]["slots"], plans[0]["n_rounds"]
    host = [0.0] * n
    copy = [0.0] * n
    comp = [0.0] * n
    free = [dict() for _ in range(n)]        # slot -> end of the last K3 that read it on this rank
    posted = [dict() for _ in range(n)]      # round -> time
    consumed = [dict() for _ in range(n)]
    for j in range(nr):
        sl = j % S
        ops = [[op for op in plans[r]["ops"] if op["round"] == j] for r in range(n)]
        for r in range(n):                                   # H2D + post
            h2d = [op for op in ops[r] if op["kind"] == "H2D"]
            if h2d and j >= S:
                host[r] = max([host[r]] + [consumed[q][j - S] for q in range(n) if q != r])
            t = max(host[r], copy[r], free[r].get(sl, 0.0))
            for op in h2d:
                t += op["bytes"] / H2D
            copy[r] = t if h2d else copy[r]
            posted[r][j] = max(comp[r], t)
        for r in range(n):                                   # K3 over all blocks, post consumed
            un = [op for op in ops[r] if op["kind"] == "UNPACK"]
            peers = {op["peer"] for op in un if op["peer"] != r}
            host[r] = max([host[r]] + [posted[p][j] for p in peers])
            remote = sum(op["b"] - op["a"] for op in un if op["peer"] != r)
            local = sum(op["b"] - op["a"] for op in un if op["peer"] == r)
            dur = max(2 * (local + remote) / HBM, remote / NVL) if un else 0.0
            t0 = max(host[r], comp[r], posted[r][j])
            comp[r] = t0 + dur
            consumed[r][j] = comp[r]
            free[r][sl] = comp[r]
    return max(comp + copy), nr, plans[0]["round_bytes"]


def main():
    from oracle import oracle as O
    from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
    from workloads import configs as W
    w = W.c3()
    rows = []
    for n in (1, 2, 4, 8):
        # one group image of C3's size (the REQUIRED + OPTIONAL groups restore one after another; their
        # round structure is the same, so one image of the summed size models the step)
        g = W.GroupSpec(0, W.REQUIRED, list(range(n)))
        for gg in w.groups:
            for t in gg.tensors:
                g.tensors.append(W.TensorSpec(f"{gg.group}.{t.name}", t.dtype, t.numel, t.kind, t.gen_id))
        lay = O.layout_of_group(g, C)
        import numpy as np
        d = np.zeros(lay.n_c, dtype=np.uint64)
        topo = [O.TopoEntry(0, O.REQUIRED, list(range(n)))]
        blobs = [O.encode_blob(r, topo, [O.Record(r, 0, O.REQUIRED, O.CLEAN, 3, lay.layout_hash, C, lay.L, d,
                                                  O.root(lay.layout_hash, d))]) for r in range(n)]
        st, sel = J.select_consistent_replica(b"".join(blobs), list(range(n)))
        t_res, nr, R = host_restore(J, sel, n)
        cap = (lay.L / n) / D2H + (512 << 20) / (HBM / 2)
        T_cap, T_res = K1_S + cap, t_res + K1_S
        rows.append({"n": n, "rounds": nr, "R_GiB": R / 2**30, "T_capture_s": round(T_cap, 3),
                     "T_restore_s": round(T_res, 3), "step_s": round(T_cap + T_res, 3),
                     "GBps": round(lay.L / (T_cap + T_res) / 1e9, 1)})
    print(json.dumps({"model": "tools/restore_sim.py (HOST restore, IPC executor on jitc_restore_plan)",
                      "workload": "C3 (128.5 GB)",
                      "rates_GBps": {"h2d": H2D / 1e9, "d2h": D2H / 1e9, "k3_rw": HBM / 1e9, "nvlink_in": NVL / 1e9},
                      "rows": rows}, indent=1))


if __name__ == "__main__":
    main()
