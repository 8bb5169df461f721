"""bench.py's reference arm (the oracle on the host cores) runs without a GPU
and prints the contract's JSON line (impl, metric, cpu_baseline, e2e)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "3", "--config", "C1", "--ref-every", "4"], capture_output=True, text=True, timeout=600,
                         cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    d = json.loads(out.stdout.strip().splitlines()[-1])
    assert d["impl"] == "reference" and d["unit"] == "GB/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["value"] == d["value"] and d["e2e"]["h2d_bytes_per_step"] == 0
    assert d["config"]["workload"].startswith("C1")


def test_cpu_baseline_d7_phases_and_digest_check():
    """bench.cpu_baseline on a small replica with an
    oracle-built 'committed image': per-phase times at nproc and 1 thread,
    coverage labels, s_to_recover, and the JF64-over-the-image check, which must
    flag exactly the chunk whose committed byte was flipped."""
    import sys
    sys.path.insert(0, ROOT)
    import numpy as np
    import bench
    from oracle import oracle as O
    from workloads import configs as W
    w = W.scaled(W.c2(world=1), 20000)
    C = 1 << 20
    committed, digests, recs, topo = {}, {}, [], []
    for g in w.groups:
        lay = O.layout_of_group(g, C)
        img = O.pack(O.gen_group(g, w.seed), lay)
        d = O.jf64(img, C, 0, lay.n_c)
        committed[g.group], digests[g.group] = img, d
        recs.append(O.Record(0, g.group, g.policy, O.CLEAN, 7, lay.layout_hash, C, lay.L, d, O.root(lay.layout_hash, d)))
        topo.append(O.TopoEntry(g.group, g.policy, [0]))
    blob = O.encode_blob(0, topo, recs)
    out = bench.cpu_baseline(w, 0, blob, committed, digests, every=4, every_1t=8)
    assert out["kind"] == "oracle" and out["unit"] == "GB/s" and out["value"] > 0 and out["cores"] >= 1
    assert set(out["phases_s"]) == {"layout", "pack", "jf64", "select", "shard", "unpack_verify"}
    assert out["s_to_recover"] > 0 and out["single_thread"]["cores"] == 1
    assert all(c["mismatch"] == 0 and c["coverage"] == "full" for c in out["digest_check"].values())
    committed[0] = committed[0].copy()
    committed[0][5 * C + 100] ^= 1
    out = bench.cpu_baseline(w, 0, blob, committed, digests, every=4, every_1t=8)
    assert out["digest_check"][0]["mismatch"] == 1 and out["digest_check"][1]["mismatch"] == 0
