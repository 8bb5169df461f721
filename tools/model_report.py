"""NEXT-3 report: the paper's wasted-time model (§5) evaluated with
the capture (o) and restore (r) times this library MEASURED on one B200
(bench.py JSON lines under profiles/), through the C ABI (jitc_waste_model).

    python tools/model_report.py profiles/r01_bench_c3_n1.json [minibatch_s]

f = 2 failures/day per 992 GPUs.  o_jit = 0 (no steady-state
work: jitc_mark is one stream-ordered 8-byte write per optimizer step).  The
minibatch time m is an input (not measured here; default 1 s).  Context for
the periodic baseline: a periodic checkpoint writes the full state, so its o
is taken as the same measured capture time (a lower bound for periodic)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J  # noqa: E402

F = 2 / (992 * 86400)


def main(path, m=1.0):
    line = json.loads(open(path).read().strip().splitlines()[-1])
    ph = line["phases_ms_median"]
    o = (ph["fingerprint"] + ph["select"] + ph["capture"] + ph["commit"]) / 1e3
    r = (ph["restore"] + ph["verify"]) / 1e3
    rows = []
    for N in (8, 1024, 8192, 16384):
        per = J.waste_model(J.MODEL_PERIODIC_OPTIMAL, N, F, o, r)
        jit = J.waste_model(J.MODEL_USER_JIT, N, F, o, r, m, 0.0)
        rows.append(dict(N=N, periodic_c_star_per_hr=round(per["c_opt"] * 3600, 3),
                         periodic_wf_pct=round(100 * per["w_f"], 4), user_jit_wf_pct=round(100 * jit["w_f"], 5)))
    out = dict(source=os.path.basename(path), workload=line["config"]["workload"], n_gpus_measured=line["n_gpus"],
               o_capture_s=round(o, 4), r_restore_s=round(r, 4), minibatch_s_assumed=m, f_per_gpu_per_s=F,
               rows=rows, note="o, r measured on B200 at N=1 (k=1 writer); with k-way sharding o shrinks ~k-fold")
    print(json.dumps(out, indent=1))
    return out


if __name__ == "__main__":
    res = main(sys.argv[1], float(sys.argv[2]) if len(sys.argv) > 2 else 1.0)
    tag = os.path.basename(sys.argv[1]).replace("bench", "model")
    json.dump(res, open(os.path.join(os.path.dirname(sys.argv[1]), tag), "w"), indent=1)
