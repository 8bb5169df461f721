"""Summarise ncu outputs brought back under gpurun_out/ into profiles/ (tracked).

    python tools/summarize_profiles.py <tag> <launches.csv> <full.ncu-rep>

Writes profiles/<tag>_launches.txt (per-kernel launch count, device time,
share, DRAM bytes from the `--metrics gpu__time_duration.sum,...` pass),
profiles/<tag>_ncu_full.txt (per-launch DRAM / SM metrics of the `--set full`
capture) and updates profiles/traffic.json (DRAM bytes per image byte of each
kernel, used by bench.py's roofline.traffic).
"""
import collections
import csv
import gzip
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")
KIND = {"seg_kernel<1>": "K1_digest", "seg_kernel<2>": "K2_pack_digest", "seg_kernel<3>": "K3_unpack_verify"}
MUL = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
TMUL = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3}


def short(name):
    for k, v in KIND.items():
        if k in name:
            return v
    return name.split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "")


def launches(path, tag):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, ui, idi = (h.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
    per = collections.defaultdict(dict)
    for r in rows[hi + 1:]:
        if len(r) > vi:
            per[(r[idi], r[ki])][r[mi]] = (float(r[vi].replace(",", "")), r[ui])
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for (_, k), m in per.items():
        a = agg[short(k)]
        a[0] += 1
        t = m["gpu__time_duration.sum"]
        a[1] += t[0] * TMUL.get(t[1], 1.0)
        for key, idx in (("dram__bytes_read.sum", 2), ("dram__bytes_write.sum", 3)):
            if key in m:
                a[idx] += m[key][0] * MUL[m[key][1]]
    tot = sum(a[1] for a in agg.values())
    ours = sum(a[1] for k, a in agg.items() if k in KIND.values())
    out = io.StringIO()
    out.write(f"# {tag}: ncu launch list (--metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum"
              f" --clock-control none); cold-cache, serialised -> compare SHARES\n")
    out.write(f"# source: {os.path.basename(path)} ({len(per)} launches)\n")
    out.write(f"{'kernel':28s} {'launches':>8s} {'total_us':>12s} {'share_all':>9s} {'share_path':>10s} {'us/launch':>10s} {'dram_rd_GB':>10s} {'dram_wr_GB':>10s}\n")
    for k, a in sorted(agg.items(), key=lambda x: -x[1][1]):
        sp = a[1] / ours if k in KIND.values() else float("nan")
        out.write(f"{k[:28]:28s} {a[0]:8d} {a[1]:12.1f} {a[1] / tot:9.3f} {sp:10.3f} {a[1] / a[0]:10.1f} "
                  f"{a[2] / 1e9:10.3f} {a[3] / 1e9:10.3f}\n")
    open(os.path.join(PROF, f"{tag}_launches.txt"), "w").write(out.getvalue())
    with open(path, "rb") as f, gzip.open(os.path.join(PROF, f"{tag}_launches.csv.gz"), "wb") as g:
        shutil.copyfileobj(f, g)
    print(out.getvalue())


def full(rep, tag):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    want = ["Kernel Name", "launch__grid_size", "launch__registers_per_thread", "gpu__time_duration.sum",
            "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__cycles_active.avg", "gpc__cycles_elapsed.max",
            "smsp__inst_executed.sum"]
    idx = [hdr.index(w) if w in hdr else None for w in want]
    out = io.StringIO()
    out.write(f"# {tag}: ncu --set full --clock-control none --import-source on (source: {os.path.basename(rep)})\n")
    out.write("# columns: " + ", ".join(f"{w} [{units[i] if i is not None else '-'}]" for w, i in zip(want, idx)) + "\n")
    traffic = {}
    for r in rows[2:]:
        vals = [r[i] if i is not None else "" for i in idx]
        vals[0] = short(vals[0])
        out.write(" | ".join(vals) + "\n")
        k = vals[0]
        if k in KIND.values():
            t_ms = float(vals[3]) * TMUL.get(units[idx[3]], 1.0) / 1e3
            rd = float(vals[4]) * MUL[units[idx[4]]]
            wr = float(vals[5]) * MUL[units[idx[5]]]
            traffic.setdefault(k, []).append((rd + wr, t_ms))
    open(os.path.join(PROF, f"{tag}_ncu_full.txt"), "w").write(out.getvalue())
    print(out.getvalue())
    return traffic


if __name__ == "__main__":
    tag, lcsv, rep = sys.argv[1:4]
    os.makedirs(PROF, exist_ok=True)
    launches(lcsv, tag)
    tr = full(rep, tag)
    # image bytes per launch of the profiled launches (tools/prof_kernels.py: 2 GiB rounds)
    image_bytes = {k: float(os.environ.get("IMG_" + k, 0)) for k in tr}
    tj = os.path.join(PROF, "traffic.json")
    cur = json.load(open(tj)) if os.path.exists(tj) else {}
    for k, v in tr.items():
        big = max(v)          # the largest (full-round) launch
        ib = image_bytes.get(k) or None
        if ib:
            cur[k] = {"dram_bytes": big[0], "image_bytes": ib, "ms": big[1], "source": f"{tag}_ncu_full.txt"}
    json.dump(cur, open(tj, "w"), indent=1)
