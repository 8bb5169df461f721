"""bench.py's N > 1 path (torchrun, one process per rank, gloo rendezvous,
the library's communicator, k = N sharded capture, N-way HOST restore,
max-over-ranks timing) run functionally on one B200 over either transport:
JITC_BENCH_SHARE_GPU puts every rank on GPU 0 (and, for NCCL, gives each rank
its own NCCL_HOSTID so NCCL accepts two ranks on one device); the numbers are
not a measurement."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("transport", ["ipc", "nccl"])
def test_bench_two_ranks_one_gpu(transport):
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ, JITC_BENCH_SHARE_GPU="1")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", str(port), "bench.py", "--gpus", "2",
                        "--steps", "3", "--warmup", "3", "--config", "C1", "--no-cpu-baseline", "--staging", "256",
                        "--slot", "64", "--hang-ctas", "0", "--transport", transport],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["writers_k"] == {"0": 2} and d["config"]["transport"] == transport
    assert d["value"] > 0 and d["gpu_launches"] > 0
    pr = d["peer_restore"]           # the last rank rebuilt from the other's live HBM (PEER mode)
    assert pr["replacement"] == 1 and pr["writers_k"] == {"0": 1} and not pr["replacement_passed_selection"]
    assert pr["replacement_ingress_bytes"] == d["config"]["image_bytes"]


def test_bench_n1_json_contract():
    """bench.py at N = 1 (C1, small rounds): one JSON line carrying every key
    the driver and the judge read."""
    r = subprocess.run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3", "--config", "C1",
                        "--staging", "256", "--slot", "64", "--hang-ctas", "8"],
                       cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["n_gpus"] == 1 and d["steps"] == 3 and d["value"] > 0 and d["gpu_launches"] > 0
    assert d["config"]["workload"].startswith("C1")
    rf = d["roofline"]
    assert rf["bound"] == "hbm" and rf["unit"] == "GB/s" and 0 < rf["frac"] and rf["peak"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["watchdog_on_hang"]["fired"] and d["under_hang"]["value_GBps"] > 0
    assert "calibrated" in d["host_link_roofline"]
