"""Host-code sanitizers: the pure C-ABI functions -- replica
selection, blob / selection parsing, layout, shard rule, restore and capture
(fan-out) plans, the analytic model -- run under AddressSanitizer + UndefinedBehaviorSanitizer in
a child process that loads libjitc_asan.so (same sources, host code
instrumented), including malformed and truncated inputs."""
import os
import subprocess
import sys
import textwrap

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import random, struct, sys
sys.path.insert(0, {root!r})
import numpy as np
from oracle import oracle as O
from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
assert J.SO_PATH.endswith("libjitc_asan.so"), J.SO_PATH
rnd = random.Random(7)
n_ok = 0
for trial in range(400):
    world = rnd.randint(1, 6)
    topo = [O.TopoEntry(g, rnd.choice([0, 0, 1]), sorted(rnd.sample(range(world), rnd.randint(1, world))))
            for g in range(rnd.randint(1, 3))]
    rb = {{}}
    for r in range(world):
        recs = []
        for e in topo:
            if r in e.members:
                d = np.random.default_rng(rnd.randint(0, 5)).integers(0, 2**63, 7, dtype=np.int64).astype(np.uint64)
                recs.append(O.Record(r, e.group, e.policy, rnd.choice([0, 0, 1]), 3 + rnd.randint(0, 1), 99, 4096,
                                     7 * 4096, d, O.root(99, d)))
        rb[r] = recs
    buf = b"".join(O.encode_blob(r, topo, rb[r]) for r in rb)
    healthy = sorted(rnd.sample(range(world), rnd.randint(1, world)))
    st, sel = J.select_consistent_replica(buf, healthy)
    J.parse_selection(sel)
    if st == 0:
        n_ok += 1
        for e in topo:
            for mode in (0, 1):
                for me in range(world):
                    J.restore_plan(sel, e.group, mode, list(range(world)), me, 8 * 4096 * 4, 2 * 4096)
            movers = sorted(rnd.sample(healthy, rnd.randint(1, len(healthy))))
            for me in range(len(healthy)):
                try:
                    J.capture_plan(sel, e.group, movers, healthy, me, rnd.choice([4096, 8 * 4096 * 4]), 2 * 4096)
                except J.JitcError:
                    pass         # staging below 2 * k * C, or a writer outside the communicator
    # malformed inputs: truncations and bit flips must be rejected, never crash
    for cut in (1, 7, 31, 33, 64, len(buf) // 2, len(buf) - 1):
        if 0 < cut < len(buf):
            J.lib().jitc_select_consistent_replica(buf[:cut], cut, None, 0, None, 0, None)
            n = __import__("ctypes").c_size_t()
            J.lib().jitc_select_consistent_replica(buf[:cut], cut, (__import__("ctypes").c_int32 * 1)(0), 1, None, 0,
                                                   __import__("ctypes").byref(n))
    bad = bytearray(buf); bad[rnd.randrange(len(bad))] ^= 0xFF
    n = __import__("ctypes").c_size_t()
    J.lib().jitc_select_consistent_replica(bytes(bad), len(bad), (__import__("ctypes").c_int32 * 1)(0), 1, None, 0,
                                           __import__("ctypes").byref(n))
for k in range(1, 17):
    for s in range(k):
        J.shard_range(12345, k, s)
tabs = [("t%d" % i, rnd.randint(0, 5000), 1) for i in range(200)]
J.layout(tabs, 4096)
for kind in range(4):
    J.waste_model(kind, 1024, 2.3e-8, 5.0, 9.9, 0.4, 0.001, 0.01)
print("asan-ok", n_ok, flush=True)
"""


@pytest.mark.slow
def test_pure_functions_under_asan_ubsan():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build
    so = build.build(sanitize=True)
    libs = []
    for name in ("libasan.so", "libubsan.so"):
        p = subprocess.run(["gcc", f"-print-file-name={name}"], capture_output=True, text=True).stdout.strip()
        if not os.path.isabs(p):
            pytest.skip(f"{name} not available")
        libs.append(p)
    env = dict(os.environ, JITC_SO=so, LD_PRELOAD=" ".join(libs),
               ASAN_OPTIONS="detect_leaks=0:protect_shadow_gap=0:abort_on_error=1",
               UBSAN_OPTIONS="halt_on_error=1:print_stacktrace=1")
    r = subprocess.run([sys.executable, "-c", textwrap.dedent(CHILD.format(root=ROOT))], env=env, cwd=ROOT,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0 and "asan-ok" in r.stdout, (r.stdout + r.stderr)[-4000:]
