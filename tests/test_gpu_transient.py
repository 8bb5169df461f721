"""NEXT-2, transient in-place recovery (§4.2.1).

(a) GPU still usable, state kept in HBM: verify-only -- K1 over the live
    state against the last record detects any damage (else proceed).
(b) driver/context state suspect: copy the state to host, reset, copy back --
    here across a real process death: one process captures its own state
    (jitc_capture_local, no replica needed) and dies with os._exit; a NEW
    process restores from the surviving /dev/shm image, bit-exact against
    the oracle."""
import os
import shutil
import subprocess
import sys
import textwrap
import uuid

import numpy as np
import pytest
import torch

from oracle import oracle as O
from workloads import configs as W

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def J():
    from paper_conf_eurosys_guptakkvgkrs24_b200 import build, jitc
    build.build()
    return jitc


def _child(code: str):
    r = subprocess.run([sys.executable, "-c", textwrap.dedent(code)], cwd=ROOT, capture_output=True, text=True,
                       timeout=600)
    assert r.returncode == 0, r.stdout + r.stderr
    return r.stdout


def test_verify_only_in_place(J):
    from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
    g = W.scaled(W.c2(), 50000).groups[0]
    st = GroupState(g, 3)
    ctx = J.Context(device=0, chunk_bytes=1 << 20, staging_bytes=64 << 20, slot_bytes=16 << 20)
    ctx.register(0, J.REQUIRED, [0], st.table(), keepalive=st)
    last = ctx.fingerprint()               # the record of the last clean step
    assert ctx.verify(0, last) == 2**64 - 1
    J.inject_bitflip(st.ptrs[17], 3, 1)
    with pytest.raises(J.JitcError) as e:
        ctx.verify(0, last)
    lay = O.layout_of_group(g, 1 << 20)
    assert e.value.status == J.ECORRUPT and e.value.first_bad == (lay.offsets[17] + 3) >> 20
    ctx.close()


def test_host_round_trip_across_process_death(J):
    shm = f"/dev/shm/jitc-tr-{os.getpid()}-{uuid.uuid4().hex[:8]}"
    try:
        out = _child(f"""
            import os, sys
            sys.path.insert(0, {ROOT!r})
            from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
            from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
            from workloads import configs as W
            w = W.scaled(W.c2(), 20000)
            ctx = J.Context(device=0, chunk_bytes=1 << 20, image_dir={shm!r}, staging_bytes=64 << 20, slot_bytes=16 << 20)
            keep = []
            for g in w.groups:
                st = GroupState(g, w.seed); keep.append(st)
                ctx.register(g.group, g.policy, [0], st.table(), keepalive=st)
                ctx.mark(g.group, 9, J.CLEAN)
            s = ctx.capture_local()
            print("captured", s["image_bytes"], flush=True)
            os._exit(0)                       # dies without closing anything
        """)
        assert "captured" in out
        out = _child(f"""
            import sys
            sys.path.insert(0, {ROOT!r})
            import numpy as np, torch
            from oracle import oracle as O
            from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J
            from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState
            from workloads import configs as W
            w = W.scaled(W.c2(), 20000)
            ctx = J.Context(device=0, chunk_bytes=1 << 20, image_dir={shm!r}, staging_bytes=64 << 20, slot_bytes=16 << 20)
            sts = {{}}
            for g in w.groups:
                st = GroupState(g, w.seed, fill=False, shuffle_seed=7); st.scramble(); sts[g.group] = st
                ctx.register(g.group, g.policy, [0], st.table(), keepalive=st)
            ctx.restore(J.ALL_GROUPS, J.HOST)
            for g in w.groups:
                ctx.verify(g.group)
            torch.cuda.synchronize()
            for g in w.groups:
                for i, t in enumerate(g.tensors):
                    assert np.array_equal(sts[g.group].tensor_bytes(i).cpu().numpy(), O.gen_tensor_bytes(t, w.seed, g.group)), t.name
            print("restored-bit-exact", flush=True)
        """)
        assert "restored-bit-exact" in out
    finally:
        shutil.rmtree(shm, ignore_errors=True)
