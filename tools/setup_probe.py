"""Setup-time probe (round 2): registers a config's state with a fresh
/dev/shm image, printing the library's populate / pin breakdown
(JITC_DEBUG_TIMING).   argv: config"""
import os
import shutil
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_eurosys_guptakkvgkrs24_b200 import jitc as J  # noqa: E402
from paper_conf_eurosys_guptakkvgkrs24_b200.state import GroupState  # noqa: E402
from workloads import configs as W  # noqa: E402

os.environ["JITC_DEBUG_TIMING"] = "1"
w = W.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else "C3"](world=1)
shm = f"/dev/shm/jitc-setup-probe-{os.getpid()}"
ctx = J.Context(device=0, chunk_bytes=1 << 20, staging_bytes=1 << 30, slot_bytes=256 << 20, image_dir=shm)
keep = []
t0 = time.perf_counter()
for g in w.groups:
    st = GroupState(g, w.seed)
    keep.append(st)
    torch.cuda.synchronize()
    t = time.perf_counter()
    ctx.register(g.group, g.policy, [0], st.table(), keepalive=st)
    print(f"group {g.group}: register {time.perf_counter() - t:.2f} s", flush=True)
print(f"setup {time.perf_counter() - t0:.2f} s  (JITC_PIN_FUSED={os.environ.get('JITC_PIN_FUSED', '0')})", flush=True)
ctx.close()
shutil.rmtree(shm, ignore_errors=True)
