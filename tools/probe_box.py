"""Phase-0 probe of a GPU box: host RAM, shm, cores, PCIe, D2H/H2D bandwidth."""
import os, subprocess, time, json
def sh(c):
    try: return subprocess.run(c, shell=True, capture_output=True, text=True, timeout=120).stdout
    except Exception as e: return str(e)
out = {}
out["nproc"] = sh("nproc").strip()
out["free"] = sh("free -g")
out["shm"] = sh("df -h /dev/shm /tmp")
out["lscpu"] = sh("lscpu | head -30")
out["numa"] = sh("numactl -H 2>/dev/null | head; cat /sys/class/drm/*/device/numa_node 2>/dev/null")
out["smi"] = sh("nvidia-smi --query-gpu=index,name,pci.bus_id,pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,memory.total,clocks.max.sm --format=csv")
out["topo"] = sh("nvidia-smi topo -m")
import torch
dev = torch.device("cuda:0")
res = {}
for gb in [1, 4]:
    n = gb << 30
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
    s = torch.cuda.Stream()
    for name, fn in [("d2h", lambda: h.copy_(d, non_blocking=True)), ("h2d", lambda: d.copy_(h, non_blocking=True))]:
        with torch.cuda.stream(s):
            fn(); torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(s)
            for _ in range(3): fn()
            e1.record(s); torch.cuda.synchronize()
        res[f"{name}_{gb}GiB_GBps"] = 3 * n / (e0.elapsed_time(e1) * 1e-3) / 1e9
    del d, h
n = 8 << 30
a = torch.empty(n, dtype=torch.uint8, device=dev); b = torch.empty_like(a)
b.copy_(a); torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(3): b.copy_(a)
e1.record(); torch.cuda.synchronize()
res["d2d_copy_GBps_rw"] = 3 * 2 * n / (e0.elapsed_time(e1) * 1e-3) / 1e9
del a, b
# big pinned alloc timing
t = time.time(); h = torch.empty(24 << 30, dtype=torch.uint8, pin_memory=True); res["pin_24GiB_s"] = time.time() - t; del h
out["bw"] = res
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
