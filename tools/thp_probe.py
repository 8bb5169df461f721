"""Would transparent huge pages help the shared /dev/shm image?  (round-2 probe)

Prints the box's THP settings for shmem, then for a G GiB /dev/shm file, with
and without madvise(MADV_HUGEPAGE) before the parallel MADV_POPULATE_WRITE:
populate time, ShmemHugePages gained, parallel cudaHostRegister time of 1 GiB
pieces, and D2H / H2D copy-engine bandwidth over the registered range
(64 MiB pieces, best of 3).   argv: GiB threads"""
import ctypes
import glob
import mmap
import os
import sys
import threading
import time

import torch

gib, T = int(sys.argv[1]), int(sys.argv[2])
cudart = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                            "libcudart.so*"))[0])
libc = ctypes.CDLL("libc.so.6", use_errno=True)
libc.madvise.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
libc.mmap.restype = ctypes.c_void_p
libc.mmap.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_long]
cudart.cudaHostRegister.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint]
cudart.cudaHostUnregister.argtypes = [ctypes.c_void_p]
MADV_HUGEPAGE, MADV_POPULATE_WRITE = 14, 23
PIECE = 1 << 30


def cat(p):
    try:
        return open(p).read().strip()
    except OSError as e:
        return f"<{e}>"


def meminfo(key):
    for line in open("/proc/meminfo"):
        if line.startswith(key + ":"):
            return int(line.split()[1]) * 1024
    return -1


print("THP enabled:", cat("/sys/kernel/mm/transparent_hugepage/enabled"))
print("THP shmem_enabled:", cat("/sys/kernel/mm/transparent_hugepage/shmem_enabled"))
print("THP defrag:", cat("/sys/kernel/mm/transparent_hugepage/defrag"))
print("nr_hugepages:", cat("/proc/sys/vm/nr_hugepages"))
print("/dev/shm mount:", [l.strip() for l in open("/proc/mounts") if " /dev/shm " in l])
print("kernel:", os.uname().release, " cpus:", os.cpu_count())
torch.empty(1, device="cuda")
n = gib << 30


def parallel(fn, count):
    ths, errs = [], []

    def work(i0):
        for i in range(i0, count, T):
            r = fn(i)
            if r:
                errs.append(r)
    for t in range(T):
        th = threading.Thread(target=work, args=(t,))
        th.start()
        ths.append(th)
    for th in ths:
        th.join()
    return errs


def bw(ptr, dev, direction):
    piece = 64 << 20
    s = torch.cuda.Stream()
    best = 0.0
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record()
            for off in range(0, dev.numel(), piece):
                kind = 2 if direction == "d2h" else 1   # cudaMemcpyDeviceToHost / HostToDevice
                dst, src = (ptr + off, dev.data_ptr() + off) if direction == "d2h" else (dev.data_ptr() + off, ptr + off)
                cudart.cudaMemcpyAsync(ctypes.c_void_p(dst), ctypes.c_void_p(src), ctypes.c_size_t(piece),
                                       ctypes.c_int(kind), ctypes.c_void_p(s.cuda_stream))
            e1.record()
        s.synchronize()
        best = max(best, dev.numel() / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    return best


cudart.cudaMemcpyAsync.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int, ctypes.c_void_p]


def run(tag, huge):
    path = f"/dev/shm/thp_probe.{tag}.{os.getpid()}"
    fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600)
    os.ftruncate(fd, n)
    p = libc.mmap(None, n, mmap.PROT_READ | mmap.PROT_WRITE, mmap.MAP_SHARED, fd, 0)
    h0 = meminfo("ShmemHugePages")
    rc_h = libc.madvise(p, n, MADV_HUGEPAGE) if huge else 0
    err_h = ctypes.get_errno() if rc_h else 0
    t = time.time()
    errs = parallel(lambda i: libc.madvise(p + i * PIECE, PIECE, MADV_POPULATE_WRITE), n // PIECE)
    t_pop = time.time() - t
    h1 = meminfo("ShmemHugePages")
    t = time.time()
    rcs = parallel(lambda i: cudart.cudaHostRegister(p + i * PIECE, PIECE, 0), n // PIECE)
    t_reg = time.time() - t
    dev = torch.empty(min(n, 4 << 30), dtype=torch.uint8, device="cuda")
    d2h = bw(p, dev, "d2h")
    h2d = bw(p, dev, "h2d")
    t = time.time()
    parallel(lambda i: cudart.cudaHostUnregister(p + i * PIECE), n // PIECE)
    t_unreg = time.time() - t
    print(f"{tag:10s} madvise(HUGEPAGE) rc={rc_h} errno={err_h}  populate {gib} GiB in {t_pop:6.2f} s "
          f"({gib / t_pop:5.1f} GiB/s, errs={len(errs)})  ShmemHugePages +{(h1 - h0) / 2**30:.1f} GiB  "
          f"register {t_reg:6.2f} s ({gib / t_reg:5.1f} GiB/s, rcs={set(rcs) or {0}})  unregister {t_unreg:.2f} s  "
          f"D2H {d2h:.2f} GB/s  H2D {h2d:.2f} GB/s", flush=True)
    os.close(fd)
    os.unlink(path)
    del dev


run("4k-pages", False)
run("thp", True)
run("4k-pages", False)
run("thp", True)
