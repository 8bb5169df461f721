"""N>1 setup probe: P processes (the ranks of one box)
each pin the SAME /dev/shm image of G GiB the way jitc_register does it now:
one posix_fallocate under an flock, then every process registers 1 GiB
pieces on T threads concurrently (no lock).  Prints each process's time and
the wall time until all are pinned.   argv: GiB P T"""
import ctypes
import fcntl
import glob
import mmap
import os
import subprocess
import sys
import threading
import time

gib, P, T = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
role = sys.argv[4] if len(sys.argv) > 4 else "parent"
path = "/dev/shm/pin_probe4"
n = gib << 30
if role == "parent":
    t0 = time.time()
    ps = [subprocess.Popen([sys.executable, __file__, str(gib), str(P), str(T), f"child{i}"], stdout=subprocess.PIPE,
                           text=True) for i in range(P)]
    outs = [p.communicate()[0].strip() for p in ps]
    print("\n".join(outs))
    print(f"P={P} T={T} {gib} GiB each: all pinned after {time.time() - t0:.1f} s (incl. process start + CUDA init)")
    os.unlink(path)
    sys.exit(0)
import torch
lib = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                         "libcudart.so*"))[0])
torch.empty(1, device="cuda")
fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600)
t = time.time()
fcntl.flock(fd, fcntl.LOCK_EX)
if os.fstat(fd).st_size != n:
    os.ftruncate(fd, n)
os.posix_fallocate(fd, 0, n)
fcntl.flock(fd, fcntl.LOCK_UN)
t_fa = time.time() - t
m = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
piece = 1 << 30
pieces = list(range(0, n, piece))
rcs = []
lock = threading.Lock()


def work():
    while True:
        with lock:
            if not pieces:
                return
            a = pieces.pop()
        r = lib.cudaHostRegister(ctypes.c_void_p(addr + a), ctypes.c_size_t(min(piece, n - a)), ctypes.c_uint(3))
        rcs.append(r)


t = time.time()
ths = [threading.Thread(target=work) for _ in range(T)]
for x in ths:
    x.start()
for x in ths:
    x.join()
print(f"{role}: fallocate(+wait) {t_fa:.1f} s, register {time.time() - t:.1f} s, rcs={set(rcs)}", flush=True)
