"""Setup-cost probe for the shared host image: how long
does pinning a /dev/shm image take as ONE cudaHostRegister vs T concurrent
registrations of disjoint pieces (after posix_fallocate), and is the device
alias of registered memory the host address (so pieces stay one contiguous
device range)?   argv: GiB [threads ...]"""
import ctypes
import glob
import mmap
import os
import sys
import threading
import time

import torch

lib = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                         "libcudart.so*"))[0])
gib = int(sys.argv[1])
threads = [int(x) for x in sys.argv[2:]] or [1, 4, 8, 16]
n = gib << 30
path = f"/dev/shm/pin_probe3.{os.getpid()}"
torch.empty(1, device="cuda")
v = ctypes.c_int()
lib.cudaDeviceGetAttribute(ctypes.byref(v), ctypes.c_int(91), ctypes.c_int(0))  # CanUseHostPointerForRegisteredMem
print(f"canUseHostPointerForRegisteredMem={v.value}", flush=True)
fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600)
os.ftruncate(fd, n)
t = time.time()
os.posix_fallocate(fd, 0, n)
print(f"posix_fallocate {gib} GiB: {time.time() - t:.2f} s", flush=True)
m = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
for T in threads:
    piece = (n // T + (2 << 20) - 1) // (2 << 20) * (2 << 20)
    rcs = [None] * T

    def reg(i):
        a = i * piece
        b = min(n, a + piece)
        if b > a:
            rcs[i] = lib.cudaHostRegister(ctypes.c_void_p(addr + a), ctypes.c_size_t(b - a), ctypes.c_uint(3))

    t = time.time()
    ths = [threading.Thread(target=reg, args=(i,)) for i in range(T)]
    for x in ths:
        x.start()
    for x in ths:
        x.join()
    dt = time.time() - t
    dp = ctypes.c_void_p()
    lib.cudaHostGetDevicePointer(ctypes.byref(dp), ctypes.c_void_p(addr + n // 2), 0)
    same = dp.value == addr + n // 2
    print(f"T={T:2d}: register {gib} GiB in {dt:.2f} s = {gib / dt:.1f} GiB/s rcs={set(rcs)} dev==host:{same}",
          flush=True)
    # a device copy across a piece boundary must work through the alias
    if T > 1:
        d = torch.empty(4 << 20, dtype=torch.uint8, device="cuda")
        r = lib.cudaMemcpy(ctypes.c_void_p(d.data_ptr()), ctypes.c_void_p(addr + piece - (2 << 20)),
                           ctypes.c_size_t(4 << 20), 4)
        print(f"   copy across piece boundary rc={r}", flush=True)
    t = time.time()
    for i in range(T):
        a = i * piece
        if a < n:
            lib.cudaHostUnregister(ctypes.c_void_p(addr + a))
    print(f"   unregister {time.time() - t:.2f} s", flush=True)
m.close()
os.close(fd)
os.unlink(path)
