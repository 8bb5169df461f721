"""Why does pinning a big /dev/shm image take ~40 s?  One process, G GiB:
posix_fallocate, then T threads populate the page tables of disjoint ranges
with madvise(MADV_POPULATE_WRITE), then T threads cudaHostRegister 1 GiB
pieces; compared with registering without the populate step (a second,
fresh file).   argv: GiB T"""
import ctypes
import glob
import mmap
import os
import sys
import threading
import time

import torch

gib, T = int(sys.argv[1]), int(sys.argv[2])
lib = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib",
                                         "libcudart.so*"))[0])
libc = ctypes.CDLL("libc.so.6", use_errno=True)
libc.madvise.argtypes = [ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
torch.empty(1, device="cuda")
n = gib << 30
piece = 1 << 30


def run(tag, populate):
    path = f"/dev/shm/pin_probe5.{tag}.{os.getpid()}"
    fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600)
    os.ftruncate(fd, n)
    t = time.time()
    os.posix_fallocate(fd, 0, n)
    t_fa = time.time() - t
    m = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
    addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
    pieces = list(range(0, n, piece))

    def pool(fn):
        q = list(pieces)
        lk = threading.Lock()
        out = []

        def w():
            while True:
                with lk:
                    if not q:
                        return
                    a = q.pop()
                out.append(fn(a))
        ths = [threading.Thread(target=w) for _ in range(T)]
        [x.start() for x in ths]
        [x.join() for x in ths]
        return out
    t = time.time()
    rc_p = set(pool(lambda a: libc.madvise(addr + a, min(piece, n - a), 23))) if populate else None
    t_pop = time.time() - t
    t = time.time()
    rcs = set(pool(lambda a: lib.cudaHostRegister(ctypes.c_void_p(addr + a), ctypes.c_size_t(min(piece, n - a)),
                                                  ctypes.c_uint(3))))
    t_reg = time.time() - t
    print(f"{tag}: fallocate {t_fa:.1f} s, populate {t_pop:.1f} s (rc {rc_p}), register {t_reg:.1f} s (rc {rcs}) "
          f"-> {gib / (t_fa + t_pop + t_reg):.1f} GiB/s overall", flush=True)
    for a in pieces:
        lib.cudaHostUnregister(ctypes.c_void_p(addr + a))
    m.close()
    os.close(fd)
    os.unlink(path)


run("register-only", False)
run("populate+register", True)
