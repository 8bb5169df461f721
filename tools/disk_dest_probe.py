"""Why is jitc_stage_in slower than the disk?  (round-2 probe, NEXT-4)
O_DIRECT preadv of one file in 64 MiB pieces by T threads into three kinds of
destination: one reused 64 MiB anonymous buffer, a G GiB anonymous mapping
(prefaulted), and a G GiB /dev/shm file mapping (prefaulted) -- the host
image's kind of memory.   argv: dir GiB threads"""
import mmap
import os
import subprocess
import sys
import threading
import time

d, gib, T = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
n, piece = gib << 30, 64 << 20
os.makedirs(d, exist_ok=True)
path = os.path.join(d, "probe.bin")
src = mmap.mmap(-1, piece)
src.write(os.urandom(1 << 20) * 64)
fd = os.open(path, os.O_WRONLY | os.O_CREAT | os.O_TRUNC | os.O_DIRECT, 0o600)
for off in range(0, n, piece):
    os.pwrite(fd, src, off)
os.fdatasync(fd)
os.close(fd)


def drop():
    subprocess.run(["sync"])
    try:
        with open("/proc/sys/vm/drop_caches", "w") as f:
            f.write("1\n")
    except OSError:
        pass


def read_into(view_of):
    drop()
    fd = os.open(path, os.O_RDONLY | os.O_DIRECT)

    def work(t):
        for off in range(t * piece, n, T * piece):
            os.preadv(fd, [view_of(off)], off)
    t0 = time.perf_counter()
    ths = [threading.Thread(target=work, args=(t,)) for t in range(T)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    dt = time.perf_counter() - t0
    os.close(fd)
    return n / dt / 1e9


small = mmap.mmap(-1, piece)
print(f"reused 64 MiB buffer : {read_into(lambda off: memoryview(small)):.2f} GB/s", flush=True)
anon = mmap.mmap(-1, n)
for off in range(0, n, 4096):
    anon[off] = 0
print(f"{gib} GiB anonymous   : {read_into(lambda off: memoryview(anon)[off:off + piece]):.2f} GB/s", flush=True)
del anon
sp = f"/dev/shm/disk_dest_probe.{os.getpid()}"
sfd = os.open(sp, os.O_RDWR | os.O_CREAT, 0o600)
os.ftruncate(sfd, n)
shm = mmap.mmap(sfd, n)
for off in range(0, n, 4096):
    shm[off] = 0
print(f"{gib} GiB /dev/shm    : {read_into(lambda off: memoryview(shm)[off:off + piece]):.2f} GB/s", flush=True)
print(f"reused 64 MiB buffer : {read_into(lambda off: memoryview(small)):.2f} GB/s", flush=True)
shm.close()
os.close(sfd)
os.unlink(sp)
os.unlink(path)
