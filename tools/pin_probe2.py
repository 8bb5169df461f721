"""Two processes cudaHostRegister the same /dev/shm file CONCURRENTLY. argv: GiB"""
import ctypes, glob, mmap, os, subprocess, sys, time
gib = int(sys.argv[1]); role = sys.argv[2] if len(sys.argv) > 2 else "parent"
path = "/dev/shm/pin_probe2"
import torch
lib = ctypes.CDLL(glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib", "libcudart.so*"))[0])
torch.empty(1, device="cuda")
n = gib << 30
if role == "parent":
    fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600); os.ftruncate(fd, n)
    mode = sys.argv[4] if len(sys.argv) > 4 else "none"
    t = time.time()
    if mode == "fallocate":
        os.posix_fallocate(fd, 0, n)
    print("prep", mode, "%.1fs" % (time.time() - t), flush=True)
    os.close(fd)
    ps = [subprocess.Popen([sys.executable, __file__, str(gib), f"child{i}", "x", mode], stdout=subprocess.PIPE, text=True) for i in range(int(sys.argv[3]) if len(sys.argv) > 3 else 2)]
    for p in ps: print(p.communicate()[0].strip(), flush=True)
    os.unlink(path)
else:
    fd = os.open(path, os.O_RDWR)
    m = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
    addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
    t = time.time()
    import fcntl
    if sys.argv[4] == "flock":
        fcntl.flock(fd, fcntl.LOCK_EX)
    r = lib.cudaHostRegister(ctypes.c_void_p(addr), ctypes.c_size_t(n), ctypes.c_uint(3))
    if sys.argv[4] == "flock":
        fcntl.flock(fd, fcntl.LOCK_UN)
    print(role, gib, "GiB concurrent register rc", r, "in %.1fs" % (time.time() - t), flush=True)
