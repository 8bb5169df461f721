"""Can two processes cudaHostRegister the same /dev/shm file mapping?  argv: GiB"""
import ctypes, mmap, os, subprocess, sys, time
gib = int(sys.argv[1]); role = sys.argv[2] if len(sys.argv) > 2 else "parent"
path = "/dev/shm/pin_probe"
cudart = ctypes.CDLL("libcudart.so.12") if False else None
import torch  # loads cudart
from ctypes import c_void_p, c_size_t, c_uint
lib = ctypes.CDLL(os.path.join(os.path.dirname(torch.__file__), "lib", "libcudart.so.12")) if os.path.exists(os.path.join(os.path.dirname(torch.__file__), "lib", "libcudart.so.12")) else None
if lib is None:
    import glob
    cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "..", "nvidia", "cuda_runtime", "lib", "libcudart.so*"))
    lib = ctypes.CDLL(cands[0])
torch.cuda.init(); torch.empty(1, device="cuda")
n = gib << 30
fd = os.open(path, os.O_RDWR | os.O_CREAT, 0o600); os.ftruncate(fd, n)
m = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
addr = ctypes.addressof(ctypes.c_char.from_buffer(m))
t = time.time()
r = lib.cudaHostRegister(c_void_p(addr), c_size_t(n), c_uint(3))
print(role, gib, "GiB register rc", r, "in %.1fs" % (time.time() - t), flush=True)
if role == "parent":
    c = subprocess.run([sys.executable, __file__, str(gib), "child"], capture_output=True, text=True)
    print(c.stdout.strip(), c.stderr.strip()[-300:])
    os.unlink(path)
