"""Does a concurrent PCIe copy-engine transfer slow an HBM-bound kernel?
Times a 256 MiB device-to-device copy (an SM kernel) alone and while a
D2H / H2D cudaMemcpyAsync of pinned memory runs on another stream."""
import torch, time
n = 256 << 20
a = torch.empty(n, dtype=torch.uint8, device="cuda"); b = torch.empty_like(a)
big = torch.empty(4 << 30, dtype=torch.uint8, device="cuda")
h = torch.empty(4 << 30, dtype=torch.uint8, pin_memory=True)
s_k, s_c = torch.cuda.Stream(), torch.cuda.Stream()
def timed(reps=20):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s_k):
        b.copy_(a)
        e0.record(s_k)
        for _ in range(reps): b.copy_(a)
        e1.record(s_k)
    e1.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3
torch.cuda.synchronize()
print("alone us/launch", timed())
for name, fn in [("d2h", lambda: h.copy_(big, non_blocking=True)), ("h2d", lambda: big.copy_(h, non_blocking=True))]:
    with torch.cuda.stream(s_c):
        fn()
    t = timed()
    print(name, "concurrent us/launch", t, "GB/s", 2 * n / t / 1e3)
    torch.cuda.synchronize()
print("alone again", timed())
