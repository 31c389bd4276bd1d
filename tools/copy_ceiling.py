"""Practical streaming ceiling at the workload's array size (dev tool): torch copy / add
of C4-sized fp64 arrays back to back, CUDA events, GB/s of read+write bytes."""
import torch

dev = torch.device("cuda:0")
n = 1312 * 36 * 260  # one C4 array (padded), fp64
for nbuf, label in ((1, "84 MB"), (4, "4x84 MB chain")):
    a = [torch.randn(n, dtype=torch.float64, device=dev) for _ in range(nbuf + 1)]
    for op in ("copy", "add2"):
        def step():
            for i in range(nbuf):
                if op == "copy":
                    a[i + 1].copy_(a[i])
                else:
                    torch.add(a[i], a[(i + 2) % (nbuf + 1)], out=a[i + 1])
        for _ in range(5):
            step()
        s, e = torch.cuda.Event(True), torch.cuda.Event(True)
        torch.cuda.synchronize()
        s.record()
        reps = 50
        for _ in range(reps):
            step()
        e.record()
        torch.cuda.synchronize()
        t = s.elapsed_time(e) / reps / nbuf * 1e-3
        byts = n * 8 * (2 if op == "copy" else 3)
        print(f"{label:14s} {op:5s} {t*1e6:7.1f} us/launch  {byts / t / 1e9:7.0f} GB/s")
big = torch.randn(1 << 28, dtype=torch.float64, device=dev)
out = torch.empty_like(big)
for _ in range(3):
    out.copy_(big)
s, e = torch.cuda.Event(True), torch.cuda.Event(True)
torch.cuda.synchronize()
s.record()
for _ in range(10):
    out.copy_(big)
e.record()
torch.cuda.synchronize()
t = s.elapsed_time(e) / 10 * 1e-3
print(f"2 GB copy       {t*1e6:7.1f} us  {2 * big.numel() * 8 / t / 1e9:7.0f} GB/s")
