"""Pinned host->device copy bandwidth with 1-4 concurrent streams (620 MB in 36-MB chunks):
the ceiling for the e2e (host-buffer) path. python scripts/h2d_bw.py"""
import torch, time
torch.cuda.set_device(0)
N = 620 * 1024 * 1024
h = torch.empty(N, dtype=torch.uint8).pin_memory()
d = torch.empty(N, dtype=torch.uint8, device="cuda")
chunk = 36 << 20
def run(nstreams, reps=5):
    ss = [torch.cuda.Stream() for _ in range(nstreams)]
    best = 0
    for _ in range(reps):
        torch.cuda.synchronize(); t0 = time.perf_counter()
        for i, off in enumerate(range(0, N, chunk)):
            with torch.cuda.stream(ss[i % nstreams]):
                d[off:off + chunk].copy_(h[off:off + chunk], non_blocking=True)
        torch.cuda.synchronize(); t = time.perf_counter() - t0
        best = max(best, N / t / 1e9)
    return best
for ns in (1, 2, 3, 4):
    print(ns, "streams:", round(run(ns), 1), "GB/s")
