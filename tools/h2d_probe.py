"""Pinned host -> device copy rate on 1, 2 and 4 concurrent streams (1 GiB, torch
copies): the link the cold path (e2e) is measured against.  B200 box, this round:
52.0 / 52.2 / 52.3 GB/s -- one stream already saturates it."""
import torch, time
N = 1 << 30
h = torch.empty(N, dtype=torch.uint8).pin_memory()
d = torch.empty(N, dtype=torch.uint8, device="cuda")
for k in (1, 2, 4):
    ss = [torch.cuda.Stream() for _ in range(k)]
    for rep in range(3):
        torch.cuda.synchronize()
        t = time.perf_counter()
        ch = N // k
        for i, s in enumerate(ss):
            with torch.cuda.stream(s):
                d[i*ch:(i+1)*ch].copy_(h[i*ch:(i+1)*ch], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t
    print(k, "streams", round(N / dt / 1e9, 1), "GB/s")
