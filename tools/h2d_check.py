import torch, time
n = 1 << 27  # 1 GiB of doubles
h = torch.empty(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device='cuda')
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for _ in range(3): d.copy_(h, non_blocking=True)
torch.cuda.synchronize()
for trial in range(2):
    t0 = time.perf_counter()
    for _ in range(5): d.copy_(h, non_blocking=True)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    print("1 stream GB/s", 5 * 8 * n / (t1 - t0) / 1e9)
    t0 = time.perf_counter()
    for _ in range(5):
        with torch.cuda.stream(s1): d[: n // 2].copy_(h[: n // 2], non_blocking=True)
        with torch.cuda.stream(s2): d[n // 2:].copy_(h[n // 2:], non_blocking=True)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    print("2 streams GB/s", 5 * 8 * n / (t1 - t0) / 1e9)
    t0 = time.perf_counter()
    ch = n // 8
    for _ in range(5):
        for k in range(8):
            with torch.cuda.stream(s1 if k % 2 == 0 else s2): d[k*ch:(k+1)*ch].copy_(h[k*ch:(k+1)*ch], non_blocking=True)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    print("8 chunks/2 streams GB/s", 5 * 8 * n / (t1 - t0) / 1e9)
