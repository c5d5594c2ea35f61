import torch, time
N = 1 << 28  # 1 GiB of int32
h = torch.empty(N, dtype=torch.int32).pin_memory()
d = torch.empty(N, dtype=torch.int32, device="cuda")
for streams in (1, 2, 4):
    ss = [torch.cuda.Stream() for _ in range(streams)]
    torch.cuda.synchronize()
    best = 0
    for rep in range(4):
        t0 = time.perf_counter()
        part = N // streams
        for i, s in enumerate(ss):
            with torch.cuda.stream(s):
                d[i*part:(i+1)*part].copy_(h[i*part:(i+1)*part], non_blocking=True)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        best = max(best, 4 * N / dt / 1e9)
    print("H2D streams", streams, "GB/s", round(best, 1))
# chunked sizes
for mb in (64, 256, 1024):
    n = mb << 18
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for i in range(0, N, n):
        d[i:i+n].copy_(h[i:i+n], non_blocking=True)
    torch.cuda.synchronize(); dt = time.perf_counter() - t0
    print("H2D chunk MB", mb, "GB/s", round(4 * N / dt / 1e9, 1))
hh = torch.empty(N, dtype=torch.int32).pin_memory()
torch.cuda.synchronize(); t0 = time.perf_counter()
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
with torch.cuda.stream(s2): hh.copy_(d, non_blocking=True)
torch.cuda.synchronize(); dt = time.perf_counter() - t0
print("duplex H2D+D2H 1 GiB each: s", round(dt, 4), "GB/s total", round(8 * N / dt / 1e9, 1))
