import torch, time
n = 8 * (1 << 30) // 4
h = torch.empty(n, dtype=torch.float32, pin_memory=True)
d = torch.empty(n, dtype=torch.float32, device='cuda')
h2 = torch.empty(n, dtype=torch.float32, pin_memory=True)
for nst in [1, 2, 4, 8]:
    streams = [torch.cuda.Stream() for _ in range(nst)]
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for rep in range(2):
        chunk = n // nst
        for i, s in enumerate(streams):
            with torch.cuda.stream(s):
                d[i*chunk:(i+1)*chunk].copy_(h[i*chunk:(i+1)*chunk], non_blocking=True)
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t0) / 2
    print(f"H2D {nst} streams: {n*4/dt/1e9:.1f} GB/s", flush=True)
# concurrent H2D + D2H
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
torch.cuda.synchronize(); t0 = time.perf_counter()
with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
with torch.cuda.stream(s2): h2.copy_(d, non_blocking=True)
torch.cuda.synchronize(); dt = time.perf_counter() - t0
print(f"H2D||D2H: {2*n*4/dt/1e9:.1f} GB/s total", flush=True)
t0 = time.perf_counter(); h2.copy_(d); torch.cuda.synchronize(); dt = time.perf_counter()-t0
print(f"D2H: {n*4/dt/1e9:.1f} GB/s")
