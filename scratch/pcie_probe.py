import time, torch, ctypes
n = 3_000_000_000 // 8
d = torch.ones(n, dtype=torch.float64, device="cuda")
h = torch.empty(n, dtype=torch.float64).pin_memory()
small_d = torch.zeros(16, dtype=torch.int64, device="cuda")
small_h = torch.zeros(16, dtype=torch.int64).pin_memory()
cs = torch.cuda.Stream(); ks = torch.cuda.Stream()
def probe(name, fn, reps=5):
    # start a big D2H on cs, then time fn on ks
    torch.cuda.synchronize()
    with torch.cuda.stream(cs):
        h.copy_(d, non_blocking=True)
    time.sleep(0.005)
    lat = []
    for _ in range(reps):
        t = time.time()
        with torch.cuda.stream(ks):
            fn()
        ks.synchronize()
        lat.append((time.time() - t) * 1e3)
    cs.synchronize()
    print(f"{name:30s}", " ".join(f"{x:7.2f}" for x in lat), "ms", flush=True)
def baseline(name, fn):
    torch.cuda.synchronize(); t = time.time()
    with torch.cuda.stream(ks): fn()
    ks.synchronize(); print(f"{name:30s} idle {(time.time()-t)*1e3:7.3f} ms")
k_add = lambda: small_d.add_(1)
k_d2h_small = lambda: small_h.copy_(small_d, non_blocking=True)
k_h2d_small = lambda: small_d.copy_(small_h, non_blocking=True)
for nm, f in (("kernel+sync", k_add), ("small D2H memcpy", k_d2h_small), ("small H2D memcpy", k_h2d_small)):
    baseline(nm, f)
    probe(nm, f)
