import sys, os, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
A, _ = config("cfg2")
dA = acs.DeviceCSR.from_host(A, "cuda")
plan = acs.Plan()
C = plan.multiply(dA, dA); torch.cuda.synchronize()
n = 400_000_000 // 8
d = torch.ones(n, dtype=torch.float64, device="cuda")
h = torch.empty(n, dtype=torch.float64).pin_memory()
cs = torch.cuda.Stream()
def d2h(k=8):
    torch.cuda.synchronize(); t = time.time()
    with torch.cuda.stream(cs):
        for _ in range(k): h.copy_(d, non_blocking=True)
    cs.synchronize(); return k * n * 8 / (time.time() - t) / 1e9
print("alone", d2h())
# concurrent with multiplies on the default stream
torch.cuda.synchronize()
t = time.time()
with torch.cuda.stream(cs):
    for _ in range(8): h.copy_(d, non_blocking=True)
for _ in range(3): C = plan.multiply(dA, dA)
cs.synchronize(); t1 = time.time() - t
print("concurrent total s", t1)
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record(cs)
with torch.cuda.stream(cs):
    for _ in range(8): h.copy_(d, non_blocking=True)
e1.record(cs)
for _ in range(3): C = plan.multiply(dA, dA)
torch.cuda.synchronize()
print("concurrent D2H GB/s", 8 * n * 8 / (e0.elapsed_time(e1) * 1e-3) / 1e9)
print("alone again", d2h())
