import sys, os, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
from types import SimpleNamespace
A, _ = config("cfg2")
h = [torch.from_numpy(np.ascontiguousarray(x)).pin_memory() for x in (A.row_ptr.astype(np.int32), A.col, A.val)]
hA = SimpleNamespace(rows=A.rows, cols=A.cols, row_ptr=h[0], col=h[1], val=h[2])
plan = acs.Plan(stage_times=True)
P = int(sys.argv[1])
out = plan.multiply_host(hA, hA, pieces=P)
out = tuple(t for t in out)
bufs = (out[0], torch.empty(out[1].numel(), dtype=torch.int32).pin_memory(), torch.empty(out[2].numel(), dtype=torch.float64).pin_memory())
for _ in range(2):
    plan.multiply_host(hA, hA, out=bufs, pieces=P)
os.environ["ACS_HP_TRACE"] = "1"
torch.cuda.synchronize(); t = time.time()
plan.multiply_host(hA, hA, out=bufs, pieces=P)
print("wall ms", (time.time() - t) * 1e3, flush=True)
# raw D2H bandwidth
d = torch.empty(out[2].numel(), dtype=torch.float64, device="cuda")
torch.cuda.synchronize(); t = time.time(); bufs[2].copy_(d); torch.cuda.synchronize(); dt = time.time() - t
print("D2H GB/s", d.numel() * 8 / dt / 1e9)
t = time.time(); d.copy_(bufs[2]); torch.cuda.synchronize(); dt = time.time() - t
print("H2D GB/s", d.numel() * 8 / dt / 1e9)
print("--- size query (no copies)", flush=True)
try:
    plan.multiply_host(hA, hA, out=(bufs[0], bufs[1][:1], bufs[2][:1]), pieces=P)
except Exception as e:
    print("expected:", str(e)[:80])
