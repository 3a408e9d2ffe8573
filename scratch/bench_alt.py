import sys, os, time, json
alt = sys.argv[1] if len(sys.argv) > 1 else None
if alt: sys.path.insert(0, alt)
sys.path.insert(1, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
print("lib:", acs.SO_PATH, "THREADS", acs.const("THREADS"), "ITEMS", acs.const("ITEMS"))
from synth import config
cfg = sys.argv[2] if len(sys.argv) > 2 else "cfg2"
A, B = config(cfg)
dA = acs.DeviceCSR.from_host(A, "cuda"); dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda")
plan = acs.Plan(stage_times=True)
for _ in range(3): C = plan.multiply(dA, dB); del C
torch.cuda.synchronize()
ts = []
for _ in range(5):
    C = plan.multiply(dA, dB); st = plan.stage_times(); ts.append(st); del C
info = plan.info()
avg = {k: sum(t[k] for t in ts)/len(ts) for k in ts[0]}
tot = sum(avg.values())
print(cfg, "GFLOPS(stages)", 2*info["products"]/(tot*1e-3)/1e9, {k: round(v,3) for k,v in avg.items()})
print({k: info[k] for k in ("nblocks","nchunks","nshared","nmulti","npath","nsearch","chunk_elems")})
