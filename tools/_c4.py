import sys, os, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import poisson3d_7pt, aggregation_prolongator
A = poisson3d_7pt(256); P = aggregation_prolongator(256)
dA = acs.DeviceCSR.from_host(A, "cuda"); dP = acs.DeviceCSR.from_host(P, "cuda")
for rep in range(2):
  for mode in ("exact", "bound"):
    plan = acs.Plan(pool_mode=mode, stage_times=True)
    for _ in range(3): C = plan.multiply(dA, dP); del C
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): C = plan.multiply(dA, dP); del C
    e1.record(); torch.cuda.synchronize()
    print(json.dumps({"mode": mode, "ms": e0.elapsed_time(e1) / 10, "st": {k: round(v, 3) for k, v in plan.stage_times().items()}}), flush=True)
    plan.close()
