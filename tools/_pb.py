import sys, os, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
A, B = config("cfg2", np.float64)
dA = acs.DeviceCSR.from_host(A, "cuda", np.float64)
for mode in ("exact", "bound"):
    plan = acs.Plan(pool_mode=mode)
    for _ in range(3): C = plan.multiply(dA, dA); del C
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): C = plan.multiply(dA, dA); del C
    e1.record(); torch.cuda.synchronize()
    i = plan.info()
    print(json.dumps({"mode": mode, "ms": e0.elapsed_time(e1) / 10, "pool_bytes": i.get("pool_bytes"), "chunk_elems": i["chunk_elems"], "nhash": i["nhash_blocks"], "ndeferred": i.get("ndeferred_blocks")}), flush=True)
    plan.close()
