"""Accumulator strategies on one workload: ms per multiply, ESC-stage parts, block counts,
and byte identity of C across strategies.

usage: python tools/strat_cmp.py [cfg2] [f64|f32] [adaptive,hash,dict] [reps]"""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
dt = np.float32 if len(sys.argv) > 2 and sys.argv[2] == "f32" else np.float64
strats = sys.argv[3].split(",") if len(sys.argv) > 3 else ["adaptive", "hash"]
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 10
A, B = config(cfg, dt)
dA = acs.DeviceCSR.from_host(A, "cuda", dt)
dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda", dt)
digests = {}
for strat in strats:
    plan = acs.Plan(stage_times=True, strategy=strat)
    for _ in range(3):
        C = plan.multiply(dA, dB)
        del C
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    st_all = []
    e0.record()
    for _ in range(reps):
        C = plan.multiply(dA, dB)
        del C
        st_all.append(plan.stage_times())
    e1.record()
    torch.cuda.synchronize()
    C = plan.multiply(dA, dB)
    h = hashlib.sha256()
    for t in (C.row_ptr, C.col, C.val):
        h.update(t.cpu().numpy().tobytes())
    digests[strat] = h.hexdigest()[:16]
    del C
    info = plan.info()
    med = {k: round(float(np.median([s[k] for s in st_all])), 3) for k in st_all[0]}
    print(json.dumps({"cfg": cfg, "dtype": str(np.dtype(dt)), "strategy": strat, "ms": e0.elapsed_time(e1) / reps,
                      "stages": med, "nblocks": info["nblocks"], 
                      "ndict": info["ndict_blocks"], "nhash": info["nhash_blocks"], "nrows": info["nrow_blocks"],
                      "sha": digests[strat]}), flush=True)
    plan.close()
print(json.dumps({"same_bytes": len(set(digests.values())) == 1, "digests": digests}))
