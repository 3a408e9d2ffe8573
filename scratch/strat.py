"""Stage times of cfg2 (27-pt 128^3) for the adaptive (k_dict first) and hash strategies.
Usage: ACSPGEMM_LIB=... python scratch/strat.py [f64|f32] [n]"""
import sys, os, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import poisson3d_27pt
dt = np.float64 if (len(sys.argv) < 2 or sys.argv[1] == "f64") else np.float32
n = int(sys.argv[2]) if len(sys.argv) > 2 else 128
A = poisson3d_27pt(n)
dA = acs.DeviceCSR.from_host(A, "cuda", dt)
for strat in (sys.argv[3].split(",") if len(sys.argv) > 3 else ("adaptive", "hash")):
    plan = acs.Plan(stage_times=True, strategy=strat)
    for _ in range(3): C = plan.multiply(dA, dA); del C
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    hs, ds = [], []
    e0.record()
    for _ in range(10):
        C = plan.multiply(dA, dA); del C
        st = plan.stage_times(); hs.append(st["HASH"]); ds.append(st["DICT"])
    e1.record(); torch.cuda.synchronize()
    info = plan.info()
    print(json.dumps({"lib": os.path.basename(os.environ.get("ACSPGEMM_LIB", "libacspgemm.so")), "dtype": str(np.dtype(dt)),
                      "strategy": strat, "ms": e0.elapsed_time(e1) / 10, "HASH": float(np.median(hs)), "DICT": float(np.median(ds)),
                      "ndict": info["ndict_blocks"], "nhash": info["nhash_blocks"], "nblocks": info["nblocks"]}), flush=True)
    plan.close()
