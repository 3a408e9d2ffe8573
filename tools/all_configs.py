"""Every BASELINE config: ms, GFLOPS, per-stage times, path counters (one JSON line each).  usage: python tools/all_configs.py [cfg1,cfg2,cfg3,cfg5,cfg4]"""
import sys, os, time, json
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config, poisson3d_7pt, aggregation_prolongator, transpose
def run(name, A, B, dt, reps=5):
    dA = acs.DeviceCSR.from_host(A, "cuda", dt); dB = dA if B is A else acs.DeviceCSR.from_host(B, "cuda", dt)
    plan = acs.Plan(stage_times=True)
    for _ in range(3): C = plan.multiply(dA, dB); del C
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps): C = plan.multiply(dA, dB); del C
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    info = plan.info(); st = plan.stage_times()
    out = {"workload": name, "dtype": str(np.dtype(dt)), "ms_per_multiply": ms, "GFLOPS": 2 * info["products"] / (ms * 1e-3) / 1e9,
           "products": info["products"], "nnz_c": info["nnz_c"], "stages_ms": {k: round(v, 3) for k, v in st.items()},
           "nshared": info["nshared"], "nmulti": info["nmulti"], "npath": info["npath"], "nsearch": info["nsearch"], "nhash": info["nhash_blocks"], "nblocks": info["nblocks"]}
    print(json.dumps(out), flush=True)
    plan.close(); del dA, dB; torch.cuda.empty_cache()
CFGS = sys.argv[1].split(",") if len(sys.argv) > 1 else ["cfg1", "cfg2", "cfg3", "cfg5", "cfg4"]
for cfg in [c for c in CFGS if c != "cfg4"]:
    for dt in ([np.float64, np.float32] if cfg != "cfg1" else [np.float64]):
        A, B = config(cfg, dt)
        run(cfg, A, B if cfg == "cfg5" else A, dt)
if "cfg4" not in CFGS: sys.exit(0)
A = poisson3d_7pt(256); P = aggregation_prolongator(256)
run("cfg4a A*P", A, P, np.float64)
# cfg4b: R·(AP) with AP from the GPU (integer values: exact), R = P^T
from synth import CSR
dA = acs.DeviceCSR.from_host(A, "cuda"); dP = acs.DeviceCSR.from_host(P, "cuda")
AP = acs.Plan().multiply(dA, dP)
rp, col, val = AP.to_numpy()
del AP, dA, dP
torch.cuda.empty_cache()
run("cfg4b R*AP", transpose(P), CSR(A.rows, P.cols, rp, col, val), np.float64)
