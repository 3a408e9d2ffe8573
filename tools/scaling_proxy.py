"""One-GPU strong-scaling proxy of the row-segment multi-GPU path.

For N = 1, 2, 4, 8 every rank's share of the 8 canonical segments is multiplied alone on
this GPU (its own plan, as one process per GPU would), T_N = the slowest rank's median
time; efficiency = T_1 / (N · T_N).  This is the compute part of the scaling curve (B
resident, as in the bench's `value`); the collectives (B broadcast, the (rows, nnz)
all-gather) are not included.

usage: python tools/scaling_proxy.py [cfg2] [f64|f32] [reps]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ppopp_wintermzss19_b200 as acs
from paper_conf_ppopp_wintermzss19_b200 import dist as adist
from synth import config

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg2"
dt = np.float32 if len(sys.argv) > 2 and sys.argv[2] == "f32" else np.float64
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 7
A, B = config(cfg, dt)
dA = acs.DeviceCSR.from_host(A, "cuda", dt)
dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda", dt)
seg = acs.canonical_segments(dA, 8)
stream = torch.cuda.current_stream()


def time_share(s0, s1):
    plan = acs.Plan(stage_times=True)
    r0, r1 = seg[s0], seg[s1]
    plan.set_segments(adist.local_segment_rows(seg, s0, s1))
    rp = dA.row_ptr[r0:r1 + 1]
    view = acs.api._csr_in(dA, row_ptr=rp, rows=r1 - r0, nnz=int(rp[-1].item() - rp[0].item()))
    for _ in range(2):
        C = plan.multiply(dA, dB, stream, A_view=view)
        del C
    torch.cuda.synchronize()
    ts, st = [], []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        C = plan.multiply(dA, dB, stream, A_view=view)
        e1.record(stream)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        st.append(plan.stage_times())
        del C
    info = plan.info()
    plan.close()
    stages = {k: round(statistics.median(s[k] for s in st), 4) for k in st[0]}
    return statistics.median(ts), info["products"], info["kernel_launches"], stages


res = {}
for N in (1, 2, 4, 8):
    per = [time_share(*adist.rank_segments(8, N, g)) for g in range(N)]
    tmax = max(p[0] for p in per)
    slow = max(per, key=lambda p: p[0])
    res[N] = {"T_ms": tmax, "ranks_ms": [round(p[0], 4) for p in per], "products": sum(p[1] for p in per),
              "launches_per_rank": slow[2], "slowest_rank_stages_ms": slow[3]}
T1 = res[1]["T_ms"]
for N in res:
    res[N]["efficiency"] = T1 / (N * res[N]["T_ms"])
    res[N]["GFLOPS_job"] = 2 * res[N]["products"] / (res[N]["T_ms"] * 1e-3) / 1e9
print(json.dumps({"workload": cfg, "dtype": str(np.dtype(dt)), "proxy": "1-GPU, each rank's share timed alone",
                  "results": res}))
