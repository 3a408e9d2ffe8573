"""Graph500-parameter R-MAT (a, b, c = .57, .19, .19; SURVEY §8(c) reading 23, §8(f)-1):
time C = A·A and report the long-row chunks' effect (run with ACSPGEMM_LIB pointing at a
build without them, ACS_PTR_LEN=2147483647, to compare).

usage: python tools/g500_time.py [scale] [reps]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import rmat

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 18
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
A = rmat(scale=scale, edge_factor=16, abc=(0.57, 0.19, 0.19), values="uniform")
deg = np.diff(A.row_ptr.astype(np.int64))
dA = acs.DeviceCSR.from_host(A, "cuda")
plan = acs.Plan(stage_times=True)
C = plan.multiply(dA, dA)
del C
torch.cuda.synchronize()
ts, st = [], []
for _ in range(reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    C = plan.multiply(dA, dA)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
    st.append(plan.stage_times())
    del C
info = plan.info()
ms = statistics.median(ts)
print(json.dumps({"workload": f"graph500 rmat s{scale} ef16", "lib": os.path.basename(os.environ.get("ACSPGEMM_LIB", "libacspgemm.so")),
                  "nnz_a": int(A.row_ptr[-1]), "max_degree": int(deg.max()), "rows_deg_gt_2048": int((deg > 2048).sum()),
                  "ms": ms, "GFLOPS": 2 * info["products"] / (ms * 1e-3) / 1e9,
                  "stages_ms": {k: round(statistics.median(s[k] for s in st), 3) for k in st[0]},
                  **{k: info[k] for k in ("products", "nnz_c", "nchunks", "nshared", "nmulti", "npath", "nsearch")}}))
