"""Run-to-run byte identity under repetition (a race-detection proxy while compute-sanitizer
is closed on the GPU pool): the same multiply many times on one plan and on fresh plans,
SHA-256 of (row_ptr, col, val) each time; every digest must be equal.

usage: python tools/stress_determinism.py [reps]"""
import hashlib
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config, poisson3d_27pt, random_rowlen_csr, from_coo


def digest(C):
    h = hashlib.sha256()
    for t in (C.row_ptr, C.col, C.val):
        h.update(t.cpu().numpy().tobytes())
    return h.hexdigest()[:16]


def run(name, A, B, dt, reps, **kw):
    dA = acs.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else acs.DeviceCSR.from_host(B, "cuda", dt)
    seen = set()
    plan = acs.Plan(**kw)
    for r in range(reps):
        if r % 5 == 4:                   # a fresh plan now and then (fresh tables, buffers)
            plan.close()
            plan = acs.Plan(**kw)
        C = plan.multiply(dA, dB)
        seen.add(digest(C))
        del C
    info = plan.info()
    plan.close()
    out = {"workload": name, "dtype": np.dtype(dt).name, "reps": reps, "distinct_digests": len(seen),
           "digest": sorted(seen)[0], "nhash_blocks": info["nhash_blocks"], "nblocks": info["nblocks"],
           "kw": kw}
    print(json.dumps(out), flush=True)
    return len(seen) == 1


reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
ok = True
rng = np.random.default_rng(5)
A2, _ = config("cfg2", np.float64)
A2u = A2.__class__(A2.rows, A2.cols, A2.row_ptr, A2.col, rng.uniform(-1, 1, A2.nnz))
ok &= run("cfg2 U(-1,1)", A2u, A2u, np.float64, reps)
ok &= run("cfg2 U(-1,1)", A2u, A2u, np.float32, reps)
ok &= run("cfg2 U(-1,1) exact pool", A2u, A2u, np.float64, max(reps // 2, 2), pool_mode="exact")
A5, B5 = config("cfg5", np.float64)
ok &= run("cfg5", A5, B5, np.float64, max(reps // 4, 2))
P = poisson3d_27pt(40)
M = random_rowlen_csr(20000, 20000, rng.integers(1, 60, 20000), seed=7)
ok &= run("27-pt 40^3 x random", P, P, np.float64, reps)
ok &= run("random rows", M, M, np.float64, reps)
print(json.dumps({"all_identical": bool(ok)}))
