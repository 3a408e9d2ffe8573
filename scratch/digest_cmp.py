import sys, os, hashlib
alt = sys.argv[1]
sys.path.insert(0, alt if alt else os.getcwd()); sys.path.insert(1, os.getcwd())
import numpy as np, torch
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config, power_law_csr, poisson3d_27pt, rmat
out = []
for name, A in [("pl", power_law_csr(20000, 20000, 10, 1.3, 2000, seed=1)), ("27pt", poisson3d_27pt(40)), ("rmat", rmat(scale=14))]:
    dA = acs.DeviceCSR.from_host(A, "cuda")
    C = acs.multiply(dA, dA); torch.cuda.synchronize()
    h = hashlib.sha256()
    for t in (C.row_ptr, C.col, C.val): h.update(t.cpu().numpy().tobytes())
    out.append(f"{name}:{h.hexdigest()[:16]}")
print(acs.SO_PATH.split('/')[-3], " ".join(out))
