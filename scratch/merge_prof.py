import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np, paper_conf_ppopp_wintermzss19_b200 as acs
from synth import config
cfg = sys.argv[1]
A, B = config(cfg)
dA = acs.DeviceCSR.from_host(A, "cuda"); dB = dA if cfg != "cfg5" else acs.DeviceCSR.from_host(B, "cuda")
plan = acs.Plan(stage_times=True)
C = plan.multiply(dA, dB)
torch.cuda.synchronize()
print(cfg, plan.info())
print(plan.stage_times())
# row length stats of C
rp = C.row_ptr.cpu().numpy().astype(np.int64); L = np.diff(rp)
print("C rows", len(L), "max", L.max(), "rows>512", (L>512).sum(), "elems in rows>512", L[L>512].sum(), "rows>2048", (L>2048).sum(), "elems", L[L>2048].sum())
