import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, "tests")
import numpy as np, torch, oracle
import paper_conf_ppopp_wintermzss19_b200 as p
from synth import power_law_csr
A = power_law_csr(5000, 5000, mean_len=10, alpha=1.3, max_len=1500, seed=9)
dA = p.DeviceCSR.from_host(A, "cuda", np.float64)
full = p.multiply(dA, dA); frp, fcol, fval = full.to_numpy()
ref = oracle.gustavson(A, A)
print("full vs oracle struct", (frp == ref.row_ptr).all(), (fcol == ref.col).all(), np.max(np.abs(fval - ref.val) / np.maximum(ref.absval, 1e-300)))
full2 = p.multiply(dA, dA); print("repeat identical", full2.to_numpy()[2].tobytes() == fval.tobytes())
S = 8; G = 2
seg = p.canonical_segments(dA, S)
pieces = []
for g in range(G):
    s0, s1 = g * S // G, (g + 1) * S // G
    r0, r1 = seg[s0], seg[s1]
    plan = p.Plan(); plan.set_segments([r - r0 for r in seg[s0:s1 + 1]])
    view = p.api._csr_in(dA, row_ptr=dA.row_ptr[r0:r1 + 1].contiguous(), rows=r1 - r0, nnz=int(A.row_ptr[r1] - A.row_ptr[r0]))
    C = plan.multiply(dA, dA, A_view=view); torch.cuda.synchronize(); pieces.append(C.to_numpy()); print(g, plan.info()["npath"], plan.info()["nmulti"])
    plan.close()
val = np.concatenate([v for _, _, v in pieces]); col = np.concatenate([c for _, c, _ in pieces])
print("cols equal", (col == fcol).all())
d = np.nonzero(val != fval)[0]
print("ndiff", len(d))
rows = np.searchsorted(frp, d, side="right") - 1
ur = np.unique(rows); print("rows", ur[:20], "row lens", np.diff(frp)[ur[:20]])
print("max rel", np.max(np.abs(val - ref.val) / np.maximum(ref.absval, 1e-300)))
