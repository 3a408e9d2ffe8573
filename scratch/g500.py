import sys, os, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch, oracle
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import rmat
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 16
A = rmat(scale=scale, edge_factor=16, abc=(0.57, 0.19, 0.19), values="uniform")
deg = np.diff(A.row_ptr.astype(np.int64))
print("scale", scale, "nnz", A.row_ptr[-1], "max deg", deg.max(), "rows > 2048:", (deg > 2048).sum(), flush=True)
dA = acs.DeviceCSR.from_host(A, "cuda")
plan = acs.Plan(stage_times=True)
C = plan.multiply(dA, dA); torch.cuda.synchronize()
t = time.time()
for _ in range(3): C = plan.multiply(dA, dA)
torch.cuda.synchronize(); ms = (time.time() - t) / 3 * 1e3
info = plan.info()
print("ms", ms, "GFLOPS", 2 * info["products"] / ms / 1e6, {k: info[k] for k in ("products", "nnz_c", "nchunks", "nshared", "nmulti", "npath", "nsearch")})
print({k: round(v, 3) for k, v in plan.stage_times().items()}, flush=True)
rp, col, val = C.to_numpy()
t = time.time(); ref = oracle.gustavson(A, A); print("oracle s", time.time() - t)
ok = (rp == ref.row_ptr).all() and (col == ref.col).all()
err = np.max(np.abs(val - ref.val) / np.maximum(ref.absval, 1e-300))
print("struct ok", ok, "max rel err", err)
