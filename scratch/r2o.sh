cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "long_row_chunks and float64" 2>&1 | grep -E "Error|assert|mismatch|tolerance" | head -20
cat > /tmp/dbg.py <<'PY'
import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.getcwd() + "/tests")
import numpy as np, torch, oracle
import paper_conf_ppopp_wintermzss19_b200 as acs
from synth import from_coo
rng = np.random.default_rng(21)
nb, ncols = 400, 6000
blen = rng.integers(5, 60, nb)
blen[rng.choice(nb, 60, replace=False)] = rng.integers(2049, 5000, 60)
long_rows = np.flatnonzero(blen > 2048); short_rows = np.flatnonzero(blen <= 2048)
r, c = [], []
for i in range(1200):
    kind = i % 6
    if kind == 0: k = [rng.choice(long_rows)]
    elif kind == 1: k = list(rng.choice(short_rows, 5, replace=False)) + [rng.choice(long_rows)]
    elif kind == 2: k = list(rng.choice(long_rows, 3, replace=False))
    elif kind == 3: k = list(rng.choice(short_rows, 8, replace=False))
    else: k = list(rng.choice(short_rows, 6, replace=False)) + list(rng.choice(long_rows, 2, replace=False))
    k = np.unique(k); r += [i]*len(k); c += k.tolist()
for i in range(1200, 1400): r.append(i); c.append(int(long_rows[i % len(long_rows)]))
rr, cc = np.array(r), np.array(c)
va = rng.integers(1, 4, rr.size) * rng.choice([-1.0, 1.0], rr.size)
A = from_coo(1400, nb, rr, cc, va)
rows_b = np.repeat(np.arange(nb), blen)
cols_b = np.concatenate([np.sort(rng.choice(ncols, L, replace=False)) for L in blen])
vb = rng.integers(-3, 4, rows_b.size).astype(np.float64)
B = from_coo(nb, ncols, rows_b, cols_b, vb)
dA = acs.DeviceCSR.from_host(A, "cuda"); dB = acs.DeviceCSR.from_host(B, "cuda")
plan = acs.Plan()
C = plan.multiply(dA, dB); torch.cuda.synchronize()
rp, col, val = C.to_numpy()
ref = oracle.gustavson(A, B)
info = plan.info()
print({k: info[k] for k in ("nblocks","nchunks","nshared","nmulti","npath","nsearch","chunk_elems","nnz_c")})
lens = np.diff(rp); rl = np.diff(ref.row_ptr)
bad = np.flatnonzero(lens != rl)
print("rows with wrong length:", len(bad), bad[:20], lens[bad[:10]], rl[bad[:10]])
if len(bad) == 0:
    badv = [i for i in range(A.rows) if not (col[rp[i]:rp[i+1]] == ref.col[ref.row_ptr[i]:ref.row_ptr[i+1]]).all() or not (val[rp[i]:rp[i+1]] == ref.val[ref.row_ptr[i]:ref.row_ptr[i+1]]).all()]
    print("rows with wrong cols/vals:", len(badv), badv[:20])
for i in bad[:5]:
    print(i, "A entries", A.col[A.row_ptr[i]:A.row_ptr[i+1]], "blens", blen[A.col[A.row_ptr[i]:A.row_ptr[i+1]]])
PY
timeout 120 python /tmp/dbg.py
