"""GPU tests of the bounded chunk pool (acspgemm_options.pool_mode, reading R40): hash
candidates own min(products, rows x 256) pool elements, candidates that end in AC-ESC
are deferred to a second pass with their exact bound.  Every case must give the bytes
of the exact pool and match the oracle."""
import hashlib

import numpy as np
import pytest
import torch

import oracle
from synth import CSR, from_coo, poisson3d_27pt, random_csr

pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


def run(A, B, dt, **kw):
    p = pkg()
    plan = p.Plan(**kw)
    dA = p.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else p.DeviceCSR.from_host(B, "cuda", dt)
    C = plan.multiply(dA, dB)
    torch.cuda.synchronize()
    rp, col, val = C.to_numpy()
    info = plan.info()
    return (rp, col, val), info, plan, dA, dB, C


def digest(c):
    h = hashlib.sha256()
    for a in c:
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()


def check_oracle(c, A, B, dt):
    rp, col, val = c
    ref = oracle.gustavson(A.astype(dt), B.astype(dt))
    assert (rp == ref.row_ptr).all() and (col == ref.col).all()
    assert (np.abs(val.astype(np.float64) - ref.val) <= TOL[dt] * ref.absval).all()


def overlapping_rows(n_rows=300, per_row=40, step=8, blen=32, seed=5):
    """Rows of 40 consecutive B rows whose columns overlap by 3/4 (hash candidates) but
    reach 8*39 + 32 = 344 > 256 distinct columns: k_hash and k_rows give them up, so in the
    bounded pool they are deferred to AC-ESC; a 27-point stencil block keeps k_hash busy."""
    rng = np.random.default_rng(seed)
    nb = n_rows + per_row
    rows, cols = [], []
    for r in range(n_rows):
        rows += [r] * per_row
        cols += list(range(r, r + per_row))
    A = from_coo(n_rows, nb, rows, cols, rng.uniform(-1, 1, len(rows)))
    brows, bcols = [], []
    for k in range(nb):
        brows += [k] * blen
        bcols += list(range(k * step, k * step + blen))
    B = from_coo(nb, nb * step + blen, brows, bcols, rng.uniform(-1, 1, len(brows)))
    return A, B


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_bound_pool_same_bytes_stencil(dt, cuda_available):
    A = poisson3d_27pt(24)
    ce, ie, *_ = run(A, A, dt, pool_mode="exact")
    cb, ib, *_ = run(A, A, dt, pool_mode="bound")
    assert digest(ce) == digest(cb)
    check_oracle(cb, A, A, dt)
    assert ie["pool_mode"] == 0 and ib["pool_mode"] == 1
    assert ib["pool_bytes"] < 0.6 * ie["pool_bytes"]          # 27 x 27 products vs <= 192 per row
    assert ib["ndeferred_blocks"] == 0 and ib["nhash_blocks"] == ie["nhash_blocks"] > 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_bound_pool_deferred_blocks(dt, cuda_available):
    A, B = overlapping_rows()
    ce, ie, *_ = run(A, B, dt, pool_mode="exact")
    cb, ib, *_ = run(A, B, dt, pool_mode="bound")
    assert ib["ndeferred_blocks"] > 0                         # candidates that ended in AC-ESC
    assert digest(ce) == digest(cb)
    check_oracle(cb, A, B, dt)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_bound_pool_row_cap(dt, cuda_available):
    """Rows of 8*23 + 32 = 216 distinct columns: within the hash table's 256 (EXACT: k_hash
    takes them) but over POOL_BOUND's cap of 192 per row (HASH_UBOUND), so in the bounded
    pool k_hash gives the blocks up and they are deferred to AC-ESC -- the same bytes."""
    A, B = overlapping_rows(n_rows=300, per_row=24, seed=11)
    ce, ie, *_ = run(A, B, dt, pool_mode="exact")
    cb, ib, *_ = run(A, B, dt, pool_mode="bound")
    assert ie["nhash_blocks"] > 0 and ie["ndeferred_blocks"] == 0
    assert ib["nhash_blocks"] < ie["nhash_blocks"] and ib["ndeferred_blocks"] > 0
    assert digest(ce) == digest(cb)
    check_oracle(cb, A, B, dt)


def test_bound_pool_mixed_and_replay(cuda_available):
    """Deferred blocks next to hash blocks and short-row blocks in one multiply, then a
    graph replay (numeric_update) with new values: the same bytes as the exact pool."""
    A1, B1 = overlapping_rows(n_rows=200, seed=9)
    P = poisson3d_27pt(12)
    # block-diagonal [[A1, 0], [0, P]] times [[B1, 0], [0, P]]
    def bdiag(X, Y):
        rows = np.concatenate([np.repeat(np.arange(X.rows), np.diff(X.row_ptr)),
                               X.rows + np.repeat(np.arange(Y.rows), np.diff(Y.row_ptr))])
        cols = np.concatenate([X.col, X.cols + Y.col])
        vals = np.concatenate([X.val, Y.val])
        return from_coo(X.rows + Y.rows, X.cols + Y.cols, rows, cols, vals)
    A = bdiag(A1, P)
    B = bdiag(B1, P)
    ce, ie, *_ = run(A, B, np.float64, pool_mode="exact")
    cb, ib, plan, dA, dB, C = run(A, B, np.float64, pool_mode="bound")
    assert ib["ndeferred_blocks"] > 0 and ib["nhash_blocks"] > 0
    assert digest(ce) == digest(cb)
    check_oracle(cb, A, B, np.float64)
    # new values, same pattern: numeric_update replays the deferred pass in a CUDA graph
    rng = np.random.default_rng(3)
    A2 = CSR(A.rows, A.cols, A.row_ptr, A.col, rng.uniform(-1, 1, A.val.shape[0]))
    B2 = CSR(B.rows, B.cols, B.row_ptr, B.col, rng.uniform(-1, 1, B.val.shape[0]))
    p = pkg()
    dA2 = p.DeviceCSR.from_host(A2, "cuda", np.float64)
    dB2 = p.DeviceCSR.from_host(B2, "cuda", np.float64)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        plan.numeric_update(dA2, dB2, C, s)
    s.synchronize()
    ref, *_ = run(A2, B2, np.float64, pool_mode="exact")
    assert digest(C.to_numpy()) == digest(ref)


def test_auto_pool_under_limit(cuda_available):
    """AUTO: the exact bound does not fit pool_limit_bytes, the bounded pool does -- the
    multiply succeeds in the bounded pool with the exact pool's bytes; EXACT fails."""
    p = pkg()
    A = poisson3d_27pt(20)
    ce, ie, *_ = run(A, A, np.float64, pool_mode="exact")
    limit = int(0.5 * ie["pool_bytes"])
    ca, ia, *_ = run(A, A, np.float64, pool_mode="auto", pool_limit_bytes=limit)
    assert ia["pool_mode"] == 1 and digest(ca) == digest(ce)
    ca2, ia2, *_ = run(A, A, np.float64, pool_mode="auto")      # no limit: exact
    assert ia2["pool_mode"] == 0 and digest(ca2) == digest(ce)
    with pytest.raises(p.AcspgemmError) as ei:
        run(A, A, np.float64, pool_mode="exact", pool_limit_bytes=limit)
    assert ei.value.status == 4                                  # OUT_OF_MEMORY


def test_bound_pool_esc_strategy_is_exact(cuda_available):
    A = random_csr(400, 400, 0.02, seed=4)
    ce, ie, *_ = run(A, A, np.float64, strategy="esc", pool_mode="exact")
    cb, ib, *_ = run(A, A, np.float64, strategy="esc", pool_mode="bound")
    assert ib["pool_mode"] == 0 and digest(ce) == digest(cb)
