"""int64 row pointers of C (acspgemm_numeric64; outputs beyond 2^31
entries).  Small products: the int64 row_ptr equals the int32 one and col/val are
byte-identical.  One product with nnz(C) > 2^31 (2^21 rows of 34 random columns squared,
fp32): the int32 numeric pass refuses it (INDEX_OVERFLOW), the int64 one delivers it;
checked by row_ptr invariants, the exact product count, and sampled rows (random,
longest, segment boundaries, the rows around entry 2^31) element by element against the
CPU oracle."""
import numpy as np
import pytest
import torch

import oracle
from synth import CSR, poisson3d_27pt, random_csr

from test_gpu_fullsize import check_rows, rowptr_invariants, sample_rows

pytestmark = pytest.mark.gpu


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_index64_matches_index32(dt, cuda_available):
    p = pkg()
    for A in (poisson3d_27pt(12), random_csr(3000, 3000, 0.004, seed=5)):
        dA = p.DeviceCSR.from_host(A, "cuda", dt)
        plan = p.Plan()
        C32 = plan.multiply(dA, dA)
        C64 = plan.multiply(dA, dA, index64=True)
        torch.cuda.synchronize()
        assert C64.row_ptr.dtype == torch.int64 and C32.row_ptr.dtype == torch.int32
        assert torch.equal(C64.row_ptr, C32.row_ptr.to(torch.int64))
        assert C64.col.cpu().numpy().tobytes() == C32.col.cpu().numpy().tobytes()
        assert C64.val.cpu().numpy().tobytes() == C32.val.cpu().numpy().tobytes()
        plan.close()


def test_index64_empty(cuda_available):
    p = pkg()
    A = CSR(5, 7, np.zeros(6, np.int32), np.zeros(0, np.int32), np.zeros(0))
    B = random_csr(7, 4, 0.5, seed=1)
    plan = p.Plan()
    C = plan.multiply(p.DeviceCSR.from_host(A, "cuda"), p.DeviceCSR.from_host(B, "cuda"), index64=True)
    torch.cuda.synchronize()
    assert C.row_ptr.dtype == torch.int64 and (C.row_ptr.cpu().numpy() == 0).all() and C.nnz == 0


@pytest.mark.slow
def test_nnz_beyond_int32(cuda_available):
    p = pkg()
    n, k = 1 << 21, 34
    rng = np.random.default_rng(2024)
    # k distinct sorted columns per row: sorted draws from [0, n-k) plus 0..k-1
    cols = (np.sort(rng.integers(0, n - k, (n, k), dtype=np.int64), axis=1) + np.arange(k)).astype(np.int32)
    A = CSR(n, n, (np.arange(n + 1, dtype=np.int64) * k).astype(np.int32), cols.ravel(),
            rng.uniform(-1, 1, n * k).astype(np.float32))
    del cols
    colcount = np.bincount(A.col, minlength=n).astype(np.int64)
    products = int((colcount * k).sum())
    assert products > 2 ** 31
    dA = p.DeviceCSR.from_host(A, "cuda", np.float32)
    plan = p.Plan()
    with pytest.raises(p.AcspgemmError) as e:
        plan.multiply(dA, dA)                         # int32 row_ptr cannot hold nnz(C)
    assert e.value.status == 3                        # ACSPGEMM_ERR_INDEX_OVERFLOW
    C = plan.multiply(dA, dA, index64=True)
    torch.cuda.synchronize()
    info = plan.info()
    assert info["products"] == products
    nnz = C.nnz
    assert 2 ** 31 < nnz <= products and info["nnz_c"] == nnz
    rp = C.row_ptr.cpu().numpy()
    rowptr_invariants(rp, n, nnz)
    rows = sample_rows(A, rp, 300, seed=7)
    r31 = int(np.searchsorted(rp, 2 ** 31, side="right")) - 1    # the row holding entry 2^31
    rows = np.unique(np.concatenate([rows, [max(r31 - 1, 0), r31, min(r31 + 1, n - 1)]]))
    # gather the sampled rows of C on the device (C itself is ~19 GB)
    idx = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in rows])
    ti = torch.from_numpy(idx).cuda()
    col_s, val_s = C.col[ti].cpu().numpy(), C.val[ti].cpu().numpy()
    sub_rp = np.zeros(n + 1, dtype=np.int64)
    lens = np.zeros(n, dtype=np.int64)
    lens[rows] = rp[rows + 1] - rp[rows]
    np.cumsum(lens, out=sub_rp[1:])
    del C, ti
    plan.close()
    torch.cuda.empty_cache()
    check_rows(A, A, rows, (sub_rp, col_s, val_s), 1e-5, exact=False)
