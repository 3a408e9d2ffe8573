"""GPU parity of the per-row accumulator for blocks of short rows (reading R34,
csrc/rows.cu): AMG prolongation A·P and the Galerkin R·(A·P).

What pins it:
  * rows that lie inside one block are the left fold of their products in A-entry order
    -- the oracle's Gustavson order -- so fp64 values equal the oracle's bit for bit;
  * structure bit-exact and values within tolerance everywhere (rows split over blocks
    are merged by MCC as for every other path);
  * blocks with a row of more than 8 distinct columns or more than 256 products are
    left to AC-ESC (counted, results still exact);
  * bit-identical run to run.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle import alg
from synth import aggregation_prolongator, from_coo, poisson2d_5pt, poisson3d_7pt, random_csr, random_rowlen_csr

from test_gpu_parity import TOL, pkg

pytestmark = pytest.mark.gpu


def run(A, B, dt, strategy="adaptive"):
    p = pkg()
    plan = p.Plan(strategy=strategy)
    dA = p.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else p.DeviceCSR.from_host(B, "cuda", dt)
    C = plan.multiply(dA, dB)
    torch.cuda.synchronize()
    out = C.to_numpy()
    info = plan.info()
    plan.close()
    return out, info


def check(out, A, B, dt):
    rp, col, val = out
    ref = oracle.gustavson(A.astype(dt), B.astype(dt))
    assert (rp == ref.row_ptr).all() and (col == ref.col).all()
    err = np.abs(val.astype(np.float64) - ref.val)
    assert not (err > TOL[dt] * ref.absval).any()
    return ref


def inside_rows(A):
    """Rows whose nonzeros lie inside one 512-entry block (blocks counted per canonical
    segment, reading R21)."""
    rp = A.row_ptr.astype(np.int64)
    seg = alg.canonical_segments(A.row_ptr, 8)
    s_of = np.searchsorted(np.asarray(seg[1:]), np.arange(A.rows), side="right")
    base = rp[np.asarray(seg)[s_of]]
    return np.nonzero((rp[1:] > rp[:-1]) & (((rp[:-1] - base) // 512) == ((rp[1:] - 1 - base) // 512)))[0]


def revalue(M, seed):
    return type(M)(M.rows, M.cols, M.row_ptr, M.col, np.random.default_rng(seed).uniform(-1, 1, M.col.shape[0]))


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_rows_prolongation(dt, cuda_available):
    """A·P (7-point stencil x 2^3 aggregation, integer values): every block is taken,
    the result is exact."""
    A, P = poisson3d_7pt(16), aggregation_prolongator(16)
    out, info = run(A, P, dt)
    ref = check(out, A, P, dt)
    assert info["nrow_blocks"] == info["nblocks"]
    assert (out[2].astype(np.float64) == ref.val).all()


def test_rows_left_fold_bit_exact_fp64(cuda_available):
    """U(-1,1) values in A and P: rows inside one block equal the oracle's left fold bit
    for bit."""
    A, P = revalue(poisson3d_7pt(24), 1), revalue(aggregation_prolongator(24), 2)
    out, info = run(A, P, np.float64)
    ref = check(out, A, P, np.float64)
    assert info["nrow_blocks"] == info["nblocks"]
    crp = ref.row_ptr.astype(np.int64)
    rows = inside_rows(A)
    assert len(rows) > 1000
    for i in rows:
        s, e = crp[i], crp[i + 1]
        assert out[2][s:e].tobytes() == ref.val[s:e].tobytes()


def test_rows_five_point_goes_to_esc(cuda_available):
    """5-point stencil squared: 13 columns per row > 8 slots, AC-ESC takes every block."""
    A = poisson2d_5pt(48)
    out, info = run(A, A, np.float64)
    ref = check(out, A, A, np.float64)
    assert info["nrow_blocks"] == 0 and (out[2] == ref.val).all()


def test_rows_galerkin(cuda_available):
    """R·(A·P) = 4·A7(n/2) exactly (2^3 aggregation); both products take the per-row path."""
    from synth import CSR, transpose
    n = 16
    A, P = poisson3d_7pt(n), aggregation_prolongator(n)
    R = transpose(P)
    (rp, col, val), info1 = run(A, P, np.float64)
    AP = CSR(A.rows, P.cols, rp, col, val)
    (rp2, col2, val2), info2 = run(R, AP, np.float64)
    A4 = poisson3d_7pt(n // 2)
    assert (rp2 == A4.row_ptr).all() and (col2 == A4.col).all() and (val2 == 4 * A4.val).all()
    assert info1["nrow_blocks"] == info1["nblocks"] and info2["nrow_blocks"] == info2["nblocks"]


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_rows_fallback_many_columns(dt, cuda_available):
    """Rows of 3 entries x B rows of 8 random columns (24 distinct > 8): no block is
    taken; mixed with rows of 1 entry (8 columns) in other blocks: those are."""
    rng = np.random.default_rng(4)
    nb = 3000
    B = random_rowlen_csr(nb, 5000, np.full(nb, 8), seed=5)
    lens = np.where(np.arange(2000) < 1000, 3, 1)          # rows 0..999: 24 products, rows 1000..: 8
    A = random_rowlen_csr(2000, nb, lens, seed=6)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert 0 < info["nrow_blocks"] < info["nblocks"]
    esc, _ = run(A, B, dt, strategy="esc")
    assert (esc[0] == out[0]).all() and (esc[1] == out[1]).all()


def test_rows_long_row_not_taken(cuda_available):
    """A row of more than 256 products keeps its block in AC-ESC."""
    n = 600
    r = [0] * 40 + list(range(1, n))
    c = list(range(40)) + list(range(1, n))
    A = from_coo(n, n, r, c, np.ones(len(r)))
    B = random_rowlen_csr(n, 50, np.full(n, 8), seed=2, values="int")
    out, info = run(A, B, np.float64)
    ref = check(out, A, B, np.float64)
    assert info["nrow_blocks"] == info["nblocks"] - 1
    assert (out[2] == ref.val).all()


def test_rows_bit_stable(cuda_available):
    A, P = revalue(poisson3d_7pt(20), 3), revalue(aggregation_prolongator(20), 4)
    outs = [run(A, P, np.float64)[0] for _ in range(3)]
    assert all(o[2].tobytes() == outs[0][2].tobytes() for o in outs)
