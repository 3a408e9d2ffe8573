"""Pins for the Gustavson oracle (oracle/gustavson.c) against things other than
itself: dense brute force, closed-form stencil squares, the Galerkin closed form,
invariants, special cases and a scipy pattern cross-check (SURVEY §8(c) "What pins
each part").  CPU only."""
import numpy as np
import pytest

import oracle
from synth import (CSR, aggregation_prolongator, from_coo, poisson2d_5pt, poisson3d_27pt,
                   poisson3d_7pt, random_csr, transpose)


def dense_check(A, B, C, rtol=1e-12):
    """Pattern = (mask(A)·mask(B) > 0); values = dense fp64 product within
    rtol·(|A|·|B|) (north_star tolerance, fp64)."""
    dA, dB = A.to_dense(), B.to_dense()
    mA = (np.zeros_like(dA) != 0)
    mB = (np.zeros_like(dB) != 0)
    rA = np.repeat(np.arange(A.rows), A.row_lengths())
    mA[rA, A.col] = True
    rB = np.repeat(np.arange(B.rows), B.row_lengths())
    mB[rB, B.col] = True
    pattern = (mA.astype(np.int64) @ mB.astype(np.int64)) > 0
    ref = dA @ dB
    absref = np.abs(dA) @ np.abs(dB)
    # structure
    rC = np.repeat(np.arange(C.rows), np.diff(C.row_ptr))
    got = np.zeros_like(pattern)
    got[rC, C.col] = True
    assert (got == pattern).all()
    assert C.nnz == int(pattern.sum())
    # ascending unique columns
    for i in range(C.rows):
        cols = C.col[C.row_ptr[i]:C.row_ptr[i + 1]]
        assert (np.diff(cols) > 0).all()
    err = np.abs(C.val - ref[rC, C.col])
    assert (err <= rtol * absref[rC, C.col] + 1e-300).all()
    assert np.allclose(C.absval, absref[rC, C.col], rtol=1e-12, atol=0)


@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_random(seed):
    rng = np.random.default_rng(1000 + seed)
    m, k, n = (int(x) for x in rng.integers(1, 65, 3))
    dA, dB = rng.uniform(0, 0.6, 2)
    A = random_csr(m, k, dA, seed=seed, empty_rows=0.2 if seed % 3 == 0 else 0.0)
    B = random_csr(k, n, dB, seed=seed + 77, values="int" if seed % 2 else "uniform")
    C = oracle.gustavson(A, B)
    dense_check(A, B, C)


def test_bruteforce_degenerate():
    # all-zero, single row/col, empty inputs
    Z = random_csr(5, 7, 0.0, seed=1)
    B = random_csr(7, 4, 0.5, seed=2)
    C = oracle.gustavson(Z, B)
    assert C.nnz == 0 and (C.row_ptr == 0).all()
    A = random_csr(1, 7, 1.0, seed=3)
    dense_check(A, B, oracle.gustavson(A, B))
    E = CSR(0, 7, np.zeros(1, np.int32), np.zeros(0, np.int32), np.zeros(0))
    C = oracle.gustavson(E, B)
    assert C.rows == 0 and C.nnz == 0
    with pytest.raises(ValueError):
        oracle.gustavson(B, B)


def test_structural_zeros_kept():
    # (1 1)·(1 -1)^T = 0 : the cancellation is kept as a stored zero (reading R2)
    A = from_coo(1, 2, [0, 0], [0, 1], np.array([1.0, 1.0]))
    B = from_coo(2, 1, [0, 1], [0, 0], np.array([1.0, -1.0]))
    C = oracle.gustavson(A, B)
    assert C.nnz == 1 and C.val[0] == 0.0 and C.absval[0] == 2.0


def test_poisson2d_closed_form():
    """A = 4I − N on 64²: (A²)_pp = 16 + deg(p); axis distance 1: −8; diagonal
    neighbours: 2; axis distance 2: 1.  nnz = 51,972, products = 100,104."""
    n = 64
    A = poisson2d_5pt(n)
    C = oracle.gustavson(A, A)
    assert C.nnz == 51972
    assert oracle.products(A, A) == 100104
    rows = np.repeat(np.arange(C.rows), np.diff(C.row_ptr))
    px, py = rows % n, rows // n
    qx, qy = C.col % n, C.col // n
    dx, dy = np.abs(qx - px), np.abs(qy - py)
    deg = (px > 0).astype(int) + (px < n - 1) + (py > 0) + (py < n - 1)
    exp = np.full(C.nnz, np.nan)
    exp[(dx == 0) & (dy == 0)] = (16 + deg)[(dx == 0) & (dy == 0)]
    exp[(dx + dy) == 1] = -8
    exp[(dx == 1) & (dy == 1)] = 2
    exp[((dx == 2) & (dy == 0)) | ((dx == 0) & (dy == 2))] = 1
    assert not np.isnan(exp).any()
    assert (C.val == exp).all()


@pytest.mark.parametrize("n", [6, 9])
def test_poisson27_closed_form(n):
    """A = 27I − M, M = T⊗T⊗T:  A² = 729I − 54M + T²⊗T²⊗T² with (T²)_ii ∈ {2,3},
    (T²)_{i,i±1} = 2, (T²)_{i,i±2} = 1.  nnz = (5n−6)³, products = (9n−10)³."""
    A = poisson3d_27pt(n)
    C = oracle.gustavson(A, A)
    assert C.nnz == (5 * n - 6) ** 3
    assert oracle.products(A, A) == (9 * n - 10) ** 3
    rows = np.repeat(np.arange(C.rows), np.diff(C.row_ptr))

    def coords(i):
        return i % n, (i // n) % n, i // (n * n)

    p, q = coords(rows), coords(C.col.astype(np.int64))

    def t2(a, b):
        d = np.abs(a - b)
        diag = np.where((a == 0) | (a == n - 1), 2, 3)
        return np.where(d == 0, diag, np.where(d == 1, 2, np.where(d == 2, 1, 0)))

    m_ = np.ones(C.nnz, dtype=np.int64)
    t2p = np.ones(C.nnz, dtype=np.int64)
    for a, b in zip(p, q):
        m_ *= (np.abs(a - b) <= 1)
        t2p *= t2(a, b)
    exp = 729 * (rows == C.col) - 54 * m_ + t2p
    assert (C.val == exp).all()


@pytest.mark.parametrize("n", [8, 16])
def test_galerkin_closed_form(n):
    """A₇ with 2³ aggregation: AP ∈ {3, −1}, nnz(AP) = N(1 + 3(n−2)/n);
    R·(A·P) = 4·A₇(n/2) exactly."""
    A = poisson3d_7pt(n)
    P = aggregation_prolongator(n)
    R = transpose(P)
    AP = oracle.gustavson(A, P)
    assert set(np.unique(AP.val)) <= {3.0, -1.0}
    N = n ** 3
    assert AP.nnz == N + 3 * N * (n - 2) // n
    APc = CSR(AP.rows, AP.cols, AP.row_ptr, AP.col, AP.val)
    RAP = oracle.gustavson(R, APc)
    A4 = poisson3d_7pt(n // 2)
    assert (RAP.row_ptr == A4.row_ptr).all() and (RAP.col == A4.col).all()
    assert (RAP.val == 4 * A4.val).all()


@pytest.mark.parametrize("seed", range(4))
def test_invariants(seed):
    rng = np.random.default_rng(seed)
    A = random_csr(200, 150, 0.05, seed=seed)
    B = random_csr(150, 180, 0.05, seed=seed + 9)
    C = oracle.gustavson(A, B)
    # sum of entries = (1ᵀA)(B1)
    s_ref = A.to_dense().sum(axis=0) @ B.to_dense().sum(axis=1)
    assert abs(C.val.sum() - s_ref) <= 1e-10 * C.absval.sum()
    # Freivalds: C·x = A·(B·x)
    x = rng.uniform(-1, 1, 180)
    Cx = np.zeros(C.rows)
    np.add.at(Cx, np.repeat(np.arange(C.rows), np.diff(C.row_ptr)), C.val * x[C.col])
    ABx = A.to_dense() @ (B.to_dense() @ x)
    assert np.allclose(Cx, ABx, rtol=0, atol=1e-10 * max(1.0, np.abs(ABx).max()))
    # nnz(C) ≤ products, products computed independently through the dense masks
    prods = int(((A.to_dense() != 0).sum(axis=0) * (B.to_dense() != 0).sum(axis=1)).sum())
    assert oracle.products(A, B) == prods and C.nnz <= prods


def test_special_cases():
    A = random_csr(40, 30, 0.2, seed=5)
    I30 = from_coo(30, 30, np.arange(30), np.arange(30), np.ones(30))
    I40 = from_coo(40, 40, np.arange(40), np.arange(40), np.ones(40))
    for C in (oracle.gustavson(A, I30), oracle.gustavson(I40, A)):
        assert (C.row_ptr == A.row_ptr).all() and (C.col == A.col).all() and (C.val == A.val).all()
    # permutation rows
    perm = np.random.default_rng(1).permutation(40)
    Pm = from_coo(40, 40, np.arange(40), perm, np.ones(40))
    C = oracle.gustavson(Pm, A)
    dA = A.to_dense()
    assert (CSR(C.rows, C.cols, C.row_ptr, C.col, C.val).to_dense() == dA[perm]).all()
    # diagonal scaling: one product per entry -> correctly rounded a*b
    d = np.random.default_rng(2).uniform(-2, 2, 40)
    D = from_coo(40, 40, np.arange(40), np.arange(40), d)
    C = oracle.gustavson(D, A)
    assert (C.val == d[np.repeat(np.arange(40), A.row_lengths())] * A.val).all()
    # outer product (n×1)(1×n): dense, single-term entries
    u = from_coo(9, 1, np.arange(9), np.zeros(9), np.arange(1.0, 10.0))
    v = from_coo(1, 9, np.zeros(9), np.arange(9), np.arange(1.0, 10.0) / 7)
    C = oracle.gustavson(u, v)
    assert C.nnz == 81
    assert (C.val == np.outer(np.arange(1.0, 10.0), np.arange(1.0, 10.0) / 7).ravel()).all()
    # dot product (1×n)(n×1): one n-term entry
    w = np.random.default_rng(3).uniform(-1, 1, 50)
    rvec = from_coo(1, 50, np.zeros(50), np.arange(50), w)
    cvec = from_coo(50, 1, np.arange(50), np.zeros(50), w)
    C = oracle.gustavson(rvec, cvec)
    assert C.nnz == 1 and abs(C.val[0] - float(w @ w)) <= 1e-14 * C.absval[0]
    # A·0 = empty
    Z = random_csr(30, 10, 0.0, seed=1)
    assert oracle.gustavson(A, Z).nnz == 0


def test_scipy_pattern_crosscheck():
    sp = pytest.importorskip("scipy.sparse")
    A = random_csr(300, 250, 0.03, seed=11, values="ones")
    B = random_csr(250, 320, 0.03, seed=12, values="ones")
    C = oracle.gustavson(A, B)
    S = (sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(300, 250)) @
         sp.csr_matrix((B.val, B.col, B.row_ptr), shape=(250, 320))).tocsr()
    S.sort_indices()
    assert (S.indptr == C.row_ptr).all() and (S.indices == C.col).all()
    assert (S.data == C.val).all()        # unit values: exact integer counts


def test_thread_count_invariance():
    A = random_csr(500, 400, 0.02, seed=21)
    B = random_csr(400, 450, 0.02, seed=22)
    C1 = oracle.gustavson(A, B, threads=1)
    C4 = oracle.gustavson(A, B, threads=4)
    assert (C1.row_ptr == C4.row_ptr).all() and (C1.col == C4.col).all()
    assert C1.val.tobytes() == C4.val.tobytes()


def test_row_range():
    A = random_csr(100, 80, 0.05, seed=31)
    B = random_csr(80, 90, 0.05, seed=32)
    full = oracle.gustavson(A, B)
    part = oracle.gustavson(A, B, row_begin=37, row_end=81)
    lo, hi = full.row_ptr[37], full.row_ptr[81]
    assert (part.row_ptr == full.row_ptr[37:82] - lo).all()
    assert (part.col == full.col[lo:hi]).all() and (part.val == full.val[lo:hi]).all()
