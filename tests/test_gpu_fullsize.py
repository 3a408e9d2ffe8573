"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(default Plan: 8 canonical segments, same kernels).  The oracle cannot finish whole
products of this size quickly, so the checks are: sampled rows (random rows, the
longest rows, segment-boundary rows) element by element against the oracle, plus
properties that hold at any size (closed forms, exact counts, row_ptr invariants)."""
import numpy as np
import pytest
import torch

import oracle
from oracle import alg
from synth import CSR, aggregation_prolongator, config, poisson3d_7pt, transpose

pytestmark = pytest.mark.gpu


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


def gpu_full(A, B, dt):
    p = pkg()
    dA = p.DeviceCSR.from_host(A, "cuda", dt)
    dB = dA if B is A else p.DeviceCSR.from_host(B, "cuda", dt)
    plan = p.Plan()
    C = plan.multiply(dA, dB)
    torch.cuda.synchronize()
    info = plan.info()
    out = (C.row_ptr.cpu().numpy(), C.col.cpu().numpy(), C.val.cpu().numpy())
    del C, dA, dB
    plan.close()
    torch.cuda.empty_cache()
    return out, info


def sample_rows(A, C_rp, k, seed):
    rng = np.random.default_rng(seed)
    lens = np.diff(C_rp.astype(np.int64))
    longest = np.argsort(lens)[-200:]
    seg = alg.canonical_segments(A.row_ptr, 8)
    bnd = [r for s in seg[1:-1] for r in (s - 1, s) if 0 <= r < A.rows]
    rows = np.unique(np.concatenate([rng.integers(0, A.rows, k), longest, bnd, [0, A.rows - 1]]))
    return rows


def check_rows(A, B, rows, got, tol, exact):
    rp, col, val = got
    sub_rp = np.zeros(len(rows) + 1, dtype=np.int64)
    lens = (A.row_ptr[rows + 1] - A.row_ptr[rows]).astype(np.int64)
    np.cumsum(lens, out=sub_rp[1:])
    idx = np.concatenate([np.arange(A.row_ptr[r], A.row_ptr[r + 1]) for r in rows]) if len(rows) else np.zeros(0, int)
    sub = CSR(len(rows), A.cols, sub_rp, A.col[idx], A.val[idx])
    ref = oracle.gustavson(sub, B)
    for t, r in enumerate(rows):
        a, b = rp[r], rp[r + 1]
        ra, rb = ref.row_ptr[t], ref.row_ptr[t + 1]
        assert b - a == rb - ra, f"row {r}: length {b - a} vs {rb - ra}"
        assert (col[a:b] == ref.col[ra:rb]).all(), f"row {r}: columns"
        v = val[a:b].astype(np.float64)
        if exact:
            assert (v == ref.val[ra:rb]).all(), f"row {r}: values"
        else:
            assert (np.abs(v - ref.val[ra:rb]) <= tol * ref.absval[ra:rb]).all(), f"row {r}: values"


def rowptr_invariants(rp, rows, nnz_expected=None):
    assert rp.shape[0] == rows + 1 and rp[0] == 0
    assert (np.diff(rp.astype(np.int64)) >= 0).all()
    if nnz_expected is not None:
        assert int(rp[-1]) == nnz_expected


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_cfg2_27pt_128_full(dt, cuda_available):
    """configs[1] (the bench workload): every entry of C = A² checked against the closed
    form A² = 729I − 54·T⊗T⊗T + T²⊗T²⊗T² (integer-valued: bit-exact), nnz = (5n−6)³,
    plus sampled rows against the oracle."""
    n = 128
    A, _ = config("cfg2", dt)
    (rp, col, val), info = gpu_full(A, A, dt)
    rowptr_invariants(rp, A.rows, (5 * n - 6) ** 3)
    assert info["products"] == (9 * n - 10) ** 3
    # closed form on all 254,840,104 entries, in slabs to bound host memory
    rows_all = A.rows
    for r0 in range(0, rows_all, 1 << 19):
        r1 = min(rows_all, r0 + (1 << 19))
        a, b = int(rp[r0]), int(rp[r1])
        rr = np.repeat(np.arange(r0, r1, dtype=np.int64), np.diff(rp[r0:r1 + 1].astype(np.int64)))
        cc = col[a:b].astype(np.int64)
        m_ = np.ones(b - a, dtype=np.int64)
        t2p = np.ones(b - a, dtype=np.int64)
        for div in (1, n, n * n):
            pa, qa = (rr // div) % n, (cc // div) % n
            d = np.abs(pa - qa)
            m_ *= d <= 1
            t2p *= np.where(d == 0, np.where((pa == 0) | (pa == n - 1), 2, 3),
                            np.where(d == 1, 2, np.where(d == 2, 1, 0)))
        exp = 729 * (rr == cc) - 54 * m_ + t2p
        assert (val[a:b].astype(np.float64) == exp).all()
    check_rows(A, A, sample_rows(A, rp, 1500, 1), (rp, col, val), 0, exact=True)


TOL = {np.float64: 1e-12, np.float32: 1e-5}


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_cfg3_rmat_full(dt, cuda_available):
    """configs[2]: R-MAT scale 20 (long skewed rows: Multi and Path Merge at scale), in
    fp64 and fp32 (L554: every matrix in float and double).  nnz(C) = 581,442,205
    (scipy); sampled rows incl. the 200 longest and the segment
    boundaries vs the oracle (on the dtype-rounded inputs)."""
    A, _ = config("cfg3", dt)
    (rp, col, val), info = gpu_full(A, A, dt)
    rowptr_invariants(rp, A.rows, 581442205)
    assert info["products"] == 585358301
    assert info["npath"] + info["nsearch"] > 0
    check_rows(A, A, sample_rows(A, rp, 1500, 3), (rp, col, val), TOL[dt], exact=False)


def test_graph500_rmat_s18_full(cuda_available):
    """§8(f)-1 stress: Graph500-parameter R-MAT (a, b, c = .57, .19, .19; SURVEY §8(c)
    reading 23) at scale 18, ef 16 -- max out-degree ~15.8k, ~2.9 G products, rows of
    C spread over hundreds of chunks (Path / Search Merge, dense slices).  Structure
    bit-exact and values within 1e-12 on sampled rows (the 200 longest included)."""
    from synth import rmat
    A = rmat(scale=18, edge_factor=16, abc=(0.57, 0.19, 0.19), values="uniform")
    deg = np.diff(A.row_ptr.astype(np.int64))
    assert deg.max() > 10000
    (rp, col, val), info = gpu_full(A, A, np.float64)
    rowptr_invariants(rp, A.rows)
    assert info["products"] == oracle.products(A, A)
    assert info["npath"] + info["nsearch"] > 0
    check_rows(A, A, sample_rows(A, rp, 400, 18), (rp, col, val), 1e-12, exact=False)


def test_cfg4_galerkin_rap_full(cuda_available):
    """configs[3]: 7-pt 256³ with 2³ aggregation.  A·P ∈ {3, −1} with nnz N(1+3(n−2)/n);
    R·(A·P) = 4·A₇(128) exactly, every entry."""
    n = 256
    A = poisson3d_7pt(n)
    P = aggregation_prolongator(n)
    (rp, col, val), info = gpu_full(A, P, np.float64)
    N = n ** 3
    rowptr_invariants(rp, N, N + 3 * N * (n - 2) // n)
    assert set(np.unique(val).tolist()) <= {3.0, -1.0}
    AP = CSR(N, P.cols, rp, col, val)
    check_rows(A, P, sample_rows(A, rp, 500, 4), (rp, col, val), 0, exact=True)
    R = transpose(P)
    del A
    (rp2, col2, val2), _ = gpu_full(R, AP, np.float64)
    A4 = poisson3d_7pt(n // 2)
    assert (rp2 == A4.row_ptr).all() and (col2 == A4.col).all() and (val2 == 4 * A4.val).all()


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_cfg5_lp_full(dt, cuda_available):
    """configs[4]: LP-like 2²⁰ × 2²², 20 nnz/col, C = A·Aᵀ (Aᵀ precomputed), fp64 and
    fp32.  Products = 2²²·20² exactly; sampled rows vs the oracle."""
    A, At = config("cfg5", dt)
    (rp, col, val), info = gpu_full(A, At, dt)
    rowptr_invariants(rp, A.rows)
    assert info["products"] == (1 << 22) * 400
    check_rows(A, At, sample_rows(A, rp, 300, 5), (rp, col, val), TOL[dt], exact=False)
