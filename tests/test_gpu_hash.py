"""GPU parity of the adaptive strategy (reading R31): the hash accumulator that blocks
try before AC-ESC (§5), against the CPU oracle and
against the ESC-only strategy, through the C ABI.

What pins it:
  * rows that lie inside one block are summed left to right in A-entry order, the order
    of the oracle's Gustavson accumulator (oracle/gustavson.c: t = a*b; acc += t), so
    fp64 values are bit-identical to the oracle's there (random U(-1,1) values);
  * structure bit-exact, values within the north-star tolerance everywhere;
  * products of one column inside a 32-product wave (short B rows sharing columns),
    empty B rows (more than a warp of them in a row), rows with more distinct columns
    than the table holds (fallback to AC-ESC) and mixed blocks;
  * bit-identical results run to run and across canonical-segment splits.
"""
import numpy as np
import pytest
import torch

import oracle
from oracle import alg
from synth import from_coo, poisson2d_5pt, poisson3d_27pt, power_law_csr, random_csr, random_rowlen_csr, rmat

from test_gpu_parity import TOL, assert_parity, digest, gpu_mult, pkg

pytestmark = pytest.mark.gpu


def run(A, B, dt, strategy="adaptive"):
    p = pkg()
    plan = p.Plan(strategy=strategy)
    dA = p.DeviceCSR.from_host(A, "cuda", dt)
    dB = p.DeviceCSR.from_host(B, "cuda", dt)
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


def test_hash_left_fold_bit_exact_fp64(cuda_available):
    """Rows of 8 entries never straddle a 512-entry block: every row is finished by
    one warp, and its fp64 sums equal the oracle's left fold bit for bit."""
    n = 4096
    A = random_rowlen_csr(n, n, np.full(n, 8), seed=11)
    B = random_rowlen_csr(n, 64, np.random.default_rng(12).integers(16, 32, n), seed=12)
    out, info = run(A, B, np.float64)
    ref = check(out, A, B, np.float64)
    assert info["nhash_blocks"] == info["nblocks"]
    assert (out[2] == ref.val).all(), "hash accumulator is not the left fold in A-entry order"


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_hash_shared_columns_across_waves(dt, cuda_available):
    """B rows drawn from few columns (and longer than a warp): every column collects
    products from many waves, added in expansion order (bit-exact left fold on rows
    inside one block)."""
    n = 600
    rng = np.random.default_rng(5)
    B = random_rowlen_csr(n, 70, rng.integers(16, 60, n), seed=7)
    A = random_rowlen_csr(300, n, rng.integers(1, 30, 300), seed=6)
    out, info = run(A, B, dt)
    ref = check(out, A, B, dt)
    assert info["nhash_blocks"] == info["nblocks"]
    if dt == np.float64:
        # rows inside one block are bit-exact (left fold); blocks of 512 nonzeros are
        # counted from each canonical segment's first nonzero (reading R21)
        rp = A.row_ptr.astype(np.int64)
        seg = alg.canonical_segments(A.row_ptr, 8)
        s_of = np.searchsorted(np.asarray(seg[1:]), np.arange(A.rows), side="right")
        base = rp[np.asarray(seg)[s_of]]
        inside = ((rp[:-1] - base) // 512) == ((rp[1:] - 1 - base) // 512)
        crp = ref.row_ptr.astype(np.int64)
        assert inside.sum() > 200
        for i in np.nonzero(inside)[0]:
            s, e = crp[i], crp[i + 1]
            assert (out[2][s:e] == ref.val[s:e]).all()


def test_hash_empty_b_rows(cuda_available):
    """Entries whose B rows are empty add no waves, including runs of them and empty
    first/last entries of a row, and rows whose B rows are all empty."""
    n = 2000
    rng = np.random.default_rng(8)
    blen = rng.integers(24, 32, n)
    blen[rng.random(n) < 0.6] = 0
    blen[100:200] = 0                       # long run of empty B rows
    B = random_rowlen_csr(n, 40, blen, seed=9)
    r, c = [], []
    for i in range(400):
        k = rng.choice(n, size=int(rng.integers(1, 16)), replace=False)
        if i % 3 == 0:
            k = np.concatenate([k, np.arange(100, 160)])   # > 32 consecutive empty entries
        if i % 7 == 0:
            k = np.arange(120, 140)                          # only empty B rows
        k = np.unique(k)
        r += [i] * len(k)
        c += k.tolist()
    A = from_coo(400, n, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))
    out, info = run(A, B, np.float64)
    check(out, A, B, np.float64)
    assert info["nhash_blocks"] > 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_short_b_rows_stay_in_esc(dt, cuda_available):
    """Blocks whose waves would leave most lanes idle (B rows of 1..8 entries) are not
    hash candidates: AC-ESC computes them."""
    rng = np.random.default_rng(2)
    A = random_rowlen_csr(2000, 3000, rng.integers(1, 40, 2000), seed=3)
    B = random_rowlen_csr(3000, 2500, rng.integers(1, 9, 3000), seed=4)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["nhash_blocks"] == 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_hash_overflow_falls_back_to_esc(dt, cuda_available):
    """A row with more than HASH_UMAX = 256 distinct columns inside an otherwise
    compacting block sends the block to AC-ESC; blocks without such rows stay in the
    hash accumulator; the result is the same C as the ESC-only strategy's."""
    rng = np.random.default_rng(3)
    nb = 4000
    # B rows 0..1999 draw from 60 columns (compacting), rows 2000.. from 20000 (wide)
    lens = rng.integers(17, 32, nb)
    r, c = [], []
    for i in range(nb):
        span = 60 if i < 2000 else 20000
        cols = np.sort(rng.choice(span, size=int(lens[i]), replace=False))
        r += [i] * len(cols)
        c += cols.tolist()
    B = from_coo(nb, 20000, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))
    r, c = [], []
    for i in range(3000):
        if i in (700, 1500, 2300):
            k = rng.choice(np.arange(2000, nb), size=40, replace=False)   # ~950 distinct columns
        else:
            k = rng.choice(2000, size=int(rng.integers(1, 8)), replace=False)
        k = np.sort(k)
        r += [i] * len(k)
        c += k.tolist()
    A = from_coo(3000, nb, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert 0 < info["nhash_blocks"] <= info["nblocks"] - 3
    esc, info_e = run(A, B, dt, strategy="esc")
    check(esc, A, B, dt)
    assert info_e["nhash_blocks"] == 0
    assert (esc[0] == out[0]).all() and (esc[1] == out[1]).all()


@pytest.mark.parametrize("strategy", ["adaptive", "esc"])
@pytest.mark.parametrize("case", ["poisson2d", "poisson27", "rmat", "powerlaw", "random"])
def test_strategies_parity(strategy, case, cuda_available):
    if case == "poisson2d":
        A = B = poisson2d_5pt(64); exact = True
    elif case == "poisson27":
        A = B = poisson3d_27pt(14); exact = True
    elif case == "rmat":
        A = B = rmat(scale=12, edge_factor=16, values="uniform"); exact = False
    elif case == "powerlaw":
        A = B = power_law_csr(3000, 3000, mean_len=12, alpha=1.4, max_len=900, seed=21); exact = False
    else:
        A = random_csr(2500, 1800, 0.01, seed=31); B = random_csr(1800, 2200, 0.01, seed=32); exact = False
    for dt in (np.float64, np.float32):
        assert_parity(A, B, dt, exact=exact and dt == np.float64, strategy=strategy)


def test_hash_bit_stable_runs_and_splits(cuda_available):
    """The adaptive strategy is bit-identical run to run and for every segment count."""
    p = pkg()
    A = poisson3d_27pt(20)
    A.val[:] = np.random.default_rng(1).uniform(-1, 1, A.val.shape)
    hs = set()
    for nseg in (1, 2, 8, 8, 37):
        plan = p.Plan(num_segments=nseg)
        dA = p.DeviceCSR.from_host(A, "cuda", np.float64)
        C = plan.multiply(dA, dA)
        torch.cuda.synchronize()
        if nseg == 8:
            hs.add(digest(*C.to_numpy()))
        assert plan.info()["nhash_blocks"] >= 0.9 * plan.info()["nblocks"]
        check(C.to_numpy(), A, A, np.float64)
        plan.close()
    assert len(hs) == 1


def test_hash_stencil_square_exact(cuda_available):
    """27-point stencil squared (integer values): every block is finished by the hash
    accumulator and the result is exact."""
    A = poisson3d_27pt(24)
    out, info = run(A, A, np.float64)
    ref = check(out, A, A, np.float64)
    assert info["nhash_blocks"] == info["nblocks"]
    assert (out[2] == ref.val).all()


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_hash_row_reuse_sentinel_corners(dt, cuda_available):
    """Row-relative keys (reading R41): a warp keeps its keys from row to row and a row
    whose touched slots equal the previous row's reuses its column order.  A value that
    reads like an untouched slot after it was touched -- a column whose products are all
    -0.0, or (fp64) a sum in (-2^-1042, 0) that shares -0.0's high word -- must not
    corrupt the row: such blocks go to AC-ESC.  The 27-point stencil's boundary rows
    (subsets of the interior pattern), a few random rows between translate-equal ones,
    and values equal to the oracle everywhere; the same bits run to run."""
    A = poisson3d_27pt(14)
    B = poisson3d_27pt(14)
    rng = np.random.default_rng(41)
    aval = np.abs(rng.uniform(0.5, 1.5, A.nnz))
    bval = rng.uniform(-1, 1, B.nnz)
    bval[np.isin(B.col, [300, 301, 1500])] = -0.0          # all products -0.0 (A > 0)
    if dt == np.float64:
        bval[np.isin(B.col, [900, 2200])] = -1e-321        # sums share -0.0's high word
    A = synth_csr(A, aval)
    B = synth_csr(B, bval)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["nhash_blocks"] > 0
    out2, _ = run(A, B, dt)
    assert digest(*out) == digest(*out2)
    # rows of a banded pattern with random rows in between (reuse on, off, on again)
    n = 3000
    r, c = [], []
    for i in range(n):
        cols = np.arange(i - 10, i + 11) if i % 50 else rng.choice(n, 21, replace=False)
        cols = np.unique(np.clip(cols, 0, n - 1))
        r += [i] * len(cols)
        c += cols.tolist()
    M = from_coo(n, n, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))
    out, info = run(M, M, dt)
    check(out, M, M, dt)
    assert info["nhash_blocks"] > 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_hash_stale_keys_clear_and_rerun(dt, cuda_available):
    """Rows whose row-relative patterns drift (row i's columns are [12i, 12i + 126): the
    relative keys shift by 11 per row) fill a warp's table with earlier rows' keys; after
    about 12 rows a row would push it past HASH_UMAX keys, clears the table and runs again
    (reading R41).  Every block stays with the hash accumulator and C equals the
    oracle's.  (Rows of 9 entries: the candidate test samples adjacent entries 63 apart,
    which rows of 8 would put on row boundaries.)"""
    n = 3000
    r = np.repeat(np.arange(n), 9)
    c = (np.arange(n)[:, None] + np.arange(9)[None, :]).ravel()
    rng = np.random.default_rng(17)
    A = from_coo(n, n + 9, r, c, rng.uniform(-1, 1, len(r)))
    rb = np.repeat(np.arange(n + 9), 30)
    cb = (12 * np.arange(n + 9)[:, None] + np.arange(30)[None, :]).ravel()
    B = from_coo(n + 9, 12 * (n + 9) + 30, rb, cb, rng.uniform(-1, 1, len(rb)))
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["nhash_blocks"] == info["nblocks"]
    out2, _ = run(A, B, dt)
    assert digest(*out) == digest(*out2)


def synth_csr(M, val):
    from synth import CSR
    return CSR(M.rows, M.cols, M.row_ptr, M.col, np.asarray(val, dtype=M.val.dtype))


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_low_compaction_rows_go_to_esc(dt, cuda_available):
    """Rows whose products hardly compact (random columns: adjacent entries' B rows share
    almost no columns) are not hash candidates; AC-ESC computes them."""
    rng = np.random.default_rng(12)
    A = random_rowlen_csr(1500, 4000, rng.integers(10, 20, 1500), seed=13)
    B = random_rowlen_csr(4000, 200000, rng.integers(24, 32, 4000), seed=14)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["nhash_blocks"] == 0


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_small_tile_esc_blocks(dt, cuda_available):
    """Blocks of <= 512 products that are not hash candidates run the small-tile AC-ESC
    (reading R32), the others the default tile: A·P of a 7-point stencil and an
    aggregation prolongator (exact, one product per A entry) next to denser rows."""
    from synth import aggregation_prolongator, poisson3d_7pt
    A = poisson3d_7pt(16)
    P = aggregation_prolongator(16)
    out, info = run(A, P, dt)
    ref = check(out, A, P, dt)
    assert info["nhash_blocks"] == 0
    assert (out[2].astype(np.float64) == ref.val).all()
    # mixed: short random rows (small blocks) and long ones (default tile)
    rng = np.random.default_rng(21)
    lens = np.where(rng.random(3000) < 0.5, 1, rng.integers(30, 120, 3000))
    lens[:1200] = 1
    A2 = random_rowlen_csr(3000, 2500, lens, seed=22)
    B2 = random_rowlen_csr(2500, 2600, rng.integers(1, 6, 2500), seed=23)
    out2, info2 = run(A2, B2, dt)
    check(out2, A2, B2, dt)
    esc2, _ = run(A2, B2, dt, strategy="esc")
    assert (esc2[0] == out2[0]).all() and (esc2[1] == out2[1]).all()
