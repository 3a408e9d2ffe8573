"""GPU parity: the CUDA path through the C ABI against the CPU oracle, element by
element, on seeded inputs spanning several tiles and ragged tails.

Bar (BASELINE.json north_star): structure (row_ptr, col_idx) bit-exact; values within
|c - c_ref| <= 1e-12·Σ|a·b| (fp64) / 1e-5·Σ|a·b| (fp32); integer-valued inputs whose
partial sums stay below 2^24 bit-exact; GPU results bit-identical across runs and
across canonical-segment splits (1/2/4/8 GPUs emulated on one device).
"""
import hashlib

import numpy as np
import pytest
import torch

import oracle
from oracle import alg
from synth import (CSR, aggregation_prolongator, from_coo, lp_like, poisson2d_5pt, poisson3d_27pt,
                   poisson3d_7pt, power_law_csr, random_csr, random_rowlen_csr, rmat, transpose)

pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


def pkg():
    import paper_conf_ppopp_wintermzss19_b200 as p
    return p


def gpu_mult(A, B, dt, plan=None, **kw):
    p = pkg()
    dA = p.DeviceCSR.from_host(A, "cuda", dt)
    dB = p.DeviceCSR.from_host(B, "cuda", dt)
    if plan is None:
        C = p.multiply(dA, dB, **kw)
    else:
        C = plan.multiply(dA, dB)
    torch.cuda.synchronize()
    return C.to_numpy()


def assert_parity(A, B, dt, exact=False, oracle_threads=0, **kw):
    rp, col, val = gpu_mult(A, B, dt, **kw)
    ref = oracle.gustavson(A.astype(dt), B.astype(dt), threads=oracle_threads)
    assert rp.shape[0] == ref.row_ptr.shape[0]
    assert (rp == ref.row_ptr).all(), "row_ptr mismatch"
    assert (col == ref.col).all(), "col mismatch"
    v = val.astype(np.float64)
    if exact:
        assert (v == ref.val).all(), "values not bit-exact on integer data"
    else:
        err = np.abs(v - ref.val)
        bad = err > TOL[dt] * ref.absval
        assert not bad.any(), f"{bad.sum()} values out of tolerance; max rel {(err / np.maximum(ref.absval, 1e-300)).max()}"
    return rp, col, val


def digest(rp, col, val):
    h = hashlib.sha256()
    for a in (rp, col, val):
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()


# ------------------------------------------------------------ whole multiply --

@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("seed", range(6))
def test_random_small(dt, seed, cuda_available):
    rng = np.random.default_rng(seed)
    m, k, n = (int(x) for x in rng.integers(1, 400, 3))
    A = random_csr(m, k, float(rng.uniform(0.001, 0.08)), seed=seed, empty_rows=0.1)
    B = random_csr(k, n, float(rng.uniform(0.001, 0.08)), seed=seed + 50)
    assert_parity(A, B, dt)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_cfg1_poisson2d_exact(dt, cuda_available):
    """configs[0]: 2D 5-point 64², A·A; integer-valued -> bit-exact."""
    A = poisson2d_5pt(64)
    rp, col, val = assert_parity(A, A, dt, exact=True)
    assert rp[-1] == 51972


def test_poisson27_small_exact(cuda_available):
    """27-point stencil at n=20 (8,000 rows, ~190K nnz: ~370 blocks, ~7 ESC iterations
    per block, 2-chunk shared rows at every block boundary)."""
    A = poisson3d_27pt(20)
    rp, col, val = assert_parity(A, A, np.float64, exact=True)
    assert rp[-1] == (5 * 20 - 6) ** 3


def test_poisson27_uniform_values(cuda_available):
    A = poisson3d_27pt(14)
    A.val = np.random.default_rng(2).uniform(-1, 1, A.nnz)
    for dt in (np.float64, np.float32):
        assert_parity(A, A, dt)


def test_galerkin_rap_exact(cuda_available):
    """configs[3] shape at n=16: AP = A·P then RAP = R·(AP) = 4·A₇(n/2) exactly."""
    n = 16
    A, P = poisson3d_7pt(n), aggregation_prolongator(n)
    R = transpose(P)
    rp, col, val = assert_parity(A, P, np.float64, exact=True)
    AP = CSR(A.rows, P.cols, rp, col, val)
    rp2, col2, val2 = assert_parity(R, AP, np.float64, exact=True)
    A4 = poisson3d_7pt(n // 2)
    assert (rp2 == A4.row_ptr).all() and (col2 == A4.col).all() and (val2 == 4 * A4.val).all()


@pytest.mark.parametrize("seed", range(3))
def test_long_rows_multi_chunk(seed, cuda_available):
    """Skewed rows: C rows far longer than KEEP, split over many chunks -> Path and
    Search Merge; B rows longer than CAP split by the work distribution (L210)."""
    A = power_law_csr(3000, 3000, mean_len=12, alpha=1.2, max_len=1500, seed=seed)
    B = power_law_csr(3000, 3000, mean_len=12, alpha=1.2, max_len=3000, seed=seed + 10)
    plan = pkg().Plan()
    assert_parity(A, B, np.float64, plan=plan)
    info = plan.info()
    assert info["nshared"] > 0
    assert info["npath"] + info["nsearch"] > 0


@pytest.mark.parametrize("ncols_log2", [11, 12, 13])
def test_path_merge_windows_dense_columns(ncols_log2, cuda_available):
    """Path Merge windows over rows that fill a power-of-two column range: the window's
    largest key reaches 2^k - 1, padding words sit between the pieces' entries, and the
    proportional staging cut (reading R12) must still rank them last."""
    n = 1 << ncols_log2
    rows, k = 8, 1500
    rng = np.random.default_rng(ncols_log2)
    r = np.repeat(np.arange(rows), k)
    c = np.concatenate([np.sort(rng.choice(6000, k, replace=False)) for _ in range(rows)])
    A = from_coo(rows, 6000, r, c, rng.uniform(-1, 1, rows * k))
    # 1500 x 5 = 7,500 products per row: several chunks, at most 4 windows (Path Merge;
    # longer dense rows go to the dense slices of reading R30)
    B = random_rowlen_csr(6000, n, np.full(6000, 5), seed=ncols_log2, values="uniform")
    plan = pkg().Plan()
    assert_parity(A, B, np.float64, plan=plan)
    assert plan.info()["npath"] >= 1


def test_path_merge_window_all_ones_key(cuda_available):
    """Deterministic Path Merge window whose largest key is all ones in its bit width.
    A = one row (1, 1, 1); B rows of exactly CAP entries, so each ESC iteration emits one
    B row as one chunk of C's row 0 (three pieces).  Proportional staging takes 682
    entries per piece; piece 1's next column 1024 is the cut and lo = 0, so the window's
    largest key is 1023 = 2^10 - 1 (piece 2) while piece 0's staged entries >= 1024 are
    padding words in front of it: the sorted bits must rank the padding after 1023."""
    rows = [list(range(0, 600)) + list(range(2000, 3448)),
            list(range(0, 682)) + list(range(1024, 2390)),
            list(range(300, 981)) + [1023] + list(range(3000, 4366))]
    assert all(len(r) == 2048 for r in rows)
    rng = np.random.default_rng(5)
    B = from_coo(3, 5000, np.repeat(np.arange(3), 2048), np.concatenate(rows), rng.uniform(-1, 1, 3 * 2048))
    A = from_coo(1, 3, [0, 0, 0], [0, 1, 2], np.array([1.0, -2.0, 0.5]))
    plan = pkg().Plan()
    assert_parity(A, B, np.float64, plan=plan)
    info = plan.info()
    assert info["npath"] == 1 and info["nchunks"] == 3


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_giant_row_dense_slices(dt, cuda_available):
    """A row gathering 2.2M products over a 200K-column range is split into more than
    SEARCH_MAXP chunks and merged by dense column slices (reading R30); small rows and an
    empty row around it take the other paths."""
    n_b, ncol = 70000, 200000
    rng = np.random.default_rng(17)
    rows = [0] * n_b + [1, 1, 3]
    cols = list(range(n_b)) + [5, 9, 11]
    A = from_coo(4, n_b, rows, cols, rng.uniform(-1, 1, len(rows)))
    B = random_rowlen_csr(n_b, ncol, np.full(n_b, 32), seed=18, values="uniform")
    plan = pkg().Plan()
    assert_parity(A, B, dt, plan=plan)
    info = plan.info()
    assert info["nsearch"] >= 1 and info["nchunks"] > 1024


def test_dense_row_search_merge(cuda_available):
    """One very long output row (> PATH_MAX_CHUNKS chunks) forces Search Merge."""
    n = 60000
    A = from_coo(2, n, [0] * 3000 + [1] * 5, list(range(0, 60000, 20)) + [1, 2, 3, 4, 5],
                 np.ones(3005))
    B = random_rowlen_csr(n, n, np.full(n, 30), seed=3, values="int")
    plan = pkg().Plan()
    assert_parity(A, B, np.float64, plan=plan)
    assert plan.info()["nsearch"] >= 1


def test_rmat_small(cuda_available):
    A = rmat(scale=12, edge_factor=16, values="uniform")
    assert_parity(A, A, np.float64)
    assert_parity(A.astype(np.float32), A.astype(np.float32), np.float32)
    Ao = rmat(scale=12, edge_factor=16, values="ones")
    assert_parity(Ao, Ao, np.float64, exact=True)


def test_lp_like_small(cuda_available):
    A, At = lp_like(rows_log2=10, cols_log2=12, per_col=20, seed=7)
    assert_parity(A, At, np.float64)


def test_edge_cases(cuda_available):
    # empty A, empty rows, A·0, 1x1, rectangular, single dense column
    Z = random_csr(50, 40, 0.0, seed=1)
    B = random_csr(40, 30, 0.2, seed=2)
    assert_parity(Z, B, np.float64)
    assert_parity(B.astype(np.float64), random_csr(30, 20, 0.0, seed=3), np.float64)
    one = from_coo(1, 1, [0], [0], np.array([3.0]))
    assert_parity(one, one, np.float64, exact=True)
    col = from_coo(500, 1, np.arange(500), np.zeros(500), np.arange(1.0, 501.0))
    row = from_coo(1, 500, np.zeros(500), np.arange(500), np.arange(1.0, 501.0))
    assert_parity(col, row, np.float64, exact=True)       # outer product: 250,000 entries
    assert_parity(row, col, np.float64)                   # dot product: one 500-term entry
    # rows exactly at block boundaries
    for L in (511, 512, 513, 1024):
        Ab = random_rowlen_csr(8, 4000, np.full(8, L), seed=L, values="int")
        Bb = random_rowlen_csr(4000, 300, np.full(4000, 3), seed=L + 1, values="int")
        assert_parity(Ab, Bb, np.float64, exact=True)


def test_dimension_mismatch(cuda_available):
    p = pkg()
    A = p.DeviceCSR.from_host(random_csr(5, 6, 0.5, seed=1), "cuda", np.float64)
    with pytest.raises(p.AcspgemmError):
        p.multiply(A, A)


def test_validate_inputs(cuda_available):
    p = pkg()
    bad = CSR(2, 3, np.array([0, 2, 3], np.int32), np.array([2, 1, 0], np.int32), np.ones(3))
    dB = p.DeviceCSR.from_host(random_csr(3, 3, 0.6, seed=1), "cuda", np.float64)
    dA = p.DeviceCSR.from_host(bad, "cuda", np.float64)
    with pytest.raises(p.AcspgemmError):
        p.multiply(dA, dB, validate=True)


def test_lib_alloc_multiply(cuda_available):
    p = pkg()
    A = poisson2d_5pt(20)
    dA = p.DeviceCSR.from_host(A, "cuda", np.float64)
    rp, col, val = p.multiply_lib_alloc(dA, dA)
    ref = oracle.gustavson(A, A)
    assert (rp == ref.row_ptr).all() and (col == ref.col).all() and (val == ref.val).all()


# ------------------------------------------------------------- determinism ---

def test_bit_stable_repeated_runs(cuda_available):
    A = power_law_csr(4000, 4000, mean_len=10, alpha=1.3, max_len=1200, seed=5)
    hs = {digest(*gpu_mult(A, A, np.float64)) for _ in range(3)}
    plan = pkg().Plan()
    hs |= {digest(*gpu_mult(A, A, np.float64, plan=plan)) for _ in range(2)}
    assert len(hs) == 1


@pytest.mark.parametrize("G", [2, 4, 8])
def test_bit_identical_across_gpu_counts(G, cuda_available):
    """Emulate G GPUs on one device: rank g runs canonical segments [g·S/G, (g+1)·S/G)
    of A as a row-range view; concatenated pieces must equal the 1-GPU C byte for byte."""
    p = pkg()
    A = power_law_csr(5000, 5000, mean_len=10, alpha=1.3, max_len=1500, seed=9)
    dA = p.DeviceCSR.from_host(A, "cuda", np.float64)
    full = p.multiply(dA, dA)
    torch.cuda.synchronize()
    frp, fcol, fval = full.to_numpy()
    S = 8
    seg = p.canonical_segments(dA, S)
    assert seg == alg.canonical_segments(A.row_ptr, S)
    pieces = []
    for g in range(G):
        s0, s1 = g * S // G, (g + 1) * S // G
        r0, r1 = seg[s0], seg[s1]
        plan = p.Plan()
        plan.set_segments([r - r0 for r in seg[s0:s1 + 1]])
        view = p.api._csr_in(dA, row_ptr=dA.row_ptr[r0:r1 + 1].contiguous(), rows=r1 - r0,
                             nnz=int(A.row_ptr[r1] - A.row_ptr[r0]))
        C = plan.multiply(dA, dA, A_view=view)
        torch.cuda.synchronize()
        pieces.append(C.to_numpy())
        plan.close()
    off = 0
    rp_cat = [np.zeros(1, np.int64)]
    for rp, col, val in pieces:
        rp_cat.append(rp[1:].astype(np.int64) + off)
        off += rp[-1]
    rp_cat = np.concatenate(rp_cat)
    col_cat = np.concatenate([c for _, c, _ in pieces])
    val_cat = np.concatenate([v for _, _, v in pieces])
    assert (rp_cat == frp).all() and (col_cat == fcol).all()
    assert val_cat.tobytes() == fval.tobytes()


# ------------------------------------------------------------ single steps ---

def test_glb_block_row_starts(cuda_available):
    """Alg. 1 output vs the step oracle, per canonical segment."""
    p = pkg()
    A = random_rowlen_csr(3000, 500, np.random.default_rng(1).integers(0, 40, 3000), seed=2)
    dA = p.DeviceCSR.from_host(A, "cuda", np.float64)
    dB = p.DeviceCSR.from_host(random_csr(500, 400, 0.01, seed=3), "cuda", np.float64)
    plan = p.Plan()
    plan.symbolic(dA, dB)
    got = plan.block_row_starts()
    seg = alg.canonical_segments(A.row_ptr, 8)
    exp = []
    for s in range(8):
        r0, r1 = seg[s], seg[s + 1]
        exp += [r + r0 for r in alg.alg1_block_row_starts(A.row_ptr[r0:r1 + 1], p.const("NPB"),
                                                           nnz_base=int(A.row_ptr[r0]))]
    assert list(got) == exp
    info = plan.info()
    assert info["products"] == oracle.products(A, random_csr(500, 400, 0.01, seed=3))
    assert info["segment_rows"] == seg


def test_work_distribution_fig3(cuda_available):
    """Alg. 2 on the GPU reproduces the paper's Fig. 3 worked example."""
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "fig3_work_distribution.json")))
    ares, bres, rem = pkg().debug_work_distribution(g["lengths"], g["draws"])
    pairs = [[int(a), int(b)] for a, b in zip(ares, bres)]
    assert pairs == [x for d in g["pairs"] for x in d]
    assert rem.tolist() == g["remaining_after"]


@pytest.mark.parametrize("seed", range(6))
def test_work_distribution_random(seed, cuda_available):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 513))
    lens = rng.choice([0, 1, 2, 3, 7, 30, 300], size=n)
    total = int(lens.sum())
    draws = []
    left = total
    while left > 0:
        d = int(min(left, rng.integers(1, 2049)))
        draws.append(d)
        left -= d
    ares, bres, rem = pkg().debug_work_distribution(lens, draws)
    wd = alg.WorkDistribution(n)
    wd.placework(list(lens))
    A_, B_, R_ = [], [], []
    for d in draws:
        a, b = wd.receivework(d)
        A_ += a
        B_ += b
        R_.append(wd.remaining())
    assert list(ares) == A_ and list(bres) == B_ and rem.tolist() == R_


@pytest.mark.parametrize("seed", range(8))
def test_sort_compact_vs_alg3(seed, cuda_available):
    """Block radix sort + Alg. 3 scan on the GPU vs the sequential oracle scan."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 2049))
    span_r = int(rng.choice([1, 3, 40, 500]))
    span_c = int(rng.choice([1, 5, 100, 70000, 3_000_000]))
    rows = rng.integers(0, span_r, n).astype(np.int32)
    cols = rng.integers(0, span_c, n).astype(np.int32)
    vals = rng.integers(-9, 10, n).astype(np.float64)    # integer: sums exact in any order
    orow, ocol, oval, ost = pkg().debug_sort_compact(rows, cols, vals)
    order = np.lexsort((np.arange(n), cols, rows))        # stable sort by (row, col)
    assert (orow == rows[order]).all() and (ocol == cols[order]).all()
    keys = list(zip(orow.tolist(), ocol.tolist()))
    ref = alg.compaction_scan(orow.tolist(), keys, vals[order].tolist())
    assert [r[3] for r in ref] == ost.tolist()
    runend = (ost & 1).astype(bool)
    assert (oval[runend] == np.array([r[2] for r in ref])[runend]).all()


@pytest.mark.parametrize("dt", [np.float64, np.float32])
@pytest.mark.parametrize("ncols_log2", [16, 24])
def test_wide_column_ranges(ncols_log2, dt, cuda_available):
    """Column ranges that need 32-bit sort words (16) and the split 32-bit + side-array
    words (24) in AC-ESC; B has few rows with columns spread over 2^ncols_log2.  (The
    oracle's dense accumulator is as wide as C: one oracle thread keeps it small.)"""
    rng = np.random.default_rng(ncols_log2)
    K, ncols = 64, 1 << ncols_log2
    A = random_rowlen_csr(600, K, rng.integers(1, 40, 600), seed=ncols_log2)
    rows, cols = [], []
    for r in range(K):
        c = np.unique(rng.integers(0, ncols, int(rng.integers(1, 200))))
        rows.append(np.full(c.size, r))
        cols.append(c)
    rows, cols = np.concatenate(rows), np.concatenate(cols)
    B = from_coo(K, ncols, rows, cols, rng.uniform(-1, 1, rows.size))
    assert_parity(A, B, dt, oracle_threads=1)
    Bi = from_coo(K, ncols, rows, cols, rng.integers(-3, 4, rows.size).astype(np.float64))
    Ai = random_rowlen_csr(600, K, rng.integers(1, 40, 600), seed=ncols_log2 + 1, values="int")
    assert_parity(Ai, Bi, dt, exact=True, oracle_threads=1)


def test_64bit_sort_words(cuda_available):
    """Keys wider than the split path (> 36 bits): 512 one-entry rows per block (9 row
    bits) times columns spread over 2^28 -> 64-bit sort words."""
    rng = np.random.default_rng(5)
    K, ncols = 32, 1 << 28
    A = from_coo(4096, K, np.arange(4096), rng.integers(0, K, 4096), rng.integers(1, 4, 4096).astype(np.float64))
    rows = np.repeat(np.arange(K), 4)
    cols = np.concatenate([np.sort(rng.choice(ncols, 4, replace=False)) for _ in range(K)])
    B = from_coo(K, ncols, rows, cols, rng.integers(-3, 4, rows.size).astype(np.float64))
    assert_parity(A, B, np.float64, exact=True, oracle_threads=1)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_long_row_chunks(dt, cuda_available):
    """§3.4 long rows (L546-L548): entries whose B row has more than CAP = 2048 entries
    become their own chunk (a·B_k, no sort) placed where their products belong.  Rows
    made of one long entry (C row = a·B_k, no merge), long entries first / in the middle /
    last among short ones, several per row, rows of only long entries, long entries at
    block boundaries, and a block with more long entries than PTR_MAX (the rest go
    through AC-ESC).  Integer values: exact; U(-1,1): within tolerance."""
    rng = np.random.default_rng(21)
    nb, ncols = 400, 6000
    blen = rng.integers(5, 60, nb)
    blen[rng.choice(nb, 60, replace=False)] = rng.integers(2049, 5000, 60)   # long B rows
    long_rows = np.flatnonzero(blen > 2048)
    short_rows = np.flatnonzero(blen <= 2048)
    r, c = [], []
    for i in range(1200):
        kind = i % 6
        if kind == 0:
            k = [rng.choice(long_rows)]                                   # a single long entry
        elif kind == 1:
            k = list(rng.choice(short_rows, 5, replace=False)) + [rng.choice(long_rows)]
        elif kind == 2:
            k = list(rng.choice(long_rows, 3, replace=False))              # only long entries
        elif kind == 3:
            k = list(rng.choice(short_rows, 8, replace=False))
        else:
            k = list(rng.choice(short_rows, 6, replace=False)) + list(rng.choice(long_rows, 2, replace=False))
        k = np.unique(k)
        r += [i] * len(k)
        c += k.tolist()
    # rows 1200..1399: 200 consecutive single long entries (> PTR_MAX = 160 in a block)
    for i in range(1200, 1400):
        r.append(i)
        c.append(int(long_rows[i % len(long_rows)]))
    rr, cc = np.array(r), np.array(c)
    for values in ("int", "uniform"):
        if values == "int":
            va = rng.integers(1, 4, rr.size) * rng.choice([-1.0, 1.0], rr.size)
        else:
            va = rng.uniform(-1, 1, rr.size)
        A = from_coo(1400, nb, rr, cc, va)
        rows_b = np.repeat(np.arange(nb), blen)
        cols_b = np.concatenate([np.sort(rng.choice(ncols, L, replace=False)) for L in blen])
        vb = rng.integers(-3, 4, rows_b.size).astype(np.float64) if values == "int" else rng.uniform(-1, 1, rows_b.size)
        B = from_coo(nb, ncols, rows_b, cols_b, vb)
        assert_parity(A, B, dt, exact=(values == "int"))
