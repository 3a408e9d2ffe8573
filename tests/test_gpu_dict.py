"""GPU parity of the column-dictionary accumulator (reading R33, csrc/dict.cu): the first
accumulator the adaptive strategy offers a candidate block (§5, SURVEY
§8(f)-4), through the C ABI.

What pins it:
  * against the CPU oracle: structure bit-exact, values within the north-star tolerance,
    fp64 rows inside one block bit-identical to the oracle's left fold (Gustavson order);
  * against the hash accumulator (strategy "hash" = adaptive without the dictionary):
    byte-identical C -- both sum every column left to right in A-entry order from -0.0;
  * the fallbacks (dictionary wider than 768 columns, column span beyond 131,072, more
    than 7,168 staged B entries) leave the block to the hash accumulator with the same
    bits; structural zeros from cancellation are kept (reading R2);
  * the default strategy offers the blocks to the hash accumulator (same bits); these
    tests force the dictionary with strategy "dict".
"""
import numpy as np
import pytest
import torch

import oracle
from synth import from_coo, poisson3d_27pt, random_rowlen_csr

from test_gpu_parity import TOL, pkg

pytestmark = pytest.mark.gpu


def run(A, B, dt, strategy="dict", nseg=8):
    p = pkg()
    plan = p.Plan(strategy=strategy, num_segments=nseg)
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


def same_bytes(x, y):
    return all(a.tobytes() == b.tobytes() for a, b in zip(x, y))


def banded_b(nb, ncols, stride, width, rng, far=None):
    """B row k holds `width` consecutive columns from k*stride (mod the column range),
    plus column `far(k)` when given; U(-1,1) values."""
    r, c = [], []
    for k in range(nb):
        cols = (k * stride + np.arange(width)) % ncols
        if far is not None:
            cols = np.concatenate([cols, [far(k) % ncols]])
        cols = np.unique(cols)
        r += [k] * len(cols)
        c += cols.tolist()
    return from_coo(nb, ncols, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))


def window_a(n, nb, per_row, rng):
    """A row i holds the per_row consecutive B rows from i (clipped): adjacent entries
    share most of their B columns (hash candidates)."""
    r, c = [], []
    for i in range(n):
        k = np.arange(i, min(i + per_row, nb))
        r += [i] * len(k)
        c += k.tolist()
    return from_coo(n, nb, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_dict_stencil_all_blocks(dt, cuda_available):
    """27-point stencil squared with U(-1,1) values: every block is finished by the
    dictionary accumulator, C equals the hash accumulator's byte for byte."""
    A = poisson3d_27pt(20)
    A.val[:] = np.random.default_rng(4).uniform(-1, 1, A.val.shape)
    out, info = run(A, A, dt)
    check(out, A, A, dt)
    assert info["ndict_blocks"] == info["nblocks"] == info["nhash_blocks"]
    hsh, info_h = run(A, A, dt, strategy="hash")
    assert info_h["ndict_blocks"] == 0 and info_h["nhash_blocks"] == info["nblocks"]
    assert same_bytes(out, hsh)
    dflt, info_a = run(A, A, dt, strategy="adaptive")
    assert info_a["ndict_blocks"] == 0 and info_a["nhash_blocks"] == info["nblocks"]   # adaptive: hash (R31)
    assert same_bytes(out, dflt)


def test_dict_stencil_exact(cuda_available):
    """Integer 27-point stencil squared: exact values (partial sums are integers)."""
    A = poisson3d_27pt(24)
    out, info = run(A, A, np.float64)
    ref = check(out, A, A, np.float64)
    assert info["ndict_blocks"] == info["nblocks"]
    assert (out[2] == ref.val).all()


def test_dict_left_fold_bit_exact_fp64(cuda_available):
    """Rows of 8 entries never straddle a block: fp64 values equal the oracle's left fold
    in A-entry order bit for bit."""
    n, nb = 4096, 200                      # <= 200 distinct B rows per block: staged <= 6,400
    A = random_rowlen_csr(n, nb, np.full(n, 8), seed=11)
    B = random_rowlen_csr(nb, 64, np.random.default_rng(12).integers(16, 31, nb), seed=12)
    out, info = run(A, B, np.float64)
    ref = check(out, A, B, np.float64)
    assert info["ndict_blocks"] == info["nblocks"]
    assert (out[2] == ref.val).all()


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_dict_long_b_rows(dt, cuda_available):
    """B rows longer than a warp (several waves per entry) sharing few columns."""
    rng = np.random.default_rng(5)
    n = 90                                 # <= 90 distinct B rows of <= 64: staged <= 5,760
    B = random_rowlen_csr(n, 90, rng.integers(33, 65, n), seed=7)
    A = random_rowlen_csr(300, n, rng.integers(1, 30, 300), seed=6)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["ndict_blocks"] == info["nblocks"]
    hsh, _ = run(A, B, dt, strategy="hash")
    assert same_bytes(out, hsh)


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_dict_wide_dictionary_falls_back(dt, cuda_available):
    """B rows of 32 columns, shifted by 16 per row: adjacent B rows share half of their
    columns (candidates), but a block's rows reach > 768 distinct columns; the blocks go
    to the hash accumulator, with the same bits."""
    rng = np.random.default_rng(9)
    nb = 3000
    B = banded_b(nb, 16 * nb + 64, 16, 32, rng)
    A = window_a(2000, nb, 8, rng)
    out, info = run(A, B, dt)
    check(out, A, B, dt)
    assert info["ndict_blocks"] == 0 and info["nhash_blocks"] > 0
    hsh, _ = run(A, B, dt, strategy="hash")
    assert same_bytes(out, hsh)


def test_dict_span_falls_back(cuda_available):
    """Every B row also holds a column ~200,000 away: the block's column span exceeds
    131,072 and the block goes to the hash accumulator (same bits)."""
    rng = np.random.default_rng(10)
    nb = 2000
    B = banded_b(nb, 400000, 2, 30, rng, far=lambda k: 2 * k + 200000 + (k % 7))
    A = window_a(1500, nb, 12, rng)
    out, info = run(A, B, np.float64)
    check(out, A, B, np.float64)
    assert info["ndict_blocks"] == 0 and info["nhash_blocks"] == info["nblocks"]
    hsh, _ = run(A, B, np.float64, strategy="hash")
    assert same_bytes(out, hsh)


def test_dict_staging_limit_falls_back(cuda_available):
    """Blocks whose distinct B rows hold more than 7,168 staged entries (B rows of 60
    columns padded to 64,
    every A entry a different B row) leave the dictionary; others in the same multiply
    stay (a mix of dictionary and hash blocks)."""
    rng = np.random.default_rng(14)
    nb = 6000
    B = banded_b(nb, 2 * nb + 200, 2, 60, rng)
    # rows 0..999: 12 consecutive B rows each (few distinct B rows per block);
    # rows 1000..1499: 24 B rows each, 8 apart: a block's distinct rows exceed 7168/64
    r, c = [], []
    for i in range(1500):
        if i < 1000:
            k = np.arange(i, i + 12)
        else:
            k = 1000 + (i - 1000) * 8 + np.arange(24)
        r += [i] * len(k)
        c += k.tolist()
    A = from_coo(1500, nb, np.array(r), np.array(c), rng.uniform(-1, 1, len(r)))
    out, info = run(A, B, np.float64)
    check(out, A, B, np.float64)
    assert 0 < info["ndict_blocks"] < info["nhash_blocks"]
    hsh, _ = run(A, B, np.float64, strategy="hash")
    assert same_bytes(out, hsh)


def test_dict_keeps_structural_zeros(cuda_available):
    """C = A·B with A rows (1, -1) on two B rows of equal values: every entry cancels to
    zero and is kept (reading R2: ESC compares keys, never values)."""
    n, nb = 800, 801
    r = np.repeat(np.arange(n), 2)
    c = np.stack([np.arange(n), np.arange(n) + 1], 1).ravel()
    v = np.tile([1.0, -1.0], n)
    A = from_coo(n, nb, r, c, v)
    B = from_coo(nb, 40, np.repeat(np.arange(nb), 20), np.tile(np.arange(20), nb), np.full(20 * nb, 0.375))
    out, info = run(A, B, np.float64)
    ref = check(out, A, B, np.float64)
    assert info["ndict_blocks"] == info["nblocks"]
    assert len(out[1]) == 20 * n and (out[2] == 0).all() and (ref.val == 0).all()


def test_dict_bit_stable_across_segments(cuda_available):
    """Bit-identical run to run and for every canonical segment count (1, 2, 8, 37)."""
    A = poisson3d_27pt(18)
    A.val[:] = np.random.default_rng(1).uniform(-1, 1, A.val.shape)
    ref8, _ = run(A, A, np.float64, nseg=8)
    again, _ = run(A, A, np.float64, nseg=8)
    assert same_bytes(ref8, again)
    for nseg in (1, 2, 37):
        out, info = run(A, A, np.float64, nseg=nseg)
        check(out, A, A, np.float64)
        assert info["ndict_blocks"] >= info["nblocks"] - nseg   # short segment tails: few entries
