"""Seeded synthetic CSR generators for the paper's workload classes.

This module is shared by the oracle tests, the CUDA parity tests and bench.py.
It holds NO SpGEMM arithmetic: it only builds input matrices (structure and
values) and the untimed transposes the paper precomputes ("We compute A·A for
square matrices and A·Aᵀ for non-square, where we precompute Aᵀ", PAPER.md
L554 §4).  Recipes follow SURVEY.md Appendix A; DESIGN.md §"Input recipe"
restates them.

All matrices are canonical CSR (§1: "Entries are sorted according
to rows"; columns ascending and unique within a row, SURVEY §8(c) reading 3),
with int32 row_ptr / col_idx and float64 or float32 values.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class CSR:
    rows: int
    cols: int
    row_ptr: np.ndarray  # int32 or int64 [rows+1]
    col: np.ndarray      # int32 [nnz]
    val: np.ndarray      # float64 / float32 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1]) - int(self.row_ptr[0])

    def astype(self, dtype) -> "CSR":
        return CSR(self.rows, self.cols, self.row_ptr, self.col, self.val.astype(dtype))

    def row_lengths(self) -> np.ndarray:
        return np.diff(self.row_ptr.astype(np.int64))

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.rows, self.cols), dtype=np.float64)
        r = np.repeat(np.arange(self.rows), self.row_lengths())
        np.add.at(d, (r, self.col.astype(np.int64)), self.val.astype(np.float64))
        return d


def _idx_dtype(n: int):
    return np.int32 if n < 2**31 else np.int64


def _stable_argsort(key: np.ndarray) -> np.ndarray:
    """np.argsort(key, kind="stable"), computed by torch's multi-threaded CPU sort when
    torch is importable (the same permutation: a stable sort is unique)."""
    try:
        import torch
    except ImportError:
        return np.argsort(key, kind="stable")
    return torch.sort(torch.from_numpy(np.ascontiguousarray(key)), stable=True).indices.numpy()


def _sorted_unique(key: np.ndarray) -> np.ndarray:
    """np.unique(key) (sorted, distinct) through a sort and a neighbour test."""
    if key.size == 0:
        return key
    k = key[_stable_argsort(key)]
    keep = np.empty(k.size, dtype=bool)
    keep[0] = True
    np.not_equal(k[1:], k[:-1], out=keep[1:])
    return k[keep]


def from_coo(rows: int, cols: int, r: np.ndarray, c: np.ndarray, v: np.ndarray,
             sum_duplicates: bool = False) -> CSR:
    """Build canonical CSR from COO triplets (sorted by (row, col))."""
    r = np.asarray(r, dtype=np.int64)
    c = np.asarray(c, dtype=np.int64)
    v = np.asarray(v)
    key = r * np.int64(cols) + c
    order = _stable_argsort(key)
    key = key[order]
    v = v[order]
    if sum_duplicates and key.size:
        uniq, first = np.unique(key, return_index=True)
        v = np.add.reduceat(v, first) if v.size else v
        key = uniq
    r = key // cols
    c = key % cols
    counts = np.bincount(r, minlength=rows) if rows else np.zeros(0, np.int64)
    rp = np.zeros(rows + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    it = _idx_dtype(int(rp[-1]))
    return CSR(rows, cols, rp.astype(it), c.astype(np.int32), v)


def transpose(A: CSR) -> CSR:
    """Precomputed transpose (untimed input preparation, §4)."""
    r = np.repeat(np.arange(A.rows, dtype=np.int64), A.row_lengths())
    return from_coo(A.cols, A.rows, A.col.astype(np.int64), r, A.val)


# ---------------------------------------------------------------- stencils --

def _stencil(shape, offsets_vals, dtype=np.float64) -> CSR:
    """Generic constant-coefficient stencil on a box grid, natural (x fastest)
    ordering.  offsets_vals: list of ((dx, dy, dz), value)."""
    nx, ny, nz = shape
    N = nx * ny * nz
    idx = np.arange(N, dtype=np.int64)
    x = idx % nx
    y = (idx // nx) % ny
    z = idx // (nx * ny)
    # sort offsets by the column offset they produce -> ascending columns
    offs = sorted(offsets_vals, key=lambda ov: ov[0][0] + nx * ov[0][1] + nx * ny * ov[0][2])
    masks, colofs = [], []
    for (dx, dy, dz), _ in offs:
        m = np.ones(N, dtype=bool)
        if dx: m &= (x + dx >= 0) & (x + dx < nx)
        if dy: m &= (y + dy >= 0) & (y + dy < ny)
        if dz: m &= (z + dz >= 0) & (z + dz < nz)
        masks.append(m)
        colofs.append(dx + nx * dy + nx * ny * dz)
    counts = np.zeros(N, dtype=np.int64)
    for m in masks:
        counts += m
    rp = np.zeros(N + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    nnz = int(rp[-1])
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=dtype)
    fill = rp[:-1].copy()
    for m, co, (_, v) in zip(masks, colofs, offs):
        pos = fill[m]
        col[pos] = (idx[m] + co).astype(np.int32)
        val[pos] = v
        fill[m] += 1
    return CSR(N, N, rp.astype(_idx_dtype(nnz)), col, val)


def poisson2d_5pt(n: int, dtype=np.float64) -> CSR:
    """2D 5-point Laplacian, A = 4I − (I⊗T₀ + T₀⊗I) (BASELINE.json configs[0])."""
    ov = [((0, 0, 0), 4.0), ((-1, 0, 0), -1.0), ((1, 0, 0), -1.0),
          ((0, -1, 0), -1.0), ((0, 1, 0), -1.0)]
    return _stencil((n, n, 1), ov, dtype)


def poisson3d_27pt(n: int, dtype=np.float64) -> CSR:
    """3D 27-point operator, A = 27I − T⊗T⊗T: diagonal 26, off-diagonals −1
    (BASELINE.json configs[1])."""
    ov = []
    for dz in (-1, 0, 1):
        for dy in (-1, 0, 1):
            for dx in (-1, 0, 1):
                ov.append(((dx, dy, dz), 26.0 if (dx, dy, dz) == (0, 0, 0) else -1.0))
    return _stencil((n, n, n), ov, dtype)


def poisson3d_7pt(n: int, dtype=np.float64) -> CSR:
    """3D 7-point Laplacian, diagonal 6, neighbours −1 (configs[3])."""
    ov = [((0, 0, 0), 6.0)]
    for d in ((1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)):
        ov.append((d, -1.0))
    return _stencil((n, n, n), ov, dtype)


def aggregation_prolongator(n: int, dtype=np.float64) -> CSR:
    """Unsmoothed 2×2×2 aggregation P: fine (x,y,z) -> coarse (x//2,y//2,z//2),
    value 1 (SURVEY §8(c) reading 24).  Shape n³ × (n/2)³."""
    assert n % 2 == 0
    N = n ** 3
    m = n // 2
    idx = np.arange(N, dtype=np.int64)
    x, y, z = idx % n, (idx // n) % n, idx // (n * n)
    c = (x // 2) + m * (y // 2) + m * m * (z // 2)
    rp = np.arange(N + 1, dtype=np.int64)
    return CSR(N, m ** 3, rp.astype(_idx_dtype(N)), c.astype(np.int32), np.ones(N, dtype=dtype))


# ------------------------------------------------------------------ R-MAT --

def rmat(scale: int = 20, edge_factor: int = 16, abc=(0.45, 0.15, 0.15), seed: int = 20190216,
         values: str = "uniform", value_seed: int = 3, dtype=np.float64) -> CSR:
    """R-MAT graph adjacency: permuted vertices, self-loops
    dropped, duplicates coalesced, values 1 ('ones') or U(−1,1)."""
    n = 1 << scale
    m = edge_factor * n
    a, b, c = abc
    rng = np.random.default_rng(seed)
    src = np.zeros(m, dtype=np.int64)
    dst = np.zeros(m, dtype=np.int64)
    for lvl in range(scale):
        r = rng.random(m)
        rowbit = r >= a + b
        colbit = ((r >= a) & (r < a + b)) | (r >= a + b + c)
        src |= rowbit.astype(np.int64) << lvl
        dst |= colbit.astype(np.int64) << lvl
    perm = rng.permutation(n)
    src, dst = perm[src], perm[dst]
    keep = src != dst
    key = _sorted_unique(src[keep] * n + dst[keep])
    r_, c_ = key // n, key % n
    nnz = key.size
    if values == "ones":
        v = np.ones(nnz, dtype=dtype)
    else:
        v = np.random.default_rng(value_seed).uniform(-1.0, 1.0, nnz).astype(dtype)
    counts = np.bincount(r_, minlength=n)
    rp = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=rp[1:])
    return CSR(n, n, rp.astype(_idx_dtype(nnz)), c_.astype(np.int32), v)


# ---------------------------------------------------------------- LP-like --

def lp_like(rows_log2: int = 20, cols_log2: int = 22, per_col: int = 20, seed: int = 7,
            dtype=np.float64):
    """Rectangular LP-like matrix: 2^rows × 2^cols, exactly `per_col` distinct
    uniform rows per column, values U(−1,1) (SURVEY §8(c) reading 25).
    Returns (A, At) where At = Aᵀ is the precomputed transpose (L554)."""
    R, Cn = 1 << rows_log2, 1 << cols_log2
    rng = np.random.default_rng(seed)
    r = rng.integers(0, R, size=(Cn, per_col), dtype=np.int64)
    while True:
        s = np.sort(r, axis=1)
        dup = (s[:, 1:] == s[:, :-1]).any(axis=1)
        if not dup.any():
            break
        r[dup] = rng.integers(0, R, size=(int(dup.sum()), per_col), dtype=np.int64)
    r = np.sort(r, axis=1)
    vals = rng.uniform(-1.0, 1.0, Cn * per_col).astype(dtype).reshape(Cn, per_col)
    # At (cols x rows): row j of At = column j of A, rows sorted
    At = CSR(Cn, R, (np.arange(Cn + 1, dtype=np.int64) * per_col).astype(_idx_dtype(Cn * per_col)),
             r.reshape(-1).astype(np.int32), vals.reshape(-1))
    A = transpose(At)
    return A, At


# ------------------------------------------------------------ small random --

def random_csr(m: int, n: int, density: float, seed: int, dtype=np.float64,
               values: str = "uniform", empty_rows: float = 0.0) -> CSR:
    """Small random CSR for parity tests.  values: 'uniform' U(−1,1), 'int'
    small integers in [−3,3]\\{0}, 'ones'."""
    rng = np.random.default_rng(seed)
    mask = rng.random((m, n)) < density
    if empty_rows > 0:
        mask[rng.random(m) < empty_rows, :] = False
    r, c = np.nonzero(mask)
    k = r.size
    if values == "ones":
        v = np.ones(k)
    elif values == "int":
        v = rng.integers(1, 4, k) * rng.choice([-1.0, 1.0], k)
    else:
        v = rng.uniform(-1.0, 1.0, k)
    return from_coo(m, n, r, c, v.astype(dtype))


def random_rowlen_csr(m: int, n: int, lengths: np.ndarray, seed: int, dtype=np.float64,
                      values: str = "uniform") -> CSR:
    """Random CSR with prescribed row lengths (distinct uniform columns)."""
    rng = np.random.default_rng(seed)
    rs, cs = [], []
    for i, L in enumerate(np.asarray(lengths, dtype=np.int64)):
        L = int(min(L, n))
        if L == 0:
            continue
        cols = rng.choice(n, size=L, replace=False)
        rs.append(np.full(L, i, dtype=np.int64))
        cs.append(cols.astype(np.int64))
    r = np.concatenate(rs) if rs else np.zeros(0, np.int64)
    c = np.concatenate(cs) if cs else np.zeros(0, np.int64)
    k = r.size
    if values == "ones":
        v = np.ones(k)
    elif values == "int":
        v = rng.integers(1, 4, k) * rng.choice([-1.0, 1.0], k)
    else:
        v = rng.uniform(-1.0, 1.0, k)
    return from_coo(m, n, r, c, v.astype(dtype))


def power_law_csr(m: int, n: int, mean_len: float, alpha: float, max_len: int, seed: int,
                  dtype=np.float64, values: str = "uniform") -> CSR:
    """Skewed row-length matrix (Zipf-like lengths) for merge-path tests."""
    rng = np.random.default_rng(seed)
    raw = rng.pareto(alpha, m) + 1.0
    lengths = np.minimum((raw / raw.mean() * mean_len).astype(np.int64), max_len)
    return random_rowlen_csr(m, n, lengths, seed + 1, dtype, values)


# ----------------------------------------------------------- named configs --

def config(name: str, dtype=np.float64):
    """BASELINE.json configs by short name.  Returns (A, B) with C = A·B.
    For 'rap' returns (A, P, R)."""
    if name == "cfg1":          # 2D 5-pt 64², A·A
        A = poisson2d_5pt(64, dtype)
        return A, A
    if name == "cfg2":          # 3D 27-pt 128³, A·A
        A = poisson3d_27pt(128, dtype)
        return A, A
    if name == "cfg3":          # R-MAT s20 ef16, A·A
        A = rmat(dtype=dtype)
        return A, A
    if name == "cfg5":          # LP-like A·Aᵀ
        A, At = lp_like(dtype=dtype)
        return A, At
    if name == "rap":           # 7-pt 256³ with 2³ aggregation
        A = poisson3d_7pt(256, dtype)
        P = aggregation_prolongator(256, dtype)
        return A, P, transpose(P)
    raise KeyError(name)
