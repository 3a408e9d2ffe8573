"""TEST INFRASTRUCTURE ONLY — the CPU parity oracle for AC-SpGEMM.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
legs may import this package.  The product path (paper_conf_ppopp_wintermzss19_b200)
never imports it, and it imports nothing from the product path: the two share no
code; only `synth` (seeded input generators, no SpGEMM arithmetic) serves both.

Contents
  gustavson(A, B)       C = A·B by sequential Gustavson SPA (gustavson.c, PAPER.md L48,
                        L76; Eq. (1)), fp64 sums plus Σ|a·b| per entry.
  products(A, B)        number of intermediate products Σ_p len(B_row(A.col[p])).
  alg.*                 Alg. 1 / Alg. 2 / Alg. 3 / pool estimate, step by step.

Parity status: every function here is pinned by tests/test_oracle_*.py (brute-force
dense products, closed-form stencil squares, invariants, Fig. 3, Table 3); see
DESIGN.md §"Oracle and pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

from . import alg  # noqa: F401

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile gustavson.c with gcc (plain -O3, OpenMP)."""
    src = os.path.join(_HERE, "gustavson.c")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        I64 = ctypes.c_int64
        lib.oracle_gustavson_count.restype = I64
        lib.oracle_gustavson_count.argtypes = [I64, I64, P, P, P, P, P, ctypes.c_int]
        lib.oracle_gustavson_fill.restype = None
        lib.oracle_gustavson_fill.argtypes = [I64, I64, P, P, P, P, P, P, P, P, P, P, ctypes.c_int]
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


class OracleCSR:
    """Oracle result: row_ptr (int64), col (int32), val (float64), absval (float64)."""

    def __init__(self, rows, cols, row_ptr, col, val, absval):
        self.rows, self.cols = rows, cols
        self.row_ptr, self.col, self.val, self.absval = row_ptr, col, val, absval

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])


def gustavson(A, B, threads: int = 0, row_begin: int = 0, row_end: int | None = None) -> OracleCSR:
    """C[row_begin:row_end] = (A·B)[row_begin:row_end] (all rows by default).

    A, B: objects with rows, cols, row_ptr, col, val (numpy).  Values are promoted to
    fp64; fp32 products are therefore exact."""
    if A.cols != B.rows:
        raise ValueError("dimension mismatch")
    lib = _load()
    r1 = A.rows if row_end is None else row_end
    arp = np.ascontiguousarray(A.row_ptr[row_begin:r1 + 1], dtype=np.int64)
    m = r1 - row_begin
    acol = np.ascontiguousarray(A.col, dtype=np.int32)
    aval = np.ascontiguousarray(A.val, dtype=np.float64)
    brp = np.ascontiguousarray(B.row_ptr, dtype=np.int64)
    bcol = np.ascontiguousarray(B.col, dtype=np.int32)
    bval = np.ascontiguousarray(B.val, dtype=np.float64)
    counts = np.zeros(max(m, 1), dtype=np.int64)
    total = lib.oracle_gustavson_count(m, B.cols, _p(arp), _p(acol), _p(brp), _p(bcol), _p(counts), threads)
    crp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts[:m], out=crp[1:])
    ccol = np.empty(max(total, 1), dtype=np.int32)
    cval = np.empty(max(total, 1), dtype=np.float64)
    cabs = np.empty(max(total, 1), dtype=np.float64)
    lib.oracle_gustavson_fill(m, B.cols, _p(arp), _p(acol), _p(aval), _p(brp), _p(bcol), _p(bval),
                              _p(crp), _p(ccol), _p(cval), _p(cabs), threads)
    return OracleCSR(m, B.cols, crp, ccol[:total], cval[:total], cabs[:total])


def products(A, B) -> int:
    """Intermediate products Σ_k nnz(A_:,k)·nnz(B_k,:) (the 'temp' of Table 2)."""
    blen = np.diff(np.asarray(B.row_ptr, dtype=np.int64))
    lo, hi = int(A.row_ptr[0]), int(A.row_ptr[-1])
    return int(blen[np.asarray(A.col[lo:hi], dtype=np.int64)].sum())


def timed_gustavson(A, B, threads: int = 0, row_begin: int = 0, row_end: int | None = None):
    """(result, seconds) — used by bench.py's cpu_baseline leg."""
    t0 = time.perf_counter()
    C = gustavson(A, B, threads, row_begin, row_end)
    return C, time.perf_counter() - t0
