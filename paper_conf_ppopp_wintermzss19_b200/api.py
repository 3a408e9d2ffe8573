"""Python binding of the AC-SpGEMM C ABI (argument marshalling only).

torch supplies device memory and streams; every step of C = A·B runs in the CUDA
kernels of libacspgemm.so.  Names follow include/acspgemm.h.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from typing import Optional, Sequence

import numpy as np
import torch

from . import _lib
from ._lib import AcspgemmError, CsrIn, CsrOut, Info, Options, check, load

F32, F64 = 0, 1
# HASH: the accumulator part of ESC (k_dict + k_hash); DICT: its k_dict part
STAGES = ("GLB", "ESC", "MCC", "MM", "PM", "SM", "SCAN", "CC", "HASH", "DICT")


@dataclass
class DeviceCSR:
    """CSR matrix in CUDA memory: row_ptr int32 (int64 for outputs of Plan.multiply(index64=True)),
    col int32, val float32 or float64."""
    rows: int
    cols: int
    row_ptr: torch.Tensor
    col: torch.Tensor
    val: torch.Tensor

    @property
    def nnz(self) -> int:
        return int(self.col.numel())

    @property
    def dtype(self):
        return self.val.dtype

    @staticmethod
    def from_numpy(rows, cols, row_ptr, col, val, device="cuda", dtype=None) -> "DeviceCSR":
        v = np.asarray(val)
        if dtype is not None:
            v = v.astype(dtype)
        return DeviceCSR(int(rows), int(cols),
                         torch.from_numpy(np.ascontiguousarray(row_ptr, dtype=np.int32)).to(device),
                         torch.from_numpy(np.ascontiguousarray(col, dtype=np.int32)).to(device),
                         torch.from_numpy(np.ascontiguousarray(v)).to(device))

    @staticmethod
    def from_host(M, device="cuda", dtype=None) -> "DeviceCSR":
        """From any object with rows, cols, row_ptr, col, val numpy arrays."""
        return DeviceCSR.from_numpy(M.rows, M.cols, M.row_ptr, M.col, M.val, device, dtype)

    def to_numpy(self):
        return (self.row_ptr.cpu().numpy(), self.col.cpu().numpy(), self.val.cpu().numpy())


def _dtype_code(t: torch.dtype) -> int:
    if t == torch.float64:
        return F64
    if t == torch.float32:
        return F32
    raise TypeError(f"unsupported value dtype {t} (float32/float64)")


def _csr_in(M: DeviceCSR, row_ptr: Optional[torch.Tensor] = None, rows: Optional[int] = None,
            nnz: Optional[int] = None) -> CsrIn:
    rp = M.row_ptr if row_ptr is None else row_ptr
    for t in (rp, M.col, M.val):
        if not t.is_cuda or not t.is_contiguous():
            raise ValueError("DeviceCSR tensors must be contiguous CUDA tensors")
    if rp.dtype != torch.int32 or M.col.dtype != torch.int32:
        raise TypeError("row_ptr / col must be int32")
    r = M.rows if rows is None else rows
    n = M.nnz if nnz is None else nnz
    return CsrIn(r, M.cols, n, rp.data_ptr(), M.col.data_ptr(), M.val.data_ptr())


def _stream_ptr(stream: Optional[torch.cuda.Stream]) -> ctypes.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


_STRATEGIES = {"adaptive": 0, "esc": 1, "hash": 2, "dict": 3}   # ACSPGEMM_STRATEGY_* (include/acspgemm.h)
_POOL_MODES = {"exact": 0, "bound": 1, "auto": 2}               # ACSPGEMM_POOL_*


class Plan:
    """A reusable multiply plan (owns the chunk pool and helper memory)."""

    def __init__(self, pool_limit_bytes: int = 0, validate: bool = False, stage_times: bool = False,
                 num_segments: int = 8, strategy: str = "adaptive", pool_mode: str = "bound"):
        """strategy: "adaptive" (hash accumulator per candidate block, per-row accumulator
        for blocks of short rows, AC-ESC fallback; readings R31, R34), "hash" (the same path;
        kept for the round-1 API), "dict" (column dictionary first, reading R33) -- these three give the
        same bits -- or "esc" (every block through AC-ESC).
        pool_mode: "exact" (every block its exact product bound), "bound" (accumulator
        candidates bounded by rows x 256, their AC-ESC fallbacks deferred to a second
        pass), "auto" (exact if it fits pool_limit_bytes, else bound) -- same bytes of C
        (include/acspgemm.h, reading R40)."""
        if strategy not in _STRATEGIES:
            raise ValueError("strategy must be one of " + ", ".join(_STRATEGIES))
        if pool_mode not in _POOL_MODES:
            raise ValueError("pool_mode must be one of " + ", ".join(_POOL_MODES))
        lib = load()
        opt = Options()
        lib.acspgemm_options_default(ctypes.byref(opt))
        opt.pool_limit_bytes = int(pool_limit_bytes)
        opt.validate_inputs = int(bool(validate))
        opt.collect_stage_times = int(bool(stage_times))
        opt.num_segments = int(num_segments)
        opt.strategy = _STRATEGIES[strategy]
        opt.pool_mode = _POOL_MODES[pool_mode]
        h = ctypes.c_void_p()
        check(lib.acspgemm_plan_create(ctypes.byref(h), ctypes.byref(opt)), "acspgemm_plan_create")
        self._h = h
        self._lib = lib
        self._dtype = None
        self._rows = 0
        self._cols = 0

    def close(self) -> None:
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.acspgemm_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_segments(self, rows: Optional[Sequence[int]]) -> None:
        if rows is None:
            check(self._lib.acspgemm_set_segments(self._h, 0, None), "acspgemm_set_segments")
            return
        arr = (ctypes.c_int64 * len(rows))(*[int(r) for r in rows])
        check(self._lib.acspgemm_set_segments(self._h, len(rows) - 1, arr), "acspgemm_set_segments")

    def symbolic(self, A: DeviceCSR, B: DeviceCSR, stream=None, A_view=None) -> int:
        if A.dtype != B.dtype:
            raise TypeError("A and B must have the same value dtype")
        a = _csr_in(A) if A_view is None else A_view
        b = _csr_in(B)
        nnz = ctypes.c_int64(0)
        check(self._lib.acspgemm_symbolic(self._h, ctypes.byref(a), ctypes.byref(b), _dtype_code(A.dtype),
                                          _stream_ptr(stream), ctypes.byref(nnz)), "acspgemm_symbolic")
        self._dtype = A.dtype
        self._rows = a.rows
        self._cols = B.cols
        return int(nnz.value)

    def numeric(self, row_ptr: torch.Tensor, col: torch.Tensor, val: torch.Tensor, stream=None) -> None:
        """Numeric pass into caller-allocated C; an int64 row_ptr selects acspgemm_numeric64."""
        c = CsrOut(0, 0, 0, row_ptr.data_ptr(), col.data_ptr(), val.data_ptr())
        if row_ptr.dtype == torch.int64:
            check(self._lib.acspgemm_numeric64(self._h, ctypes.byref(c), _stream_ptr(stream)), "acspgemm_numeric64")
        elif row_ptr.dtype == torch.int32:
            check(self._lib.acspgemm_numeric(self._h, ctypes.byref(c), _stream_ptr(stream)), "acspgemm_numeric")
        else:
            raise TypeError("row_ptr must be int32 or int64")

    def multiply(self, A: DeviceCSR, B: DeviceCSR, stream=None, A_view=None, index64: bool = False) -> DeviceCSR:
        """symbolic -> allocate C with torch on the device -> numeric.  index64: C.row_ptr
        in int64 (required when nnz(C) >= 2^31; columns stay int32)."""
        nnz = self.symbolic(A, B, stream, A_view)
        if not index64 and nnz >= 2 ** 31:
            raise AcspgemmError(3, "Plan.multiply: nnz(C) >= 2^31 needs index64=True")   # INDEX_OVERFLOW
        dev = A.val.device
        rows = self._rows
        # one allocation for C (row_ptr | col | val, each 256-byte aligned): the host gap
        # between the symbolic read-back and the numeric launches is on the critical path
        rdt = torch.int64 if index64 else torch.int32
        rpb = (rows + 1) * (8 if index64 else 4)
        n1 = max(nnz, 1)
        o1 = (rpb + 255) // 256 * 256
        o2 = o1 + (n1 * 4 + 255) // 256 * 256
        buf = torch.empty(o2 + n1 * A.val.element_size(), dtype=torch.uint8, device=dev)
        rp = buf[:rpb].view(rdt)
        col = buf[o1:o1 + n1 * 4].view(torch.int32)
        val = buf[o2:].view(A.dtype)
        self.numeric(rp, col, val, stream)
        return DeviceCSR(rows, B.cols, rp, col[:nnz], val[:nnz])

    def numeric_update(self, A: DeviceCSR, B: DeviceCSR, C: DeviceCSR, stream=None) -> DeviceCSR:
        """Recompute C's values for new values of A and B on the pattern of this plan's last
        multiply (same structure, same dtype; C from that multiply, int32 row_ptr).
        Sync-free: replays the recorded sizes inside a CUDA graph (acspgemm_numeric_update)."""
        if C.row_ptr.dtype != torch.int32:
            raise TypeError("numeric_update writes an int32 row_ptr")
        a, b = _csr_in(A), _csr_in(B)
        c = CsrOut(0, 0, 0, C.row_ptr.data_ptr(), C.col.data_ptr(), C.val.data_ptr())
        check(self._lib.acspgemm_numeric_update(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c),
                                                _stream_ptr(stream)), "acspgemm_numeric_update")
        return C

    def multiply_budget(self, A: DeviceCSR, B: DeviceCSR, stream=None):
        """C = A·B within this plan's pool_limit_bytes through acspgemm_multiply_budget:
        pieces of whole canonical segments, a piece over budget retried on fewer segments
        (a "restart").  Bit-identical to multiply().  Returns ((row_ptr, col, val) as host
        numpy arrays, pieces, restarts)."""
        if A.dtype != B.dtype:
            raise TypeError("A and B must have the same value dtype")
        a, b = _csr_in(A), _csr_in(B)
        c = CsrOut()
        npc, nrs = ctypes.c_int(0), ctypes.c_int(0)
        st = _stream_ptr(stream)
        check(self._lib.acspgemm_multiply_budget(self._h, ctypes.byref(a), ctypes.byref(b), _dtype_code(A.dtype), st,
                                                 ctypes.byref(c), ctypes.byref(npc), ctypes.byref(nrs)),
              "acspgemm_multiply_budget")
        try:
            rp = np.empty(c.rows + 1, dtype=np.int32)
            col = np.empty(c.nnz, dtype=np.int32)
            val = np.empty(c.nnz, dtype=np.float64 if A.dtype == torch.float64 else np.float32)
            torch.cuda.synchronize()
            _memcpy_d2h(rp, c.row_ptr)
            _memcpy_d2h(col, c.col_idx)
            _memcpy_d2h(val, c.val)
            return (rp, col, val), int(npc.value), int(nrs.value)
        finally:
            check(self._lib.acspgemm_free_csr(ctypes.byref(c), st), "acspgemm_free_csr")
            torch.cuda.synchronize()

    def multiply_host(self, A, B, out=None, pieces: int = 4, stream=None):
        """End to end through acspgemm_multiply_host: A and B on the host (objects with
        rows, cols, row_ptr, col, val as numpy arrays or CPU tensors; int32 indices),
        C returned on the host.  `out` = (row_ptr, col, val) host buffers (pinned CPU
        tensors or numpy arrays; col/val capacity = their length); without it a size
        query runs first and pinned tensors are allocated.  Returns (row_ptr, col, val)
        trimmed to nnz(C)."""
        dt = _host_dtype(A.val)
        if _host_dtype(B.val) != dt:
            raise TypeError("A and B must have the same value dtype")
        a, keep_a = _host_csr_in(A)
        b, keep_b = (a, keep_a) if B is A else _host_csr_in(B)
        st = _stream_ptr(stream)
        code = 1 if dt == np.float64 else 0
        c = CsrOut()
        if out is None:
            rp = torch.empty(A.rows + 1, dtype=torch.int32).pin_memory()
            c.row_ptr = rp.data_ptr()
            st_code = self._lib.acspgemm_multiply_host(self._h, ctypes.byref(a), ctypes.byref(b), code, st,
                                                       int(pieces), ctypes.byref(c), 0)
            if st_code not in (0, 1):
                check(st_code, "acspgemm_multiply_host")
            n = int(c.nnz)
            tdt = torch.float64 if dt == np.float64 else torch.float32
            out = (rp, torch.empty(max(n, 1), dtype=torch.int32).pin_memory(),
                   torch.empty(max(n, 1), dtype=tdt).pin_memory())
        orp, ocol, oval = out
        if len(orp) < A.rows + 1 or len(ocol) != len(oval):
            raise ValueError("out buffers: row_ptr needs rows+1 entries, col and val the same capacity")
        c = CsrOut()
        c.row_ptr, c.col_idx, c.val = _host_ptr(orp), _host_ptr(ocol), _host_ptr(oval)
        check(self._lib.acspgemm_multiply_host(self._h, ctypes.byref(a), ctypes.byref(b), code, st, int(pieces),
                                               ctypes.byref(c), len(ocol)), "acspgemm_multiply_host")
        n = int(c.nnz)
        del keep_a, keep_b
        return orp[:A.rows + 1], ocol[:n], oval[:n]

    def info(self) -> dict:
        inf = Info()
        check(self._lib.acspgemm_plan_info(self._h, ctypes.byref(inf)), "acspgemm_plan_info")
        d = {name: getattr(inf, name) for name, _ in Info._fields_ if name != "segment_rows"}
        d["segment_rows"] = [inf.segment_rows[i] for i in range(inf.nsegments + 1)] if inf.nsegments else []
        return d

    def set_trace(self, enable: bool = True) -> None:
        """Record (SM, start, end) per block of the stage-2 kernels in the next multiplies."""
        check(self._lib.acspgemm_set_trace(self._h, int(bool(enable))), "acspgemm_set_trace")

    def sm_load(self, kernel: str = "hash") -> dict:
        """Multiprocessor load of one kernel of the last traced multiply (Table 3's mpL):
        {"mpl": min/max of the per-SM busy time, "per_sm_ms": [...], "blocks": n}."""
        k = {"hash": 0, "rows": 1, "esc": 2, "esc_small": 3}[kernel]
        nsm = torch.cuda.get_device_properties(torch.cuda.current_device()).multi_processor_count
        per = (ctypes.c_double * nsm)()
        mpl = ctypes.c_double()
        nb = ctypes.c_int64()
        check(self._lib.acspgemm_sm_load(self._h, k, per, nsm, ctypes.byref(mpl), ctypes.byref(nb)), "acspgemm_sm_load")
        return {"mpl": float(mpl.value), "per_sm_ms": [float(per[i]) for i in range(nsm)], "blocks": int(nb.value)}

    def stage_times(self) -> dict:
        buf = (ctypes.c_float * len(STAGES))()
        check(self._lib.acspgemm_stage_times(self._h, buf, len(STAGES)), "acspgemm_stage_times")
        return {k: float(buf[i]) for i, k in enumerate(STAGES)}

    def block_row_starts(self) -> np.ndarray:
        n = self.info()["nblocks"]
        out = np.zeros(max(n, 1), dtype=np.int32)
        check(self._lib.acspgemm_block_row_starts(self._h, out.ctypes.data_as(_lib.PI32), n),
              "acspgemm_block_row_starts")
        return out[:n]


def _host_dtype(v):
    if isinstance(v, torch.Tensor):
        return {torch.float64: np.float64, torch.float32: np.float32}[v.dtype]
    return np.dtype(v.dtype).type


def _host_ptr(x) -> int:
    if isinstance(x, torch.Tensor):
        if x.is_cuda or not x.is_contiguous():
            raise ValueError("host buffers must be contiguous CPU tensors")
        return x.data_ptr()
    if not x.flags["C_CONTIGUOUS"]:
        raise ValueError("host arrays must be C-contiguous")
    return x.ctypes.data


def _host_csr_in(M):
    """CsrIn over host arrays (int32 indices required; numpy arrays of another integer
    type are converted, the returned list keeps the converted arrays alive)."""
    keep = []
    arrs = []
    for x, want in ((M.row_ptr, np.int32), (M.col, np.int32), (M.val, None)):
        if isinstance(x, torch.Tensor):
            if want is not None and x.dtype != torch.int32:
                raise TypeError("row_ptr / col must be int32")
        elif want is not None and x.dtype != want:
            x = np.ascontiguousarray(x, dtype=want)
        keep.append(x)
        arrs.append(_host_ptr(x))
    nnz = int(M.row_ptr[M.rows]) - int(M.row_ptr[0]) if M.rows > 0 else 0
    return CsrIn(M.rows, M.cols, nnz, arrs[0], arrs[1], arrs[2]), keep


def multiply_host(A, B, out=None, pieces: int = 4, stream=None, **plan_kw):
    """C = A·B with host inputs and host result (one-shot plan; see Plan.multiply_host)."""
    p = Plan(**plan_kw)
    try:
        return p.multiply_host(A, B, out, pieces, stream)
    finally:
        p.close()


def multiply(A: DeviceCSR, B: DeviceCSR, stream=None, **plan_kw) -> DeviceCSR:
    """C = A·B with a temporary plan (two-phase API, C allocated by torch)."""
    p = Plan(**plan_kw)
    try:
        return p.multiply(A, B, stream)
    finally:
        p.close()


def rap(R: DeviceCSR, A: DeviceCSR, P: DeviceCSR, stream=None, **plan_kw) -> DeviceCSR:
    """Galerkin triple product R·(A·P) (two ordered multiplies, C allocated by torch)."""
    if R.cols != A.rows or A.cols != P.rows:
        raise ValueError("dimension mismatch")
    p = Plan(**plan_kw)
    try:
        AP = p.multiply(A, P, stream)
        return p.multiply(R, AP, stream)
    finally:
        p.close()


def rap_lib_alloc(R: DeviceCSR, A: DeviceCSR, P: DeviceCSR, stream=None):
    """R·(A·P) through acspgemm_rap (library-allocated C); returns host numpy arrays."""
    lib = load()
    r, a_, p_ = _csr_in(R), _csr_in(A), _csr_in(P)
    c = CsrOut()
    st = _stream_ptr(stream)
    check(lib.acspgemm_rap(ctypes.byref(r), ctypes.byref(a_), ctypes.byref(p_), ctypes.byref(c), st,
                           _dtype_code(A.dtype)), "acspgemm_rap")
    try:
        rp = np.empty(c.rows + 1, dtype=np.int32)
        col = np.empty(c.nnz, dtype=np.int32)
        val = np.empty(c.nnz, dtype=np.float64 if A.dtype == torch.float64 else np.float32)
        torch.cuda.synchronize()
        _memcpy_d2h(rp, c.row_ptr)
        _memcpy_d2h(col, c.col_idx)
        _memcpy_d2h(val, c.val)
        return rp, col, val
    finally:
        check(lib.acspgemm_free_csr(ctypes.byref(c), st), "acspgemm_free_csr")
        torch.cuda.synchronize()


def multiply_lib_alloc(A: DeviceCSR, B: DeviceCSR, stream=None):
    """C = A·B through acspgemm_multiply (the library allocates C with cudaMallocAsync).
    Returns host numpy arrays (row_ptr, col, val) and frees the device C."""
    lib = load()
    a, b = _csr_in(A), _csr_in(B)
    c = CsrOut()
    st = _stream_ptr(stream)
    check(lib.acspgemm_multiply(ctypes.byref(a), ctypes.byref(b), ctypes.byref(c), st, _dtype_code(A.dtype)),
          "acspgemm_multiply")
    try:
        n = c.nnz
        rp = np.empty(c.rows + 1, dtype=np.int32)
        col = np.empty(n, dtype=np.int32)
        val = np.empty(n, dtype=np.float64 if A.dtype == torch.float64 else np.float32)
        torch.cuda.synchronize()
        _memcpy_d2h(rp, c.row_ptr)
        _memcpy_d2h(col, c.col_idx)
        _memcpy_d2h(val, c.val)
        return rp, col, val
    finally:
        check(lib.acspgemm_free_csr(ctypes.byref(c), st), "acspgemm_free_csr")
        torch.cuda.synchronize()


def _memcpy_d2h(dst: np.ndarray, src_ptr) -> None:
    if dst.nbytes:
        _cuda_memcpy(dst.ctypes.data, int(src_ptr), dst.nbytes)


_cudart = None


def _cuda_memcpy(dst: int, src: int, n: int) -> None:
    global _cudart
    if _cudart is None:
        import glob
        import os
        cands = glob.glob(os.path.join(os.path.dirname(torch.__file__), "lib", "libcudart*.so*"))
        cands += glob.glob("/usr/local/cuda/lib64/libcudart.so*")
        _cudart = ctypes.CDLL(cands[0])
        _cudart.cudaMemcpy.restype = ctypes.c_int
        _cudart.cudaMemcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
    rc = _cudart.cudaMemcpy(ctypes.c_void_p(dst), ctypes.c_void_p(src), ctypes.c_size_t(n), 2)
    if rc != 0:
        raise RuntimeError(f"cudaMemcpy failed ({rc})")


def canonical_segments(A: DeviceCSR, nseg: int = 8, stream=None) -> list:
    lib = load()
    a = _csr_in(A)
    out = (ctypes.c_int64 * (nseg + 1))()
    check(lib.acspgemm_canonical_segments(ctypes.byref(a), nseg, out, _stream_ptr(stream)),
          "acspgemm_canonical_segments")
    return [int(out[i]) for i in range(nseg + 1)]


def pool_estimate_bytes(nA, nnzA, nB, mB, nnzB, value_bytes) -> float:
    return float(load().acspgemm_pool_estimate_bytes(nA, nnzA, nB, mB, nnzB, value_bytes))


def const(name: str) -> int:
    ids = {"NPB": 0, "THREADS": 1, "ITEMS": 2, "CAP": 3, "KEEP": 4, "RADIX_BITS": 5, "SEGMENTS": 6,
           "PATH_MAX_CHUNKS": 7}
    return int(load().acspgemm_const(ids[name]))


def debug_work_distribution(lengths: Sequence[int], draws: Sequence[int]):
    """Alg. 2 on the GPU (one CTA): returns (ares, bres, remaining[ndraws, nentries])."""
    lib = load()
    L = np.ascontiguousarray(lengths, dtype=np.int32)
    D = np.ascontiguousarray(draws, dtype=np.int32)
    tot = int(D.sum())
    ares = np.zeros(max(tot, 1), np.int32)
    bres = np.zeros(max(tot, 1), np.int32)
    rem = np.zeros(max(len(L) * len(D), 1), np.int32)
    check(lib.acspgemm_debug_work_distribution(L.ctypes.data_as(_lib.PI32), len(L), D.ctypes.data_as(_lib.PI32),
                                               len(D), ares.ctypes.data_as(_lib.PI32),
                                               bres.ctypes.data_as(_lib.PI32), rem.ctypes.data_as(_lib.PI32)),
          "acspgemm_debug_work_distribution")
    return ares[:tot], bres[:tot], rem[:len(L) * len(D)].reshape(len(D), len(L))


def debug_sort_compact(rows, cols, vals):
    """Block radix sort + Alg. 3 compaction scan on the GPU (one CTA, n <= CAP)."""
    lib = load()
    r = np.ascontiguousarray(rows, dtype=np.int32)
    c = np.ascontiguousarray(cols, dtype=np.int32)
    v = np.ascontiguousarray(vals, dtype=np.float64)
    n = len(r)
    orow, ocol = np.zeros(max(n, 1), np.int32), np.zeros(max(n, 1), np.int32)
    oval, ost = np.zeros(max(n, 1), np.float64), np.zeros(max(n, 1), np.uint32)
    dp = ctypes.POINTER(ctypes.c_double)
    check(lib.acspgemm_debug_sort_compact(r.ctypes.data_as(_lib.PI32), c.ctypes.data_as(_lib.PI32),
                                          v.ctypes.data_as(dp), n, orow.ctypes.data_as(_lib.PI32),
                                          ocol.ctypes.data_as(_lib.PI32), oval.ctypes.data_as(dp),
                                          ost.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))),
          "acspgemm_debug_sort_compact")
    return orow[:n], ocol[:n], oval[:n], ost[:n]
