"""ctypes loader and signatures of libacspgemm.so (the C ABI of include/acspgemm.h).

Argument marshalling only.  There is no fallback: if the shared library is missing or
cannot be loaded the import of any product entry point raises.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# ACSPGEMM_LIB: an in-tree build variant (e.g. libacspgemm_w4.so from build.py with ACS_BUILD_TAG)
SO_PATH = os.environ.get("ACSPGEMM_LIB") or os.path.join(HERE, "libacspgemm.so")

I32, I64, U32 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
VP = ctypes.c_void_p
PI32 = ctypes.POINTER(ctypes.c_int32)
PI64 = ctypes.POINTER(ctypes.c_int64)


class CsrIn(ctypes.Structure):
    _fields_ = [("rows", I64), ("cols", I64), ("nnz", I64),
                ("row_ptr", VP), ("col_idx", VP), ("val", VP)]


class CsrOut(ctypes.Structure):
    _fields_ = [("rows", I64), ("cols", I64), ("nnz", I64),
                ("row_ptr", VP), ("col_idx", VP), ("val", VP)]


# acspgemm_csr_out64: the same layout (int64 row_ptr behind the pointer)
CsrOut64 = CsrOut


class Options(ctypes.Structure):
    _fields_ = [("pool_limit_bytes", ctypes.c_size_t), ("validate_inputs", ctypes.c_int),
                ("collect_stage_times", ctypes.c_int), ("num_segments", ctypes.c_int),
                ("strategy", ctypes.c_int), ("pool_mode", ctypes.c_int)]


class Info(ctypes.Structure):
    _fields_ = [("products", I64), ("nnz_c", I64), ("nblocks", I64), ("nchunks", I64),
                ("chunk_elems", I64), ("nshared", I64), ("nmulti", I64), ("npath", I64),
                ("nsearch", I64), ("nmulti_groups", I64), ("merge_elems", I64),
                ("pool_bytes", I64), ("helper_bytes", I64), ("pool_estimate_bytes", ctypes.c_double),
                ("kernel_launches", I64), ("nsegments", I32), ("segment_rows", I64 * 65),
                ("nhash_blocks", I64), ("ndict_blocks", I64), ("nrow_blocks", I64),
                ("ndeferred_blocks", I64), ("pool_mode", I32)]


# name -> (restype, argtypes); every symbol include/acspgemm.h declares
SIGNATURES = {
    "acspgemm_options_default": (None, [ctypes.POINTER(Options)]),
    "acspgemm_plan_create": (ctypes.c_int, [ctypes.POINTER(VP), ctypes.POINTER(Options)]),
    "acspgemm_plan_destroy": (None, [VP]),
    "acspgemm_set_segments": (ctypes.c_int, [VP, ctypes.c_int, PI64]),
    "acspgemm_canonical_segments": (ctypes.c_int, [ctypes.POINTER(CsrIn), ctypes.c_int, PI64, VP]),
    "acspgemm_symbolic": (ctypes.c_int, [VP, ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn), ctypes.c_int, VP, PI64]),
    "acspgemm_numeric": (ctypes.c_int, [VP, ctypes.POINTER(CsrOut), VP]),
    "acspgemm_numeric64": (ctypes.c_int, [VP, ctypes.POINTER(CsrOut64), VP]),
    "acspgemm_numeric_update": (ctypes.c_int, [VP, ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn),
                                               ctypes.POINTER(CsrOut), VP]),
    "acspgemm_multiply": (ctypes.c_int, [ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn), ctypes.POINTER(CsrOut), VP,
                                         ctypes.c_int]),
    "acspgemm_multiply_host": (ctypes.c_int, [VP, ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn), ctypes.c_int, VP,
                                              ctypes.c_int, ctypes.POINTER(CsrOut), I64]),
    "acspgemm_multiply_budget": (ctypes.c_int, [VP, ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn), ctypes.c_int, VP,
                                                ctypes.POINTER(CsrOut), ctypes.POINTER(ctypes.c_int),
                                                ctypes.POINTER(ctypes.c_int)]),
    "acspgemm_rap": (ctypes.c_int, [ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn), ctypes.POINTER(CsrIn),
                                    ctypes.POINTER(CsrOut), VP, ctypes.c_int]),
    "acspgemm_free_csr": (ctypes.c_int, [ctypes.POINTER(CsrOut), VP]),
    "acspgemm_stage_times": (ctypes.c_int, [VP, ctypes.POINTER(ctypes.c_float), ctypes.c_int]),
    "acspgemm_plan_info": (ctypes.c_int, [VP, ctypes.POINTER(Info)]),
    "acspgemm_block_row_starts": (ctypes.c_int, [VP, PI32, I64]),
    "acspgemm_set_trace": (ctypes.c_int, [VP, ctypes.c_int]),
    "acspgemm_sm_load": (ctypes.c_int, [VP, ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.c_int,
                                        ctypes.POINTER(ctypes.c_double), PI64]),
    "acspgemm_pool_estimate_bytes": (ctypes.c_double, [I64, I64, I64, I64, I64, ctypes.c_int]),
    "acspgemm_debug_work_distribution": (ctypes.c_int, [PI32, ctypes.c_int, PI32, ctypes.c_int, PI32, PI32, PI32]),
    "acspgemm_debug_sort_compact": (ctypes.c_int, [PI32, PI32, ctypes.POINTER(ctypes.c_double), ctypes.c_int,
                                                   PI32, PI32, ctypes.POINTER(ctypes.c_double),
                                                   ctypes.POINTER(ctypes.c_uint32)]),
    "acspgemm_const": (ctypes.c_int, [ctypes.c_int]),
    "acspgemm_status_string": (ctypes.c_char_p, [ctypes.c_int]),
    "acspgemm_last_error": (ctypes.c_char_p, []),
    "acspgemm_abi_version": (ctypes.c_int, []),
}

_lib = None


def load() -> ctypes.CDLL:
    """Load libacspgemm.so (raises if it is missing: no CPU fallback exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(SO_PATH):
            raise ImportError(f"{SO_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`"
                              " (the CUDA path has no fallback)")
        lib = ctypes.CDLL(SO_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(lib, name)
            fn.restype = res
            fn.argtypes = args
        _lib = lib
    return _lib


class AcspgemmError(RuntimeError):
    def __init__(self, status: int, where: str):
        lib = load()
        msg = lib.acspgemm_status_string(status).decode()
        detail = (lib.acspgemm_last_error() or b"").decode()
        super().__init__(f"{where}: {msg} ({detail})")
        self.status = status


def check(status: int, where: str) -> None:
    if status != 0:
        raise AcspgemmError(status, where)
