"""AC-SpGEMM on B200 (sm_100a): adaptive chunk-based ESC sparse matrix-matrix
multiplication (Winter et al., PPoPP'19) as a C-ABI CUDA library with a thin Python
binding.  See include/acspgemm.h and DESIGN.md."""
from .api import (DeviceCSR, Plan, STAGES, canonical_segments, const, debug_sort_compact,
                  debug_work_distribution, multiply, multiply_host, multiply_lib_alloc, pool_estimate_bytes,
                  rap, rap_lib_alloc)
from ._lib import AcspgemmError, SIGNATURES, SO_PATH, load

__all__ = ["DeviceCSR", "Plan", "STAGES", "canonical_segments", "const", "debug_sort_compact",
           "debug_work_distribution", "multiply", "multiply_host", "multiply_lib_alloc", "pool_estimate_bytes", "rap", "rap_lib_alloc",
           "AcspgemmError", "SIGNATURES", "SO_PATH", "load"]
