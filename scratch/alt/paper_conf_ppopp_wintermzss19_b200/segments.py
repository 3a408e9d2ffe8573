"""Host restatement of the canonical segmentation (same definition as k_segments in
csrc/glb.cu) for host-side multi-process logic when the CUDA library is not used to
compute it (CPU gloo tests): boundary s = first row r with
row_ptr[r] − row_ptr[0] ≥ ceil(s·nnz/S)."""
from __future__ import annotations

import numpy as np


def canonical_segments_host(row_ptr, S: int):
    rp = np.asarray(row_ptr.cpu() if hasattr(row_ptr, "cpu") else row_ptr, dtype=np.int64)
    rp = rp - rp[0]
    nnz = int(rp[-1])
    rows = rp.size - 1
    out = [0]
    for s in range(1, S):
        target = -(-(s * nnz) // S)
        out.append(int(np.searchsorted(rp, target, side="left")))
    out.append(rows)
    return [min(max(x, 0), rows) for x in out]
