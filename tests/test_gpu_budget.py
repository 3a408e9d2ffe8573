"""Multiplies within a chunk-pool budget (acspgemm_multiply_budget; the
paper restarts when its pool runs out, L254, L844): pieces of whole canonical segments,
a piece over budget retried on fewer segments.  C must be byte-identical to the
one-piece multiply whatever the budget (the blocks are the canonical ones, reading R21),
with the expected piece and restart counts."""
import numpy as np
import pytest
import torch

import oracle
from synth import poisson3d_27pt, rmat

from test_gpu_parity import TOL, pkg

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_budget_pieces_bit_identical(dt, cuda_available):
    p = pkg()
    for A in (poisson3d_27pt(20), rmat(scale=12, edge_factor=16, values="uniform")):
        dA = p.DeviceCSR.from_host(A, "cuda", dt)
        plan = p.Plan()
        C = plan.multiply(dA, dA)
        torch.cuda.synchronize()
        ref_bytes = [t.cpu().numpy().tobytes() for t in (C.row_ptr, C.col, C.val)]
        pool = plan.info()["pool_bytes"]
        ref = oracle.gustavson(A.astype(dt), A.astype(dt))
        seen = set()
        for frac in (1.0, 0.6, 0.3, 0.15):
            bplan = p.Plan(pool_limit_bytes=int(pool * frac) + 1)
            (rp, col, val), pieces, restarts = bplan.multiply_budget(dA, dA)
            assert [rp.tobytes(), col.tobytes(), val.tobytes()] == ref_bytes, f"budget {frac}"
            assert (rp == ref.row_ptr).all() and (col == ref.col).all()
            assert not (np.abs(val.astype(np.float64) - ref.val) > TOL[dt] * ref.absval).any()
            assert pieces >= (1 if frac == 1.0 else 2) and restarts >= pieces - 1 >= 0
            seen.add(pieces)
            bplan.close()
        assert len(seen) >= 3
        plan.close()


def test_budget_too_small(cuda_available):
    p = pkg()
    A = poisson3d_27pt(12)
    dA = p.DeviceCSR.from_host(A, "cuda")
    plan = p.Plan(pool_limit_bytes=1024)
    with pytest.raises(p.AcspgemmError) as e:
        plan.multiply_budget(dA, dA)
    assert e.value.status == 4                  # OUT_OF_MEMORY: one segment exceeds the budget


def test_budget_empty_and_update_empty(cuda_available):
    """Empty products through the budget and the update paths."""
    from synth import CSR, random_csr
    p = pkg()
    A = CSR(5, 7, np.zeros(6, np.int32), np.zeros(0, np.int32), np.zeros(0))
    B = random_csr(7, 4, 0.5, seed=1)
    dA, dB = p.DeviceCSR.from_host(A, "cuda"), p.DeviceCSR.from_host(B, "cuda")
    plan = p.Plan(pool_limit_bytes=1 << 20)
    (rp, col, val), pieces, restarts = plan.multiply_budget(dA, dB)
    assert (rp == 0).all() and len(col) == 0 and pieces == 1 and restarts == 0
    C = plan.multiply(dA, dB)
    plan.numeric_update(dA, dB, C)
    torch.cuda.synchronize()
    assert (C.row_ptr.cpu().numpy() == 0).all() and C.nnz == 0
