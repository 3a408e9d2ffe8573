"""Numeric re-multiplication with new values on a fixed pattern (SURVEY §8(f)-2,
acspgemm_numeric_update): byte-identical to a fresh multiply of the new values, for every
path (column dictionary, hash table, AC-ESC, Path / Search Merge, dense slices), through
the CUDA graph (re-launched, re-captured on new pointers) and on the default stream."""
import numpy as np
import pytest
import torch

import oracle
from synth import from_coo, poisson3d_27pt, power_law_csr, random_csr, random_rowlen_csr

from test_gpu_parity import TOL, pkg

pytestmark = pytest.mark.gpu


def revalue(M, seed, dt):
    M2 = type(M)(M.rows, M.cols, M.row_ptr, M.col, np.random.default_rng(seed).uniform(-1, 1, M.col.shape[0]))
    return M2.astype(dt)


def same(C1, C2):
    return all(x.cpu().numpy().tobytes() == y.cpu().numpy().tobytes()
               for x, y in ((C1.row_ptr, C2.row_ptr), (C1.col, C2.col), (C1.val, C2.val)))


def cases():
    n_b = 20000
    rng = np.random.default_rng(3)
    giantA = from_coo(3, n_b, [0] * n_b + [1, 1], list(range(n_b)) + [5, 9], rng.uniform(-1, 1, n_b + 2))
    return [
        ("27pt", poisson3d_27pt(12), None),
        ("powerlaw", power_law_csr(2000, 2000, mean_len=12, alpha=1.2, max_len=1200, seed=4),
         power_law_csr(2000, 2000, mean_len=12, alpha=1.2, max_len=2000, seed=14)),
        ("random", random_csr(1500, 1200, 0.01, seed=8), random_csr(1200, 1400, 0.01, seed=9)),
        ("giant", giantA, random_rowlen_csr(n_b, 60000, np.full(n_b, 32), seed=18)),
    ]


@pytest.mark.parametrize("strategy", ["adaptive", "esc", "dict"])
@pytest.mark.parametrize("dt", [np.float64, np.float32])
def test_numeric_update_matches_fresh(dt, strategy, cuda_available):
    p = pkg()
    stream = torch.cuda.Stream()
    for name, A, B in cases():
        B = A if B is None else B
        plan = p.Plan(strategy=strategy)
        with torch.cuda.stream(stream):
            dA, dB = p.DeviceCSR.from_host(A, "cuda", dt), p.DeviceCSR.from_host(B, "cuda", dt)
            C = plan.multiply(dA, dB, stream)
            for it in range(3):                  # capture, relaunch, relaunch
                A2, B2 = revalue(A, 10 + it, dt), revalue(B, 20 + it, dt)
                dA2 = p.DeviceCSR(dA.rows, dA.cols, dA.row_ptr, dA.col, torch.from_numpy(A2.val).cuda())
                dB2 = p.DeviceCSR(dB.rows, dB.cols, dB.row_ptr, dB.col, torch.from_numpy(B2.val).cuda())
                if it < 2:                           # same pointers: capture, then relaunch
                    dA.val.copy_(dA2.val)
                    if dB is not dA:
                        dB.val.copy_(dB2.val)
                    plan.numeric_update(dA, dB, C, stream)
                else:                                # new pointers: re-capture
                    plan.numeric_update(dA2, dB2, C, stream)
                fresh = p.Plan(strategy=strategy).multiply(dA2, dB2, stream)
                stream.synchronize()
                assert same(C, fresh), f"{name} iteration {it}"
                ref = oracle.gustavson(A2, B2)
                err = np.abs(C.val.cpu().numpy().astype(np.float64) - ref.val)
                assert not (err > TOL[dt] * ref.absval).any()
        plan.close()


def test_numeric_update_default_stream_and_errors(cuda_available):
    p = pkg()
    A = poisson3d_27pt(8)
    dA = p.DeviceCSR.from_host(A, "cuda")
    plan = p.Plan()
    with pytest.raises(p.AcspgemmError):
        plan.numeric_update(dA, dA, p.DeviceCSR(0, 0, torch.zeros(1, dtype=torch.int32, device="cuda"),
                                                 torch.zeros(1, dtype=torch.int32, device="cuda"),
                                                 torch.zeros(1, device="cuda", dtype=torch.float64)))
    C = plan.multiply(dA, dA)
    A2 = revalue(A, 5, np.float64)
    dA2 = p.DeviceCSR.from_host(A2, "cuda")
    plan.numeric_update(dA2, dA2, C)             # legacy default stream: uncaptured replay
    torch.cuda.synchronize()
    assert same(C, p.Plan().multiply(dA2, dA2))
    B = random_csr(A.cols, 50, 0.1, seed=2)
    with pytest.raises(p.AcspgemmError):         # other dimensions than the recorded pattern
        plan.numeric_update(dA, p.DeviceCSR.from_host(B, "cuda"), C)
